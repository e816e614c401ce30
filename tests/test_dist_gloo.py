"""Multi-rank host logic of the sharded path, on CPU with the gloo backend (world_size 2).

The local per-rank compute is the oracle here (a test-injected stand-in for the GPU kernels);
what is under test is paper_conf_ppopp_niuljs0022_b200.dist: the product-balanced tile-row
partition, the broadcast of B's arrays, the uneven all-gather and the offset rebasing.
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ppopp_niuljs0022_b200 import dist as tdist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_partition_balances_products():
    from workloads import gen

    for A in (gen.rmat(11), gen.config("C1"), gen.strip_fem(4, 40, 6)):
        w = tdist.tile_row_products(A, A)
        import oracle

        assert w.sum() == oracle.products(A, A)
        for world in (1, 2, 3, 4, 8):
            cuts = tdist.partition_tile_rows(A, A, world)
            assert cuts[0] == 0 and cuts[-1] == w.size and np.all(np.diff(cuts) >= 0) and len(cuts) == world + 1
            loads = [w[cuts[g]:cuts[g + 1]].sum() for g in range(world)]
            # no shard exceeds its fair share by more than one tile row's weight
            assert max(loads) <= w.sum() / world + w.max()


def test_partition_more_ranks_than_rows():
    from workloads import gen

    A = gen.random_sparse(20, 20, 0.3, 1)  # 2 tile rows
    cuts = tdist.partition_tile_rows(A, A, 8)
    assert cuts[0] == 0 and cuts[-1] == 2 and len(cuts) == 9 and np.all(np.diff(cuts) >= 0)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _to_torch(T):
    return {"tile_ptr": torch.from_numpy(T.tile_ptr), "tile_col": torch.from_numpy(T.tile_col),
            "tile_nnz": torch.from_numpy(T.tile_nnz), "row_ptr": torch.from_numpy(T.row_ptr),
            "mask": torch.from_numpy(T.mask.view(np.int16)).view(torch.uint16), "idx": torch.from_numpy(T.idx),
            "val": torch.from_numpy(T.val)}


def _worker(rank, world, port, result_path):
    import sys

    sys.path.insert(0, ROOT)
    import oracle
    from workloads import gen

    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        A = gen.rmat(10)
        # 1) broadcast B's tile arrays from rank 0
        TB = oracle.csr_to_tiles(A)
        meta = (A.m, A.n, TB.num_tiles, TB.nnz) if rank == 0 else None
        arrs = _to_torch(TB) if rank == 0 else None
        meta_r, got = tdist.broadcast_tiles(arrs, meta, 0, torch.device("cpu"))
        ref = _to_torch(TB)
        ok_b = meta_r == (A.m, A.n, TB.num_tiles, TB.nnz, torch.float64) and all(
            torch.equal(got[k].view(torch.int16) if k == "mask" else got[k],
                        ref[k].view(torch.int16) if k == "mask" else ref[k]) for k in tdist.ARRAYS)
        # 2) local shard of C tile rows (oracle stands in for the GPU kernels)
        cuts = tdist.partition_tile_rows(A, A, world)
        I0, I1 = int(cuts[rank]), int(cuts[rank + 1])
        rows = np.arange(16 * I0, min(16 * I1, A.m), dtype=np.int64)
        sub = oracle.spgemm(A, A, fma=True, rows=rows)
        Cl = oracle.csr_to_tiles(gen.CSR(len(rows), A.n, sub.rowptr, sub.col, sub.val))
        piece = dict(m=len(rows), n=A.n, **_to_torch(Cl))
        # 3) count-exact all-gather + rebasing (every rank), and gatherv to rank 0 only
        exp = oracle.expected_tiles(A, A, fma=True)

        def same(res):
            if res is None:
                return False
            m, n, full = res
            ok = (m, n) == (A.m, A.n)
            for k in tdist.ARRAYS:
                a = full[k].view(torch.int16).numpy().view(np.uint16) if k == "mask" else full[k].numpy()
                ok &= bool(np.array_equal(a, getattr(exp, k)))
            return ok

        ok_c = same(tdist.allgatherv_tiles(piece))
        g = tdist.gatherv_tiles(piece, dst=0)
        ok_g = same(g) if rank == 0 else g is None
        with open(f"{result_path}.{rank}", "w") as f:
            f.write(f"{int(ok_b)} {int(ok_c)} {int(ok_g)} {I0} {I1}")
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_broadcast_allgatherv_gatherv(tmp_path, world):
    """World 2 and 3 (gloo, CPU): B broadcast, product-balanced shards, count-exact all-gather on
    every rank and gatherv to rank 0 both reassemble exactly the oracle's C = A^2."""
    port = _free_port()
    mp.spawn(_worker, args=(world, port, str(tmp_path / "res")), nprocs=world, join=True)
    spans = []
    for r in range(world):
        ok_b, ok_c, ok_g, i0, i1 = open(tmp_path / f"res.{r}").read().split()
        assert ok_b == "1", f"broadcast mismatch on rank {r}"
        assert ok_c == "1", f"all-gathered C mismatch on rank {r}"
        assert ok_g == "1", f"gatherv result wrong on rank {r}"
        spans.append((int(i0), int(i1)))
    assert spans[0][0] == 0 and all(spans[g][1] == spans[g + 1][0] for g in range(world - 1))


def test_exact_integer_cuts_match_float_searchsorted():
    """The integer cut rule (first i with pre[i] * world >= g * total) is searchsorted-left of the
    real-valued targets g * total / world."""
    rng = np.random.default_rng(3)
    for _ in range(50):
        w = rng.integers(0, 1000, rng.integers(1, 300))
        for world in (2, 3, 5, 8):
            cuts = tdist.cuts_from_weights(w, world)
            pre = np.concatenate(([0], np.cumsum(w)))
            ref = np.maximum.accumulate(np.concatenate(
                ([0], np.searchsorted(pre, np.arange(1, world) * pre[-1] / world, side="left"), [w.size])))
            assert np.array_equal(cuts, ref)


def _gpu_worker(rank, world, port, result_path):
    """Both ranks on cuda:0 with gloo (one GPU): the library's own sharded product -- device
    partition, row slice, tsg_spgemm -- and the reassembly of CUDA tensors through gloo (staged via
    host), against the oracle."""
    import sys

    sys.path.insert(0, ROOT)
    import oracle
    import paper_conf_ppopp_niuljs0022_b200 as tsg
    from workloads import gen

    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        A = gen.rmat(11)
        T = tsg.csr_to_tiles(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(),
                             torch.from_numpy(A.val).cuda(), (A.m, A.n))
        exp = oracle.expected_tiles(A, A, fma=True)

        def same(res):
            m, n, full = res
            ok = (m, n) == (A.m, A.n)
            for k in tdist.ARRAYS:
                x = full[k].cpu()
                a = x.view(torch.int16).numpy().view(np.uint16) if k == "mask" else x.numpy()
                ok &= bool(np.array_equal(a, getattr(exp, k)))
            return ok

        _, cuts, g = tdist.spgemm_sharded(T, T, reassemble="gather")
        ok_g = same(g) if rank == 0 else g is None
        _, _, a = tdist.spgemm_sharded(T, T, reassemble="all")
        ok_a = same(a)
        meta = (T.m, T.n, T.num_tiles, T.nnz, T.val.dtype) if rank == 0 else None
        meta_r, got = tdist.broadcast_tiles(T.arrays() if rank == 0 else None, meta, 0, torch.device("cuda"))
        ok_b = meta_r == (T.m, T.n, T.num_tiles, T.nnz, torch.float64) and all(
            torch.equal(got[k].view(torch.int16) if k == "mask" else got[k],
                        T.arrays()[k].view(torch.int16) if k == "mask" else T.arrays()[k]) for k in tdist.ARRAYS)
        with open(f"{result_path}.{rank}", "w") as f:
            f.write(f"{int(ok_g)} {int(ok_a)} {int(ok_b)} {int(cuts[rank])} {int(cuts[rank + 1])}")
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
def test_gloo_sharded_spgemm_on_gpu(tmp_path):
    """World 2 on one GPU (gloo): spgemm_sharded with gatherv and with all-gather, and the broadcast
    of a device tile matrix, equal the oracle's C = A^2 / the source arrays."""
    world = 2
    port = _free_port()
    mp.spawn(_gpu_worker, args=(world, port, str(tmp_path / "res")), nprocs=world, join=True)
    spans = []
    for r in range(world):
        ok_g, ok_a, ok_b, i0, i1 = open(tmp_path / f"res.{r}").read().split()
        assert ok_g == "1", f"gathered C wrong on rank {r}"
        assert ok_a == "1", f"all-gathered C wrong on rank {r}"
        assert ok_b == "1", f"broadcast wrong on rank {r}"
        spans.append((int(i0), int(i1)))
    assert spans[0][0] == 0 and spans[0][1] == spans[1][0]
