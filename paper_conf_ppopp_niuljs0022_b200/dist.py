"""Multi-GPU sharding of the TileSpGEMM hot path (no counterpart in the paper,
which runs on one GPU -- P:3760-3766 calls distributed blocking SpGEMM related work).

C tile rows are independent: tile row I of C needs tile row I of A and all of B.  So

1. ``partition_tile_rows``: contiguous tile-row ranges [I_g, I_{g+1}) cut at equal shares of the
   prefix sum of per-tile-row intermediate products (load balance by work, not rows);
2. ``broadcast_tiles``: rank ``src`` holds B; its seven Section-3.2 arrays go to every rank with
   ``torch.distributed.broadcast`` (NCCL over NVLink on the B200 box);
3. each rank runs the local ``tsg.spgemm(slice_rows(A, I_g, I_{g+1}), B)``;
4. ``allgatherv_tiles``: the per-rank C shards are gathered (uneven all_gather, padded) and the
   ``tile_ptr`` / ``tile_nnz`` offsets rebased by the exclusive scan of the per-rank counts
   (``assemble``), giving every rank the full C.

Only collectives and host bookkeeping live here; every arithmetic step of the method runs in
libtsg's kernels.  ``assemble`` and the collectives are device-agnostic (torch tensors), so the
world_size-2 gloo tests in tests/test_dist_gloo.py cover them on CPU.
"""
from __future__ import annotations

import numpy as np

TILE = 16
ARRAYS = ("tile_ptr", "tile_col", "tile_nnz", "row_ptr", "mask", "idx", "val")


def tile_row_products(A, B) -> np.ndarray:
    """Intermediate products per tile row of A*B from host CSR (the partition weights)."""
    rn = np.diff(B.rowptr).astype(np.int64)
    w = rn[A.col.astype(np.int64)] if A.col.size else np.zeros(0, np.int64)
    cs = np.concatenate(([0], np.cumsum(w)))
    row = cs[A.rowptr[1:]] - cs[A.rowptr[:-1]]
    tm = (A.m + TILE - 1) // TILE
    pad = np.zeros(tm * TILE, np.int64)
    pad[:A.m] = row
    return pad.reshape(tm, TILE).sum(axis=1)


def partition_tile_rows(A, B, world: int) -> np.ndarray:
    """cuts[g] .. cuts[g+1] = tile rows of rank g; equal shares of the product prefix sum."""
    w = tile_row_products(A, B)
    tm = w.size
    if world <= 1 or tm == 0:
        return np.array([0, tm] if world <= 1 else [0] * world + [tm], dtype=np.int64)
    pre = np.concatenate(([0], np.cumsum(w)))
    total = pre[-1]
    targets = (np.arange(1, world) * total) / world
    inner = np.searchsorted(pre, targets, side="left")
    cuts = np.concatenate(([0], np.clip(inner, 0, tm), [tm])).astype(np.int64)
    return np.maximum.accumulate(cuts)


def _wire(t):
    """Byte view of 16-bit masks for the wire (neither NCCL nor gloo carries 16-bit integers)."""
    import torch

    return t.view(torch.uint8) if t.dtype in (torch.uint16, torch.int16) else t


def broadcast_tiles(arrays: dict | None, meta: tuple | None, src: int, device, group=None):
    """Broadcast the seven arrays of a tile matrix from ``src``; returns (meta, arrays) everywhere.

    meta = (m, n, num_tiles, nnz) for fp64 values, or (m, n, num_tiles, nnz, dtype) with dtype a
    torch value type (f3).  On non-src ranks pass arrays=None, meta=None; they receive the 4-tuple
    for fp64 and the 5-tuple otherwise.
    """
    import torch
    import torch.distributed as dist

    codes = [torch.float64, torch.float32, torch.float16]
    if meta is not None:
        vals = list(meta[:4]) + [codes.index(meta[4]) if len(meta) > 4 else 0]
    else:
        vals = [0, 0, 0, 0, 0]
    mt = torch.tensor(vals, dtype=torch.int64, device=device)
    dist.broadcast(mt, src, group=group)
    m, n, nt, nnz, dc = (int(x) for x in mt.tolist())
    tm = (m + TILE - 1) // TILE
    shapes = {"tile_ptr": (tm + 1, torch.int64), "tile_col": (nt, torch.int32), "tile_nnz": (nt + 1, torch.int64),
              "row_ptr": (16 * nt, torch.uint8), "mask": (32 * nt, torch.uint8), "idx": (nnz, torch.uint8),
              "val": (nnz, codes[dc])}
    out = {}
    for k in ARRAYS:
        if arrays is not None:
            t = _wire(arrays[k].contiguous())
        else:
            t = torch.empty(shapes[k][0], dtype=shapes[k][1], device=device)
        if t.numel():
            dist.broadcast(t, src, group=group)
        out[k] = t.view(torch.uint16) if k == "mask" else t
    return ((m, n, nt, nnz) if dc == 0 else (m, n, nt, nnz, codes[dc])), out


def allgatherv(t, group=None):
    """Uneven all_gather of a 1-D tensor: returns the list of every rank's tensor."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    n = torch.tensor([_wire(t).numel()], dtype=torch.int64, device=t.device)
    sizes = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(sizes, n, group=group)
    sizes = [int(s.item()) for s in sizes]
    mx = max(sizes) if sizes else 0
    if mx == 0:
        return [t[:0] for _ in range(world)]
    src = _wire(t)
    pad = torch.zeros(mx, dtype=src.dtype, device=t.device)
    pad[:src.numel()] = src
    bufs = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(bufs, pad, group=group)
    res = [b[:s] for b, s in zip(bufs, sizes)]
    if t.dtype != src.dtype:
        res = [r.view(t.dtype) for r in res]
    return res


def assemble(pieces: list, n: int):
    """Concatenate per-rank C shards (contiguous tile-row ranges, in rank order) into one matrix.

    pieces[g] = dict(m=rows, arrays...) with rank-local offsets.  tile_ptr and tile_nnz are
    rebased by the exclusive scan of the per-rank tile and nonzero counts.
    Returns (m, n, arrays) with torch tensors.
    """
    import torch

    tile_base, nnz_base = 0, 0
    out = {k: [] for k in ARRAYS}
    m = 0
    for g, p in enumerate(pieces):
        tp, tz = p["tile_ptr"], p["tile_nnz"]
        nt, nz = int(tp[-1].item()), int(tz[-1].item())
        out["tile_ptr"].append((tp[:-1] if g < len(pieces) - 1 else tp) + tile_base)
        out["tile_nnz"].append((tz[:-1] if g < len(pieces) - 1 else tz) + nnz_base)
        for k in ("tile_col", "row_ptr", "mask", "idx", "val"):
            out[k].append(_wire(p[k]))
        tile_base += nt
        nnz_base += nz
        m += int(p["m"])
    res = {k: torch.cat(v) for k, v in out.items()}
    res["mask"] = res["mask"].view(torch.uint16)
    return m, n, res


def allgatherv_tiles(C, group=None):
    """Gather every rank's C shard (a Tiles object or an arrays dict with key 'm') on all ranks."""
    arrays = C.arrays() if hasattr(C, "arrays") else {k: C[k] for k in ARRAYS}
    m_local = C.m if hasattr(C, "m") else C["m"]
    n = C.n if hasattr(C, "n") else C["n"]
    import torch

    dev = arrays["tile_ptr"].device
    gathered = {k: allgatherv(arrays[k], group) for k in ARRAYS}
    ms = allgatherv(torch.tensor([m_local], dtype=torch.int64, device=dev), group)
    world = len(ms)
    pieces = [dict(m=int(ms[g][0].item()), **{k: gathered[k][g] for k in ARRAYS}) for g in range(world)]
    return assemble(pieces, n)


def spgemm_sharded(A_tiles, B_tiles, A_csr, B_csr, group=None):
    """C = A*B with C tile rows sharded over the process group; returns (local C shard, full C arrays).

    A_tiles/B_tiles must be present on every rank (see broadcast_tiles); A_csr/B_csr (host CSR)
    give the partition weights.
    """
    import torch.distributed as dist

    from . import slice_rows, spgemm

    world, rank = dist.get_world_size(group), dist.get_rank(group)
    cuts = partition_tile_rows(A_csr, B_csr, world)
    shard = slice_rows(A_tiles, int(cuts[rank]), int(cuts[rank + 1]))
    Cl = spgemm(shard, B_tiles)
    return Cl, allgatherv_tiles(Cl, group)
