"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

Bar (BASELINE.json north_star): structure bit-exact (tile_ptr, tile_col, tile_nnz, row_ptr, mask,
idx, CSR row_ptr/col) and fp64 values within |c - c_ref| <= 1e-12 * sum|a*b| per entry.  The
kernels sum in ascending k with FMA (reading A8/A16), so values are also compared bitwise
against the oracle's fma mode (+0 == -0).
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from tests.helpers import assert_values_close, bitwise_equal_values, csr_dense
from workloads import gen

pytestmark = pytest.mark.gpu

ARRAYS = ("tile_ptr", "tile_col", "tile_nnz", "row_ptr", "mask", "idx", "val")


@pytest.fixture(scope="module")
def tsg(cuda_device):
    import paper_conf_ppopp_niuljs0022_b200 as m

    return m


def to_dev(A):
    import torch

    return (torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(), torch.from_numpy(A.val).cuda())


def tiles_of(tsg, A):
    rp, ci, v = to_dev(A)
    return tsg.csr_to_tiles(rp, ci, v, (A.m, A.n))


def host(T) -> dict:
    import torch

    out = {}
    for k in ARRAYS:
        x = getattr(T, k)
        if x.dtype == torch.uint16:
            x = x.view(torch.int16)
        a = x.cpu().numpy()
        out[k] = a.view(np.uint16) if k == "mask" else a
    return out


def assert_tiles_equal(got: dict, ref, values="bitwise", absref=None):
    for k in ARRAYS[:-1]:
        exp = getattr(ref, k)
        assert got[k].shape == exp.shape, (k, got[k].shape, exp.shape)
        assert np.array_equal(got[k], exp), k
    if values == "bitwise":
        assert bitwise_equal_values(got["val"], ref.val)


# ------------------------------------------------------------------------------------------
# a5 / a6: conversion
# ------------------------------------------------------------------------------------------
CONVERT_CASES = [
    lambda: gen.config("C1"),
    lambda: gen.random_sparse(1, 1, 1.0, 1),
    lambda: gen.random_sparse(15, 17, 0.3, 2),
    lambda: gen.random_sparse(17, 100, 0.05, 3),
    lambda: gen.random_sparse(1000, 1000, 0.003, 4, empty_rows=[0, 5, 999]),
    lambda: gen.random_sparse(0, 5, 0.5, 5),
    lambda: gen.random_sparse(40, 40, 0.0, 6),
    lambda: gen.dense_block(48, 33),
    lambda: gen.rmat(11),
    lambda: gen.hub(700, hub_rows=(3,), hub_cols=(5,), density=0.002),
]


@pytest.mark.parametrize("case", range(len(CONVERT_CASES)))
def test_csr_to_tiles_bitwise(tsg, case):
    A = CONVERT_CASES[case]()
    T = tiles_of(tsg, A)
    ref = oracle.csr_to_tiles(A)
    assert (T.m, T.n, T.num_tiles, T.nnz) == (A.m, A.n, ref.num_tiles, ref.nnz)
    assert_tiles_equal(host(T), ref)
    rp, ci, v = tsg.tiles_to_csr(T)
    assert np.array_equal(rp.cpu().numpy(), A.rowptr)
    assert np.array_equal(ci.cpu().numpy(), A.col)
    assert np.array_equal(v.cpu().numpy(), A.val)


def test_csr_to_tiles_host_input_and_validation(tsg):
    A = gen.random_sparse(100, 90, 0.05, 7)
    T = tsg.csr_to_tiles(A.rowptr, A.col, A.val, (A.m, A.n), validate=True)
    assert_tiles_equal(host(T), oracle.csr_to_tiles(A))
    bad = gen.CSR(2, 4, np.array([0, 2, 3]), np.array([2, 1, 0], np.int32), np.ones(3))
    with pytest.raises(tsg.TsgError) as e:
        tsg.csr_to_tiles(bad.rowptr, bad.col, bad.val, (2, 4), validate=True)
    assert e.value.name == "TSG_ERR_UNSORTED"


# ------------------------------------------------------------------------------------------
# a0-a4: spgemm parity
# ------------------------------------------------------------------------------------------
def pair_cases():
    c = []
    A = gen.config("C1")
    c.append(("C1", A, A))
    c.append(("C1-pinned", gen.poisson2d(64, "pinned"), gen.poisson2d(64, "pinned")))
    S = gen.stencil27(10)
    c.append(("stencil27-10", S, S))
    F = gen.strip_fem(8, 30, 6)
    c.append(("strip-fem-8x30", F, F))  # dense-accumulator tiles
    R = gen.rmat(12)
    c.append(("rmat-12", R, R))
    c.append(("rect", gen.random_sparse(37, 50, 0.08, 1), gen.random_sparse(50, 23, 0.1, 2)))
    c.append(("ragged", gen.random_sparse(100, 115, 0.03, 3), gen.random_sparse(115, 81, 0.03, 4)))
    c.append(("single", gen.from_coo(20, 20, [7], [11], [2.5]), gen.from_coo(20, 20, [11], [3], [-4.0])))
    c.append(("empty-A", gen.random_sparse(64, 64, 0.0, 1), gen.random_sparse(64, 64, 0.1, 1)))
    c.append(("no-products", gen.from_coo(32, 32, [0], [1], [1.0]), gen.from_coo(32, 32, [2], [3], [1.0])))
    D = gen.dense_block(64, 64)
    c.append(("dense-64", D, D))
    # 50 dense C tiles per tile row: the row path's dense class walks a row's C tiles in chunks of 32
    c.append(("dense-wide", D, gen.dense_block(64, 800)))
    c.append(("hub", gen.hub(2048, hub_rows=(0, 1000), hub_cols=(0, 7), density=0.004),
              gen.hub(2048, hub_rows=(0, 1000), hub_cols=(0, 7), density=0.004)))
    W = gen.hub(8192, hub_rows=(0, 5000), hub_cols=(), density=0.002)
    c.append(("hub-wide", W, W))  # hub tile rows of ~10^5 candidates: the bitmap-rank step 1
    c.append(("identity", gen.identity(300, 3.0), gen.random_sparse(300, 300, 0.02, 9)))
    c.append(("perm", gen.permutation(257, 1), gen.permutation(257, 2)))
    return c


PAIRS = pair_cases()


@pytest.mark.parametrize("mode", ["default", "per-tile", "rows"])
@pytest.mark.parametrize("name,A,B", PAIRS, ids=[p[0] for p in PAIRS])
def test_spgemm_matches_oracle(tsg, name, A, B, mode):
    """Both pipelines against the oracle: the default dispatch, the per-C-tile pipeline forced with
    path_general, and the row path forced wherever every tile row of A is narrow (path_rows)."""
    TA, TB = tiles_of(tsg, A), tiles_of(tsg, B)
    general = mode == "per-tile"
    C = tsg.spgemm(TA, TB, stats=True, products=True, structural=True, path_general=general,
                   path_rows=mode == "rows")
    ref = oracle.expected_tiles(A, B)
    ref_fma = oracle.expected_tiles(A, B, fma=True)
    got = host(C)
    assert_tiles_equal(got, ref, values=None)
    absref = oracle.csr_to_tiles(_abs_csr(A, B)).val
    assert_values_close(got["val"], ref.val, absref)
    assert bitwise_equal_values(got["val"], ref_fma.val), "ascending-k FMA order must match the oracle bitwise"
    d = oracle.diagnostics(A, B)
    st = C.stats
    assert st["tiles_c"] == d["tiles_c"] == C.num_tiles
    assert st["nnz_c"] == d["nnz_c"]
    assert st["pairs"] == d["pairs"]
    assert st["products"] == d["products"]
    assert st["tiles_dense"] == int((np.diff(ref.tile_nnz) >= tsg.DENSE_NNZ).sum())
    # |C'| of the paper's step 1, empty tiles included, against the oracle's O4
    assert st["tiles_structural"] == d["tiles_structural"] >= st["tiles_c"]
    assert st["path"] == (0 if general else st["path"])
    # CSR assembly of the result
    rp, ci, v = tsg.tiles_to_csr(C)
    O = oracle.spgemm(A, B, fma=True)
    assert np.array_equal(rp.cpu().numpy(), O.rowptr) and np.array_equal(ci.cpu().numpy(), O.col)
    assert bitwise_equal_values(v.cpu().numpy(), O.val)


def _abs_csr(A, B):
    O = oracle.spgemm(A, B)
    return gen.CSR(O.m, O.n, O.rowptr, O.col, O.abs)


@pytest.mark.parametrize("opts", [dict(scan_only=True), dict(list_always=True), dict(dense_threshold=1),
                                  dict(dense_threshold=257), dict(dense_threshold=100), dict(path_general=True),
                                  dict(path_general=True, dense_threshold=1), dict(list_always=True, dense_threshold=1),
                                  dict(path_rows=True), dict(path_rows=True, dense_threshold=1),
                                  dict(path_rows=True, list_always=True),
                                  dict(sort_only=True), dict(sort_only=True, list_always=True),
                                  dict(sort_only=True, scan_only=True), dict(small_stage=True, path_general=True),
                                  dict(small_stage=False, path_general=True)])
def test_modes_give_identical_results(tsg, opts):
    """Step-1 modes and the accumulator threshold change the work split, never the result."""
    for A in (gen.rmat(11), gen.strip_fem(6, 20, 6), gen.config("C1"), gen.stencil27(12),
              gen.hub(8192, hub_rows=(0, 5000), hub_cols=(), density=0.002)):
        T = tiles_of(tsg, A)
        base = host(tsg.spgemm(T, T))
        alt = host(tsg.spgemm(T, T, **opts))
        for k in ARRAYS[:-1]:
            assert np.array_equal(base[k], alt[k]), (opts, k)
        assert bitwise_equal_values(base["val"], alt["val"])


def test_step1_merge_coverage(tsg):
    """Tile rows with <= 32 A tiles take the warp merge, wider rows the expand/sort path; both exact."""
    hub = gen.hub(2048, hub_rows=(0, 1000), hub_cols=(0, 7), density=0.0005)  # 2 tile rows of 128 tiles
    for A, allmerge in ((gen.stencil27(12), True), (gen.strip_fem(6, 20, 6), True), (hub, False)):
        T = tiles_of(tsg, A)
        C = tsg.spgemm(T, T, stats=True)
        nrows = int(np.count_nonzero(np.diff(T.tile_ptr.cpu().numpy())))
        st = C.stats
        if allmerge:
            assert st["step1_merge_rows"] == nrows
        else:
            assert 0 < st["step1_merge_rows"] < nrows
        assert tsg.spgemm(T, T, stats=True, sort_only=True).stats["step1_merge_rows"] == 0
        assert_tiles_equal(host(C), oracle.expected_tiles(A, A, fma=True))


def test_row_path_coverage(tsg):
    """Narrow inputs (every tile row <= 32 A tiles: stencil, FEM, C1) that are small or dense-tiled
    take the per-tile-row pipeline; inputs with a wide tile row take the per-C-tile pipeline;
    path_general forces the latter, path_rows the former where possible.  Both make 2 blocking
    reads once the scratch arena has grown to the problem (a warm-up call).  Same C bit for bit."""
    hub = gen.hub(2048, hub_rows=(0, 1000), hub_cols=(0, 7), density=0.004)
    for A, narrow in ((gen.stencil27(12), True), (gen.strip_fem(6, 20, 6), True), (gen.config("C1"), True),
                      (hub, False)):
        T = tiles_of(tsg, A)
        tsg.spgemm(T, T)  # warm-up: the arena reaches the problem's scratch
        C = tsg.spgemm(T, T, stats=True)
        st = C.stats
        assert st["path"] == (1 if narrow else 0)
        assert st["host_syncs"] == 2
        G = tsg.spgemm(T, T, stats=True, path_general=True)
        assert G.stats["path"] == 0 and G.stats["host_syncs"] == 2
        R = tsg.spgemm(T, T, stats=True, path_rows=True)
        assert R.stats["path"] == (1 if narrow else 0)
        ref = oracle.expected_tiles(A, A, fma=True)
        assert_tiles_equal(host(C), ref)
        assert_tiles_equal(host(G), ref)
        assert_tiles_equal(host(R), ref)


@pytest.mark.parametrize("th", [None, 192])
def test_threshold_boundary_tiles(tsg, th):
    """C tiles with nnz t-1, t, t+1 straddle t_nnz (the default, and the paper's 192)."""
    rng = np.random.default_rng(0)
    t = th or tsg.DENSE_NNZ
    for target in (t - 1, t, t + 1):
        # C = I16 * B where B is one 16x16 tile with `target` nonzeros -> C tile nnz = target
        cells = rng.choice(256, target, replace=False)
        B = gen.from_coo(16, 16, cells // 16, cells % 16, rng.uniform(-1, 1, target))
        I = gen.identity(16, 1.5)
        C = tsg.spgemm(tiles_of(tsg, I), tiles_of(tsg, B), stats=True, dense_threshold=th)
        assert C.stats["tiles_dense"] == (1 if target >= t else 0)
        ref = oracle.expected_tiles(I, B, fma=True)
        assert_tiles_equal(host(C), ref)


def test_nonfinite_and_cancellation(tsg):
    # dense tiles with an Inf and a NaN inside: the dense path must not turn Inf*0 into NaN
    A = gen.dense_block(16, 16)
    A.val[5] = np.inf
    A.val[40] = np.nan
    B = gen.random_sparse(16, 16, 0.5, 3)
    for a, b in ((A, B), (B, A), (A, A)):
        for th in (1, 257):
            C = tsg.spgemm(tiles_of(tsg, a), tiles_of(tsg, b), dense_threshold=th)
            ref = oracle.expected_tiles(a, b, fma=True)
            assert_tiles_equal(host(C), ref)
    # exact cancellation keeps the structural entry (reading A11)
    X = gen.from_coo(16, 16, [0, 0], [0, 1], [1.0, 1.0])
    Y = gen.from_coo(16, 16, [0, 1], [0, 0], [1.0, -1.0])
    C = tsg.spgemm(tiles_of(tsg, X), tiles_of(tsg, Y))
    assert C.nnz == 1 and host(C)["val"][0] == 0.0


def test_determinism_and_symmetry(tsg):
    R = gen.random_sparse(400, 400, 0.01, 4)
    S = (R.to_scipy() + R.to_scipy().T).tocsr()
    S.sort_indices()
    A = gen.CSR(400, 400, S.indptr.astype(np.int64), S.indices.astype(np.int32), S.data.astype(np.float64))
    T = tiles_of(tsg, A)
    c1, c2 = host(tsg.spgemm(T, T)), host(tsg.spgemm(T, T))
    for k in ARRAYS:
        assert np.array_equal(c1[k], c2[k])
    rp, ci, v = tsg.tiles_to_csr(tsg.spgemm(T, T))
    D = csr_dense(400, 400, rp.cpu().numpy(), ci.cpu().numpy(), v.cpu().numpy())
    assert bitwise_equal_values(D, D.T)


def test_chained_output_as_input(tsg):
    """A^3 = (A^2) A with the exported C tiles fed straight back."""
    A = gen.stencil27(8)
    T = tiles_of(tsg, A)
    C2 = tsg.spgemm(T, T)
    C3 = tsg.spgemm(C2, T)
    A2 = oracle.spgemm(A, A, fma=True)
    A2c = gen.CSR(A2.m, A2.n, A2.rowptr, A2.col, A2.val)
    ref = oracle.expected_tiles(A2c, A, fma=True)
    assert_tiles_equal(host(C3), ref)


def test_galerkin_rap_chain(tsg):
    """The paper's AMG motivation for a tile-resident format: the Galerkin coarse
    operator P^T (A P) with a piecewise-constant aggregation prolongator, every product fed the
    previous one's tiles (and P^T from tsg_tiles_transpose) without conversion; equal to the
    oracle's chain in fma mode."""
    A = gen.poisson2d(32)
    n, nc = A.m, A.m // 4
    rows = np.arange(n)
    P = gen.from_coo(n, nc, rows, rows // 4, np.full(n, 0.5), name="aggregation")
    TA, TP = tiles_of(tsg, A), tiles_of(tsg, P)
    AP = tsg.spgemm(TA, TP)
    RAP = tsg.spgemm(tsg.transpose(TP), AP)
    ap = oracle.spgemm(A, P, fma=True)
    APc = gen.CSR(ap.m, ap.n, ap.rowptr, ap.col, ap.val)
    ref = oracle.expected_tiles(oracle.transpose(P), APc, fma=True)
    assert (RAP.m, RAP.n) == (nc, nc)
    assert_tiles_equal(host(RAP), ref)


def test_slice_rows_and_wrap(tsg):
    A = gen.rmat(11)
    T = tiles_of(tsg, A)
    full = oracle.spgemm(A, A, fma=True)
    # (0, 40): a prefix slice shares B's array pointers but not its tile count (rank 0 / block 0)
    for b, e in ((17, 60), (0, 40), (0, T.tile_m)):
        V = tsg.slice_rows(T, b, e)
        CV = tsg.spgemm(V, T)
        rows = np.arange(16 * b, 16 * e)
        sub = oracle.spgemm(A, A, fma=True, rows=rows)
        ref = oracle.csr_to_tiles(gen.CSR(len(rows), A.n, sub.rowptr, sub.col, sub.val))
        assert_tiles_equal(host(CV), ref)
    W = tsg.wrap(A.m, A.n, T.arrays(), keepalive=T)
    CW = tsg.spgemm(W, W)
    assert_tiles_equal(host(CW), oracle.csr_to_tiles(gen.CSR(full.m, full.n, full.rowptr, full.col, full.val)))


def test_launch_counter_advances(tsg):
    A = gen.config("C1")
    T = tiles_of(tsg, A)
    tsg.spgemm(T, T)
    n0 = tsg.kernel_launch_count()
    C = tsg.spgemm(T, T, stats=True)
    assert tsg.kernel_launch_count() - n0 == C.stats["kernel_launches"] > 5
    assert C.stats["host_syncs"] == 2


# ------------------------------------------------------------------------------------------
# full-size configurations, in the launch configuration bench.py times
# ------------------------------------------------------------------------------------------
CLOSED = {  # SURVEY §8(c) closed forms (structure and counts are value independent)
    "C2": dict(nnz_c=254_840_104, products=1_489_355_288),
    "C3": dict(nnz_c=28_850_976, products=562_529_664),
}


@pytest.mark.slow
@pytest.mark.parametrize("cfg,opts", [("C2", {}), ("C2", dict(path_rows=True)), ("C3", {}),
                                      ("C3", dict(path_general=True)), ("C4", {})],
                         ids=["C2", "C2-rows", "C3", "C3-per-tile", "C4"])
def test_full_size_sampled_rows(tsg, cfg, opts):
    import torch

    A = gen.config(cfg)
    T = tiles_of(tsg, A)
    C = tsg.spgemm(T, T, stats=True, products=True, **opts)
    st = C.stats
    if cfg in CLOSED:
        assert st["nnz_c"] == CLOSED[cfg]["nnz_c"] and st["products"] == CLOSED[cfg]["products"]
    else:
        assert st["products"] == oracle.products(A, A)
    # properties at any size (chunked to bound memory): sum of popcounts == nnz, row offsets
    # consistent with the masks, every tile non-empty
    total = 0
    CH = 1 << 24
    for t0 in range(0, C.num_tiles, CH):
        t1 = min(C.num_tiles, t0 + CH)
        mask = C.mask[16 * t0:16 * t1].view(torch.int16).to(torch.int32) & 0xFFFF
        pop = torch.zeros_like(mask)
        for b in range(16):
            pop += (mask >> b) & 1
        total += int(pop.sum())
        pop2 = pop.view(-1, 16)
        rp = C.row_ptr[16 * t0:16 * t1].view(-1, 16).to(torch.int32)
        assert torch.equal(rp, torch.cumsum(pop2, 1) - pop2)
        del mask, pop, pop2, rp
    assert total == C.nnz
    assert bool((C.tile_nnz[1:] > C.tile_nnz[:-1]).all())
    # sampled rows against the oracle, one by one
    rng = np.random.default_rng(11)
    rows = np.unique(np.concatenate([[0, A.m - 1], rng.integers(0, A.m, 300)]))
    sub = oracle.spgemm(A, A, fma=True, rows=rows)
    crp, cci, cv = tsg.tiles_to_csr(C)
    crp_h = crp.cpu().numpy()
    for t, i in enumerate(rows):
        b, e = int(crp_h[i]), int(crp_h[i + 1])
        s0, s1 = int(sub.rowptr[t]), int(sub.rowptr[t + 1])
        assert np.array_equal(cci[b:e].cpu().numpy(), sub.col[s0:s1]), i
        assert bitwise_equal_values(cv[b:e].cpu().numpy(), sub.val[s0:s1]), i


@pytest.mark.slow
def test_full_size_c5_row_block(tsg):
    """C5 (R-MAT scale 22) in bench.py's launch configuration on one GPU: C is computed in four
    tile-row blocks cut at equal product shares (its C is ~144 GB in tile form).  The first block
    is checked: products against the oracle's count, size-independent properties, and sampled rows
    of the block one by one against the oracle."""
    import torch

    from paper_conf_ppopp_niuljs0022_b200 import dist as tdist

    A = gen.config("C5")
    T = tiles_of(tsg, A)
    cuts = tdist.partition_tile_rows(A, A, 4)
    b0, b1 = int(cuts[0]), int(cuts[1])
    Ab = tsg.slice_rows(T, b0, b1)
    C = tsg.spgemm(Ab, T, stats=True, products=True)
    r0, r1 = 16 * b0, min(A.m, 16 * b1)
    assert C.stats["products"] == oracle.products(gen.row_block(A, r0, r1), A)
    pop = torch.zeros((), dtype=torch.int64, device=C.mask.device)
    CH = 1 << 24
    for t0 in range(0, C.num_tiles, CH):
        m = C.mask[16 * t0:16 * min(C.num_tiles, t0 + CH)].view(torch.int16).to(torch.int32) & 0xFFFF
        for b in range(16):
            pop += ((m >> b) & 1).sum()
        del m
    assert int(pop) == C.nnz
    assert bool((C.tile_nnz[1:] > C.tile_nnz[:-1]).all())
    rng = np.random.default_rng(5)
    rows = np.unique(np.concatenate([[r0, r1 - 1], rng.integers(r0, r1, 200)]))
    sub = oracle.spgemm(A, A, fma=True, rows=rows)
    crp, cci, cv = tsg.tiles_to_csr(C)
    crp_h = crp.cpu().numpy()
    for t, i in enumerate(rows):
        b, e = int(crp_h[i - r0]), int(crp_h[i - r0 + 1])
        s0, s1 = int(sub.rowptr[t]), int(sub.rowptr[t + 1])
        assert np.array_equal(cci[b:e].cpu().numpy(), sub.col[s0:s1]), i
        assert bitwise_equal_values(cv[b:e].cpu().numpy(), sub.val[s0:s1]), i


# ------------------------------------------------------------------------------------------
# tile transpose and C = A * A^T (the paper's second workload)
# ------------------------------------------------------------------------------------------
TRANSPOSE_CASES = [
    ("rect", gen.random_sparse(37, 50, 0.08, 1)),
    ("ragged", gen.random_sparse(100, 115, 0.03, 3)),
    ("rmat-11", gen.rmat(11)),
    ("hub", gen.hub(2048, hub_rows=(0, 1000), hub_cols=(0, 7), density=0.004)),
    ("C1", gen.config("C1")),
    ("empty", gen.random_sparse(40, 24, 0.0, 1)),
    ("single", gen.from_coo(20, 33, [7], [31], [2.5])),
]


@pytest.mark.parametrize("name,A", TRANSPOSE_CASES, ids=[c[0] for c in TRANSPOSE_CASES])
def test_transpose_bitwise(tsg, name, A):
    T = tiles_of(tsg, A)
    At = tsg.transpose(T)
    assert (At.m, At.n) == (A.n, A.m)
    assert_tiles_equal(host(At), oracle.csr_to_tiles(oracle.transpose(A)))
    Att = tsg.transpose(At)
    assert_tiles_equal(host(Att), oracle.csr_to_tiles(A))


@pytest.mark.parametrize("name,A", [c for c in TRANSPOSE_CASES if c[0] in ("rect", "ragged", "rmat-11", "C1")],
                         ids=["rect", "ragged", "rmat-11", "C1"])
def test_aat_matches_oracle(tsg, name, A):
    T = tiles_of(tsg, A)
    C = tsg.spgemm(T, tsg.transpose(T), stats=True, products=True)
    At = oracle.transpose(A)
    ref = oracle.expected_tiles(A, At, fma=True)
    assert_tiles_equal(host(C), ref)
    assert C.stats["products"] == oracle.products(A, At)


def test_space_and_peak_memory_reporting(tsg):
    """tile-format bytes vs CSR (Fig 11) and the call's device memory
    (Fig 9) are reported and consistent with the arrays actually held."""
    for A in (gen.config("C1"), gen.strip_fem(6, 20, 6), gen.rmat(11)):
        T = tiles_of(tsg, A)
        C = tsg.spgemm(T, T, stats=True)
        for M in (T, C):
            sp = M.space()
            held = sum(x.numel() * x.element_size() for x in M.arrays().values())
            assert sp["tile_bytes"] == held
            assert sp["csr_bytes"] == 8 * (M.m + 1) + 12 * M.nnz
        st = C.stats
        assert st["bytes_out"] >= C.space()["tile_bytes"]
        assert st["bytes_scratch"] > 0


# ------------------------------------------------------------------------------------------
# f3: precision variants (fp32, and the paper's half-in / single-out setup)
# ------------------------------------------------------------------------------------------
def _typed(A, np_dtype):
    return gen.CSR(A.m, A.n, A.rowptr, A.col, A.val.astype(np_dtype), A.name)


PREC_CASES = [("C1", gen.config("C1")), ("stencil27-10", gen.stencil27(10)),
              ("strip-fem-8x30", gen.strip_fem(8, 30, 6)), ("rmat-12", gen.rmat(12)),
              ("dense-64", gen.dense_block(64, 64)),
              ("hub", gen.hub(2048, hub_rows=(0, 1000), hub_cols=(0, 7), density=0.004))]


@pytest.mark.parametrize("np_dtype", [np.float32, np.float16], ids=["f32", "f16"])
@pytest.mark.parametrize("name,A", PREC_CASES, ids=[c[0] for c in PREC_CASES])
def test_precision_variants_match_oracle(tsg, name, A, np_dtype):
    """Steps 1-2 are value-free; step 3 in fp32 (fp16 inputs widened exactly) sums in ascending k
    with fmaf, so the result equals the oracle's single-precision fma loop bit for bit."""
    At = _typed(A, np_dtype)
    T = tiles_of(tsg, At)
    assert T.dtype == np.dtype(np_dtype).name and T.val.dtype == getattr(__import__("torch"), T.dtype)
    assert np.array_equal(T.val.cpu().numpy(), oracle.csr_to_tiles(A).val.astype(np_dtype))
    for th in (None, 1):  # default classes, and every tile through the dense accumulator
        C = tsg.spgemm(T, T, stats=True, dense_threshold=th)
        assert C.dtype == "float32"
        ref = oracle.expected_tiles(At, At, fma=True, prec="f32")
        got = host(C)
        assert_tiles_equal(got, ref, values=None)
        assert got["val"].dtype == np.float32
        assert bitwise_equal_values(got["val"].astype(np.float64), ref.val.astype(np.float64)), (name, th)
    # the other entry points keep the value type
    rp, ci, v = tsg.tiles_to_csr(C)
    O = oracle.spgemm(At, At, fma=True, prec="f32")
    assert v.dtype == __import__("torch").float32 and np.array_equal(v.cpu().numpy(), O.val)
    TT = tsg.transpose(T)
    assert TT.dtype == T.dtype
    ref_t = oracle.csr_to_tiles(oracle.transpose(A))
    assert np.array_equal(TT.val.cpu().numpy(), ref_t.val.astype(np_dtype))
    h = T.copy_to_host()
    assert h["val"].dtype == np.dtype(np_dtype) and np.array_equal(h["val"], T.val.cpu().numpy())


def test_mixed_precision_inputs_rejected(tsg):
    A = gen.config("C1")
    T64, T32 = tiles_of(tsg, A), tiles_of(tsg, _typed(A, np.float32))
    with pytest.raises(tsg.TsgError) as e:
        tsg.spgemm(T64, T32)
    assert e.value.name == "TSG_ERR_INVALID_ARG"


def test_copy_to_host_async_pipeline(tsg):
    """tsg_tiles_copy_to_host_async on a second stream, overlapping the next block's SpGEMM (the
    bench's e2e leg): every block's host copy equals the oracle's tiles of that row block."""
    import torch

    A = gen.stencil27(12)
    T = tiles_of(tsg, A)
    cuts = [0, T.tile_m // 3, 2 * T.tile_m // 3, T.tile_m]
    ref = oracle.expected_tiles(A, A, fma=True)
    s_copy = torch.cuda.Stream()
    outs, live = [], []
    for b0, b1 in zip(cuts[:-1], cuts[1:]):
        C = tsg.spgemm(tsg.slice_rows(T, b0, b1), T)
        ev = torch.cuda.Event()
        ev.record()
        s_copy.wait_event(ev)
        bufs = {k: torch.empty(v.numel(), dtype=torch.int16 if v.dtype == torch.uint16 else v.dtype, pin_memory=True)
                for k, v in C.arrays().items()}
        C.copy_to_host(bufs, stream=s_copy, blocking=False)
        outs.append(bufs)
        live.append(C)
    s_copy.synchronize()
    # stitch the blocks back together and compare with C = A^2
    tp = [0]
    cols, nnzs, rps, masks, idxs, vals = [], [], [], [], [], []
    base_t = base_z = 0
    for h in outs:
        tp.extend((h["tile_ptr"][1:].numpy() + base_t).tolist())
        nnzs.append(h["tile_nnz"][:-1].numpy() + base_z)
        base_t += int(h["tile_ptr"][-1])
        base_z += int(h["tile_nnz"][-1])
        cols.append(h["tile_col"].numpy())
        rps.append(h["row_ptr"].numpy())
        masks.append(h["mask"].numpy().view(np.uint16))
        idxs.append(h["idx"].numpy())
        vals.append(h["val"].numpy())
    nnzs.append(np.array([base_z]))
    assert np.array_equal(np.array(tp), ref.tile_ptr)
    assert np.array_equal(np.concatenate(cols), ref.tile_col)
    assert np.array_equal(np.concatenate(nnzs), ref.tile_nnz)
    assert np.array_equal(np.concatenate(rps), ref.row_ptr)
    assert np.array_equal(np.concatenate(masks), ref.mask)
    assert np.array_equal(np.concatenate(idxs), ref.idx)
    assert bitwise_equal_values(np.concatenate(vals), ref.val)


@pytest.mark.parametrize("chunk", [0, 1, 3])
def test_work_distribution_gives_identical_results(tsg, chunk):
    """Per-C-tile pipeline work distribution: static grid-stride (0) or the work queue with 1 or 3
    groups per request (small test inputs otherwise take the static path)."""
    cases = (gen.stencil27(12), gen.strip_fem(6, 20, 6), gen.rmat(11),
             gen.hub(8192, hub_rows=(0, 5000), hub_cols=(), density=0.002))
    for A in cases:
        T = tiles_of(tsg, A)
        b = host(tsg.spgemm(T, T))
        got = host(tsg.spgemm(T, T, path_general=True, queue_chunk=chunk))
        for k in ARRAYS[:-1]:
            assert np.array_equal(got[k], b[k]), (chunk, k)
        assert bitwise_equal_values(got["val"], b["val"])
    A = cases[0]
    assert_tiles_equal(host(tsg.spgemm(tiles_of(tsg, A), tiles_of(tsg, A), path_general=True, queue_chunk=chunk)),
                       oracle.expected_tiles(A, A, fma=True))


def test_unknown_flags_rejected(tsg):
    import ctypes as C

    from paper_conf_ppopp_niuljs0022_b200 import _lib

    A = gen.config("C1")
    T = tiles_of(tsg, A)
    out = C.c_void_p()
    for bad in (0x80, 0x8000, 1 << 29):  # 0x80: the removed tensor-core flag
        rc = _lib.load().tsg_spgemm(T.ptr, T.ptr, bad, None, None, C.byref(out), None)
        assert rc == 1 and out.value is None


def test_host_input_dtypes_and_row_ptr_validation(tsg):
    """Host CSR given as torch CPU tensors of the wrong integer width is converted; an
    unsupported value type raises; TSG_VALIDATE rejects row_ptr[m] != nnz with INVALID_ARG."""
    import torch

    A = gen.random_sparse(100, 90, 0.05, 7)
    ref = oracle.csr_to_tiles(A)
    T = tsg.csr_to_tiles(torch.from_numpy(A.rowptr).to(torch.int32), torch.from_numpy(A.col).to(torch.int64),
                         torch.from_numpy(A.val), (A.m, A.n))
    assert_tiles_equal(host(T), ref)
    with pytest.raises(TypeError):
        tsg.csr_to_tiles(A.rowptr, A.col, A.val.astype(np.complex128), (A.m, A.n))
    with pytest.raises(ValueError):
        tsg.csr_to_tiles(A.rowptr[:-1], A.col, A.val, (A.m, A.n))
    # device input: row_ptr[m] larger than the column array
    rp = torch.from_numpy(A.rowptr).cuda()
    rp[-1] += 5
    with pytest.raises(tsg.TsgError) as e:
        tsg.csr_to_tiles(rp, torch.from_numpy(A.col).cuda(), torch.from_numpy(A.val).cuda(), (A.m, A.n),
                         validate=True)
    assert e.value.name == "TSG_ERR_INVALID_ARG"


def test_free_is_ordered_on_the_producing_stream(tsg):
    """A handle made under a side stream frees its arrays on that stream: dropping C
    right after the call must not let the next allocation overwrite it while step 3 still runs."""
    import torch

    A = gen.stencil27(16)
    T = tiles_of(tsg, A)
    ref = host(tsg.spgemm(T, T))
    s = torch.cuda.Stream()
    for _ in range(3):
        with torch.cuda.stream(s):
            C = tsg.spgemm(T, T)
            assert C.handle.stream == s.cuda_stream
            del C
            D = tsg.spgemm(T, T)
        s.synchronize()
        got = host(D)
        for k in ARRAYS:
            assert np.array_equal(got[k], ref[k]), k


def test_concurrent_calls_on_two_streams(tsg):
    """Programmatic dependent launch keeps stream order: two host threads issuing calls on their own
    streams at the same time (every kernel launched with programmatic serialization, each waiting
    on its predecessor in its own stream) give the sequential results bit for bit, on both
    pipelines and on a hypersparse input."""
    import threading

    import torch

    cases = [(gen.stencil27(14), {}), (gen.strip_fem(6, 20, 6), {}), (gen.rmat(11), {}),
             (gen.stencil27(12), dict(path_general=True))]
    tiles = [(tiles_of(tsg, A), o) for A, o in cases]
    refs = [host(tsg.spgemm(T, T, **o)) for T, o in tiles]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    out = [[None] * len(tiles) for _ in streams]

    def worker(w):
        with torch.cuda.stream(streams[w]):
            for rep in range(3):
                for i in range(len(tiles)):
                    j = (i + w) % len(tiles)  # the two threads run different cases at once
                    T, o = tiles[j]
                    out[w][j] = tsg.spgemm(T, T, stream=streams[w], **o)
        streams[w].synchronize()

    th = [threading.Thread(target=worker, args=(w,)) for w in range(2)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    for w in range(2):
        for j, ref in enumerate(refs):
            got = host(out[w][j])
            for k in ARRAYS[:-1]:
                assert np.array_equal(got[k], ref[k]), (w, j, k)
            assert bitwise_equal_values(got["val"], ref["val"]), (w, j)


def test_device_partition_matches_host_rule(tsg):
    """tsg_partition_tile_rows: per-tile-row products counted on the device and
    cut at equal shares equal the host-CSR rule, and the total equals the oracle's products."""
    from paper_conf_ppopp_niuljs0022_b200 import dist as tdist

    for A in (gen.config("C1"), gen.rmat(11), gen.strip_fem(4, 40, 6), gen.stencil27(12),
              gen.random_sparse(100, 115, 0.03, 3)):
        B = gen.random_sparse(A.n, 77, 0.05, 5) if A.m != A.n else A
        TA, TB = tiles_of(tsg, A), tiles_of(tsg, B)
        for parts in (1, 2, 3, 8, 31):
            cuts, prods = tsg.partition_tile_rows(TA, TB, parts)
            assert np.array_equal(cuts, tdist.partition_tile_rows(A, B, parts)), (A.name, parts)
            assert prods == oracle.products(A, B)


def _high_word_view(tsg, T, bias=1 << 32):
    """A handle over T's arrays whose nonzero offsets carry +bias (tile_nnz + bias) against idx /
    val base pointers moved back by bias elements: every A/B value address the kernels form is
    unchanged, but only if they keep the offsets' high words."""
    import ctypes as C

    import torch

    from paper_conf_ppopp_niuljs0022_b200 import _lib

    tz = (T.tile_nnz + bias).contiguous()
    v = _lib.TilesView()
    v.m, v.n, v.tile_m, v.tile_n, v.num_tiles, v.nnz = T.m, T.n, T.tile_m, T.tile_n, T.num_tiles, T.nnz
    v.tile_ptr, v.tile_col, v.tile_nnz = T.tile_ptr.data_ptr(), T.tile_col.data_ptr(), tz.data_ptr()
    v.row_ptr, v.mask = T.row_ptr.data_ptr(), T.mask.data_ptr()
    v.idx = T.idx.data_ptr() - bias
    v.val = T.val.data_ptr() - bias * T.val.element_size()
    v.dtype = {torch.float64: 0, torch.float32: 1, torch.float16: 2}[T.val.dtype]
    out = C.c_void_p()
    _lib.check(_lib.load().tsg_tiles_wrap(C.byref(v), None, C.byref(out)))

    class View:  # only the handle: its idx/val base pointers are not allocations torch could wrap
        pass

    V = View()
    V.handle = tsg._Handle(out.value)
    V.ptr = C.c_void_p(out.value)
    V.keep = (T, tz)
    return V


@pytest.mark.parametrize("opts", [{}, dict(path_general=True), dict(path_rows=True), dict(dense_threshold=1)],
                         ids=["default", "per-tile", "rows", "dense"])
def test_int64_offsets_with_high_words(tsg, opts):
    """64-bit offset paths (T4): inputs whose nonzero offsets exceed 2^32 and C's offsets biased by
    2^32 inside the call (TSG_DEBUG_HIGH_OFFSETS) give the same C bit for bit."""
    for A in (gen.config("C1"), gen.rmat(11), gen.strip_fem(6, 20, 6), gen.stencil27(10),
              gen.hub(2048, hub_rows=(0, 1000), hub_cols=(0, 7), density=0.004)):
        T = tiles_of(tsg, A)
        ref = host(tsg.spgemm(T, T, **opts))
        V = _high_word_view(tsg, T)
        got = host(tsg.spgemm(V, V, debug_high_offsets=True, **opts))
        for k in ARRAYS[:-1]:
            assert np.array_equal(got[k], ref[k]), (A.name, k)
        assert bitwise_equal_values(got["val"], ref["val"])


def test_scratch_retry_after_arena_release(tsg):
    """Step 1's scratch is sized from the cached arena before the candidate total is known; after
    tsg_workspace_release the first call overflows it, is redone with a grown arena (one extra
    blocking read), and returns the same C; the next call makes 2 reads."""
    for A in (gen.rmat(12), gen.stencil27(16)):
        T = tiles_of(tsg, A)
        ref = host(tsg.spgemm(T, T))
        tsg.workspace_release()
        C1 = tsg.spgemm(T, T, stats=True)
        C2 = tsg.spgemm(T, T, stats=True)
        assert C1.stats["host_syncs"] >= 3 and C2.stats["host_syncs"] == 2
        for C in (C1, C2):
            got = host(C)
            for k in ARRAYS:
                assert np.array_equal(got[k], ref[k]), k


# ------------------------------------------------------------------------------------------
# seeded random sweep: shapes, densities and tile structures mixed, every pipeline and class
# ------------------------------------------------------------------------------------------
def _sweep_case(rng, kind):
    """One (A, B) pair of a given structure kind, sizes drawn so that tails are ragged."""
    m, k, n = (int(x) for x in rng.integers(1, 200, 3))
    dens = float(rng.choice([0.002, 0.02, 0.1, 0.45]))
    if kind == 0:  # uniform random
        return gen.random_sparse(m, k, dens, int(rng.integers(1 << 30))), gen.random_sparse(k, n, dens, int(rng.integers(1 << 30)))
    if kind == 1:  # banded (stencil-like tiles), random bandwidth
        bw = int(rng.integers(0, 20))
        def band(r, c):
            rows, cols = [], []
            for i in range(r):
                lo, hi = max(0, i - bw), min(c, i + bw + 1)
                rows += [i] * max(0, hi - lo)
                cols += list(range(lo, hi))
            return gen.from_coo(r, c, rows, cols, rng.uniform(-1, 1, len(rows)))
        return band(m, k), band(k, n)
    if kind == 2:  # random dense 16x16 blocks on a sparse background (dense, medium and small C tiles)
        def blocks(r, c):
            coo_r, coo_c = [], []
            for bi in range(-(-r // 16)):
                for bj in range(-(-c // 16)):
                    p = rng.random()
                    if p < 0.25:  # full block
                        for i in range(bi * 16, min(r, bi * 16 + 16)):
                            for j in range(bj * 16, min(c, bj * 16 + 16)):
                                coo_r.append(i)
                                coo_c.append(j)
                    elif p < 0.5:  # a few entries
                        for _ in range(int(rng.integers(1, 6))):
                            coo_r.append(int(rng.integers(bi * 16, min(r, bi * 16 + 16))))
                            coo_c.append(int(rng.integers(bj * 16, min(c, bj * 16 + 16))))
            return gen.from_coo(r, c, coo_r, coo_c, rng.uniform(-1, 1, len(coo_r)))
        return blocks(m, k), blocks(k, n)
    # kind 3: wide tile rows (> 32 A tiles in a tile row: the per-C-tile pipeline's hub classes)
    kw = int(rng.integers(33 * 16, 70 * 16))
    A = gen.random_sparse(max(m, 17), kw, dens / 4, int(rng.integers(1 << 30)))
    rows = np.concatenate([np.repeat(np.arange(A.m), np.diff(A.rowptr)), np.zeros(kw, np.int64)])
    cols = np.concatenate([A.col, np.arange(kw)])
    A = gen.from_coo(A.m, kw, rows, cols, rng.uniform(-1, 1, len(rows)))  # row 0 dense: its tile row is wide
    return A, gen.random_sparse(kw, n, dens, int(rng.integers(1 << 30)))


@pytest.mark.parametrize("seed", range(24))
def test_random_parity_sweep(tsg, seed):
    """Seeded random (A, B) of four structure kinds with ragged shapes; every pipeline (default,
    per-C-tile, per-tile-row), every tile through the dense class, and fp32: all bit for bit
    against the oracle's fma mode."""
    rng = np.random.default_rng(7000 + seed)
    for kind in range(4):
        A, B = _sweep_case(rng, kind)
        TA, TB = tiles_of(tsg, A), tiles_of(tsg, B)
        ref = oracle.expected_tiles(A, B, fma=True)
        for opts in ({}, dict(path_general=True), dict(path_rows=True), dict(path_rows=True, dense_threshold=1),
                     dict(path_general=True, dense_threshold=1), dict(path_general=True, small_stage=True),
                     dict(list_always=True, sort_only=True)):
            assert_tiles_equal(host(tsg.spgemm(TA, TB, **opts)), ref), (seed, kind, opts)
        A32, B32 = _typed(A, np.float32), _typed(B, np.float32)
        got = host(tsg.spgemm(tiles_of(tsg, A32), tiles_of(tsg, B32)))
        ref32 = oracle.expected_tiles(A32, B32, fma=True, prec="f32")
        assert_tiles_equal(got, ref32, values=None)
        assert bitwise_equal_values(got["val"].astype(np.float64), ref32.val.astype(np.float64)), (seed, kind)
