"""Pins for the CPU oracle (oracle/) against things other than itself.

Each test fixes the oracle to the paper or to mathematics: values the paper prints (Fig 5),
closed forms (tridiagonal, 5-point Laplacian, Kronecker stencils), brute force on tiny inputs
(dense matmul, exact integer arithmetic), special cases (identity, permutations), invariants
(symmetry, row sums, nnz <= products) and a second independent formulation (Algorithm 2's
bit-mask OR vs the tiled Gustavson result; a numpy tiler vs the C tiler).
"""
from __future__ import annotations

import os

import numpy as np
import pytest
import scipy.sparse as sp

import oracle
from tests.helpers import (GOLDEN, assert_values_close, bitwise_equal_values, csr_dense, csr_pattern,
                           read_golden_kv, read_golden_matrix)
from workloads import gen

pytestmark = pytest.mark.filterwarnings("ignore::RuntimeWarning")


# ------------------------------------------------------------------------------------------
# O1 Gustavson vs brute force
# ------------------------------------------------------------------------------------------
SHAPES = [(1, 1, 1), (5, 7, 3), (15, 16, 17), (16, 16, 16), (17, 33, 15), (40, 25, 31), (64, 64, 64)]


@pytest.mark.parametrize("m,k,n", SHAPES)
@pytest.mark.parametrize("density", [0.05, 0.3])
def test_gustavson_matches_dense_bruteforce(m, k, n, density):
    A = gen.random_sparse(m, k, density, seed=m * 7 + k, empty_rows=[0] if m > 2 else [], empty_cols=[1] if k > 2 else [])
    B = gen.random_sparse(k, n, density, seed=n * 11 + k + 1)
    C = oracle.spgemm(A, B)
    DA, DB = csr_dense(m, k, A.rowptr, A.col, A.val), csr_dense(k, n, B.rowptr, B.col, B.val)
    PA, PB = csr_pattern(m, k, A.rowptr, A.col), csr_pattern(k, n, B.rowptr, B.col)
    # structure = pairs (i,j) with at least one product (structural, no cancellation: reading A11)
    S = (PA.astype(np.int64) @ PB.astype(np.int64)) > 0
    assert np.array_equal(csr_pattern(m, n, C.rowptr, C.col), S)
    # sorted unique columns per row
    for i in range(m):
        seg = C.col[C.rowptr[i]:C.rowptr[i + 1]]
        assert np.all(np.diff(seg) > 0)
    dense = DA @ DB
    absb = np.abs(DA) @ np.abs(DB)
    rows = np.repeat(np.arange(m), np.diff(C.rowptr))
    assert_values_close(C.val, dense[rows, C.col], np.maximum(absb[rows, C.col], 1e-300) * 4)
    # the abs-sum bound returned by the oracle is sum |a*b|
    assert np.allclose(C.abs, absb[rows, C.col], rtol=1e-12, atol=0)


@pytest.mark.parametrize("fma", [False, True])
def test_gustavson_exact_on_integers(fma):
    """Small-integer values make every product and sum exact: compare to Python ints exactly."""
    rng = np.random.default_rng(5)
    A = gen.random_sparse(23, 19, 0.25, seed=1)
    B = gen.random_sparse(19, 29, 0.25, seed=2)
    A.val = rng.integers(-9, 10, A.nnz).astype(np.float64)
    B.val = rng.integers(-9, 10, B.nnz).astype(np.float64)
    C = oracle.spgemm(A, B, fma=fma)
    # pure-Python triple loop (tiny case)
    ref = {}
    for i in range(A.m):
        for p in range(A.rowptr[i], A.rowptr[i + 1]):
            kk = int(A.col[p])
            for q in range(B.rowptr[kk], B.rowptr[kk + 1]):
                key = (i, int(B.col[q]))
                ref[key] = ref.get(key, 0) + int(A.val[p]) * int(B.val[q])
    got = {}
    for i in range(C.m):
        for p in range(C.rowptr[i], C.rowptr[i + 1]):
            got[(i, int(C.col[p]))] = C.val[p]
    assert set(got) == set(ref)
    assert all(got[k] == ref[k] for k in ref)


def test_gustavson_keeps_cancelled_zeros_and_propagates_nonfinite():
    # row 0 of A = [1, 1]; B = [[1],[ -1]] -> C[0,0] = 0 exactly, must be kept (reading A11)
    A = gen.from_coo(2, 2, [0, 0, 1], [0, 1, 1], [1.0, 1.0, np.inf])
    B = gen.from_coo(2, 2, [0, 1, 1], [0, 0, 1], [1.0, -1.0, 2.0])
    C = oracle.spgemm(A, B)
    D = {(i, int(C.col[p])): C.val[p] for i in range(2) for p in range(C.rowptr[i], C.rowptr[i + 1])}
    assert D[(0, 0)] == 0.0 and (0, 0) in D
    assert D[(0, 1)] == 2.0
    assert D[(1, 0)] == -np.inf and D[(1, 1)] == np.inf
    # NaN input propagates
    A2 = gen.from_coo(1, 1, [0], [0], [np.nan])
    C2 = oracle.spgemm(A2, A2)
    assert np.isnan(C2.val[0])


# ------------------------------------------------------------------------------------------
# closed forms
# ------------------------------------------------------------------------------------------
def test_tridiagonal_square_closed_form():
    T = gen.tridiagonal(8)
    C = oracle.spgemm(T, T)
    expect = read_golden_matrix("tridiag8_squared.txt")
    got = csr_dense(8, 8, C.rowptr, C.col, C.val)
    assert np.array_equal(got, expect)
    assert C.nnz == np.count_nonzero(expect)


def test_poisson2d_square_closed_form():
    g = 64
    A = gen.poisson2d(g, "pinned")
    gold = read_golden_kv("c1_poisson2d64.txt")
    assert A.nnz == gold["nnz_a"]
    C = oracle.spgemm(A, A)
    assert C.nnz == gold["nnz_c"] == sum((g - abs(dx)) * (g - abs(dy)) for dx in range(-2, 3) for dy in range(-2, 3)
                                         if abs(dx) + abs(dy) <= 2)
    assert oracle.products(A, A) == gold["products"] == 4 * 9 + 248 * 16 + 3844 * 25
    rows = np.repeat(np.arange(A.m), np.diff(C.rowptr))
    cols = C.col.astype(np.int64)
    x0, y0, x1, y1 = rows % g, rows // g, cols % g, cols // g
    dx, dy = np.abs(x0 - x1), np.abs(y0 - y1)
    # degree of the middle grid point = number of in-grid axis neighbours
    deg = ((x0 > 0).astype(int) + (x0 < g - 1) + (y0 > 0) + (y0 < g - 1))
    expect = np.select([(dx == 0) & (dy == 0), dx + dy == 1, (dx == 1) & (dy == 1), dx + dy == 2],
                       [16.0 + deg, -8.0, 2.0, 1.0], np.nan)
    assert np.array_equal(C.val, expect)
    assert set(np.unique(C.val[(dx == 0) & (dy == 0)])) == {18.0, 19.0, 20.0}


@pytest.mark.parametrize("g", [3, 5, 7])
def test_stencil27_kronecker_closed_form(g):
    """A = T⊗T⊗T with T = tridiag(1,1,1): A^2 = T^2⊗T^2⊗T^2 (scipy kron, not the oracle)."""
    A = gen.stencil27(g, "ones")
    T = sp.diags([np.ones(g - 1), np.ones(g), np.ones(g - 1)], [-1, 0, 1]).tocsr()
    KA = sp.kron(sp.kron(T, T), T).tocsr()
    assert np.array_equal(A.to_scipy().toarray(), KA.toarray())
    T2 = (T @ T).tocsr()
    KC = sp.kron(sp.kron(T2, T2), T2).toarray()
    C = oracle.spgemm(A, A)
    assert np.array_equal(csr_dense(A.m, A.n, C.rowptr, C.col, C.val), KC)
    assert A.nnz == (3 * g - 2) ** 3 and C.nnz == (5 * g - 6) ** 3
    assert oracle.products(A, A) == (9 * g - 10) ** 3


def test_c2_c3_counts_at_full_size_closed_forms():
    """The closed forms of SURVEY §8(c) at the configurations' own sizes (counts only)."""
    g = 128
    assert (3 * g - 2) ** 3 == 55_742_968 and (5 * g - 6) ** 3 == 254_840_104 and (9 * g - 10) ** 3 == 1_489_355_288
    A = gen.strip_fem(32, 1042, 6, "ones")
    assert A.nnz == 3124 * 94 * 36 == 10_571_616


@pytest.mark.parametrize("nx,ny,b", [(4, 5, 2), (3, 7, 6)])
def test_strip_fem_kronecker_closed_form(nx, ny, b):
    """A = (T_ny ⊗ T_nx) ⊗ J_b  =>  A^2 = b * (T_ny^2 ⊗ T_nx^2) ⊗ J_b."""
    A = gen.strip_fem(nx, ny, b, "ones")
    Ty = sp.diags([np.ones(ny - 1), np.ones(ny), np.ones(ny - 1)], [-1, 0, 1])
    Tx = sp.diags([np.ones(nx - 1), np.ones(nx), np.ones(nx - 1)], [-1, 0, 1])
    J = sp.csr_matrix(np.ones((b, b)))
    KA = sp.kron(sp.kron(Ty, Tx), J).toarray()
    assert np.array_equal(A.to_scipy().toarray(), KA)
    KC = b * sp.kron(sp.kron(Ty @ Ty, Tx @ Tx), J).toarray()
    C = oracle.spgemm(A, A)
    assert np.array_equal(csr_dense(A.m, A.n, C.rowptr, C.col, C.val), KC)


def test_identity_and_permutations():
    A = gen.random_sparse(50, 50, 0.1, seed=9)
    I = gen.identity(50)
    for C in (oracle.spgemm(I, A), oracle.spgemm(A, I)):
        assert np.array_equal(C.rowptr, A.rowptr) and np.array_equal(C.col, A.col)
        assert np.array_equal(C.val, A.val)
    P, Q = gen.permutation(50, 1), gen.permutation(50, 2)
    pP = P.col.astype(np.int64)
    PA = oracle.spgemm(P, A)
    DA = csr_dense(50, 50, A.rowptr, A.col, A.val)
    assert np.array_equal(csr_dense(50, 50, PA.rowptr, PA.col, PA.val), DA[pP])  # row permutation
    PQ = oracle.spgemm(P, Q)
    assert np.array_equal(PQ.col.astype(np.int64), Q.col.astype(np.int64)[pP])  # composed permutation


# ------------------------------------------------------------------------------------------
# invariants
# ------------------------------------------------------------------------------------------
@pytest.mark.parametrize("fma", [False, True])
def test_symmetric_square_is_bitwise_symmetric(fma):
    """Ascending-k summation (reading A8) makes A^2 of a symmetric A bitwise symmetric."""
    R = gen.random_sparse(120, 120, 0.04, seed=4)
    S = (R.to_scipy() + R.to_scipy().T).tocsr()
    S.sort_indices()
    A = gen.CSR(120, 120, S.indptr.astype(np.int64), S.indices.astype(np.int32), S.data.astype(np.float64))
    C = oracle.spgemm(A, A, fma=fma)
    D = csr_dense(120, 120, C.rowptr, C.col, C.val)
    assert bitwise_equal_values(D, D.T)


def test_row_sums_and_counts_invariants():
    A = gen.rmat(9, values="random")
    B = gen.random_sparse(A.n, 300, 0.02, seed=8)
    C = oracle.spgemm(A, B)
    ones = np.ones(B.n)
    lhs = oracle.spmv(gen.CSR(C.m, C.n, C.rowptr, C.col, C.val), ones)
    rhs = oracle.spmv(A, oracle.spmv(B, ones))
    bound = oracle.spmv(gen.CSR(C.m, C.n, C.rowptr, C.col, C.abs), ones)
    assert np.all(np.abs(lhs - rhs) <= 1e-12 * bound + 1e-300)
    assert C.nnz <= oracle.products(A, B)


def test_row_subset_matches_full():
    A = gen.config("C1")
    full = oracle.spgemm(A, A)
    rows = np.array([4095, 0, 17, 2048], dtype=np.int64)
    sub = oracle.spgemm(A, A, rows=rows)
    for t, i in enumerate(rows):
        a, b = full.rowptr[i], full.rowptr[i + 1]
        c, d = sub.rowptr[t], sub.rowptr[t + 1]
        assert np.array_equal(full.col[a:b], sub.col[c:d]) and np.array_equal(full.val[a:b], sub.val[c:d])


# ------------------------------------------------------------------------------------------
# O2/O3 tile format
# ------------------------------------------------------------------------------------------
def numpy_tiler(A):
    """A second, independent construction of Section 3.2's arrays via a lexicographic sort."""
    rows = np.repeat(np.arange(A.m, dtype=np.int64), np.diff(A.rowptr))
    cols = A.col.astype(np.int64)
    I, J, r, c = rows // 16, cols // 16, rows % 16, cols % 16
    order = np.lexsort((c, r, J, I))
    I, J, r, c, v = I[order], J[order], r[order], c[order], A.val[order]
    key = I * ((A.n + 15) // 16 + 1) + J
    first = np.concatenate(([True], key[1:] != key[:-1])) if key.size else np.zeros(0, bool)
    tI, tJ = I[first], J[first]
    tm = (A.m + 15) // 16
    tile_ptr = np.zeros(tm + 1, np.int64)
    np.add.at(tile_ptr, tI + 1, 1)
    tile_ptr = np.cumsum(tile_ptr)
    tid = np.cumsum(first) - 1
    nt = int(first.sum())
    tile_nnz = np.zeros(nt + 1, np.int64)
    np.add.at(tile_nnz, tid + 1, 1)
    tile_nnz = np.cumsum(tile_nnz)
    mask = np.zeros(16 * nt, np.uint16)
    np.bitwise_or.at(mask, tid * 16 + r, (1 << c).astype(np.uint16))
    cnt = np.zeros(16 * nt, np.int64)
    np.add.at(cnt, tid * 16 + r, 1)
    row_ptr = (np.cumsum(cnt.reshape(nt, 16), axis=1) - cnt.reshape(nt, 16)).reshape(-1).astype(np.uint8)
    return tile_ptr, tJ.astype(np.int32), tile_nnz, row_ptr, mask, ((r << 4) | c).astype(np.uint8), v


@pytest.mark.parametrize("m,n,d", [(1, 1, 1.0), (15, 17, 0.3), (16, 16, 1.0), (17, 100, 0.05), (100, 33, 0.1),
                                   (0, 5, 0.5), (1000, 1000, 0.003)])
def test_tiles_match_numpy_tiler_and_roundtrip(m, n, d):
    A = gen.random_sparse(m, n, d, seed=m + n)
    T = oracle.csr_to_tiles(A)
    ref = numpy_tiler(A)
    for got, exp in zip((T.tile_ptr, T.tile_col, T.tile_nnz, T.row_ptr, T.mask, T.idx, T.val), ref):
        assert np.array_equal(got, exp)
    R = oracle.tiles_to_csr(T)
    assert np.array_equal(R.rowptr, A.rowptr) and np.array_equal(R.col, A.col) and np.array_equal(R.val, A.val)


def check_tile_invariants(T):
    assert np.all(np.diff(T.tile_nnz) > 0), "no empty tiles"
    for I in range(T.tm):
        seg = T.tile_col[T.tile_ptr[I]:T.tile_ptr[I + 1]]
        assert np.all(np.diff(seg) > 0)
    pop = np.array([bin(x).count("1") for x in T.mask], dtype=np.int64).reshape(-1, 16)
    assert pop.sum() == T.nnz
    rp = T.row_ptr.reshape(-1, 16).astype(np.int64)
    assert np.array_equal(rp, np.cumsum(pop, axis=1) - pop)
    for t in range(T.num_tiles):
        seg = T.idx[T.tile_nnz[t]:T.tile_nnz[t + 1]]
        assert np.all(np.diff(seg.astype(np.int64)) > 0), "idx strictly increasing (reading A1)"


def test_tile_invariants_on_configs():
    for A in (gen.config("C1"), gen.rmat(10), gen.dense_block(40, 40)):
        check_tile_invariants(oracle.csr_to_tiles(A))


# ------------------------------------------------------------------------------------------
# O4: step 1 / step 2 formulations against each other and against the paper
# ------------------------------------------------------------------------------------------
def test_fig5_mask_or():
    """PAPER Fig 5: c10 = b10 | b12 = 1100 | 1010 = 1110."""
    with open(os.path.join(GOLDEN, "fig5_mask.txt")) as f:
        line = [ln for ln in f if ln.strip() and not ln.startswith("#")][0].split()
    acols = [int(x) for x in line[0].split(",")]
    bits = lambda s: [i for i, ch in enumerate(s) if ch == "1"]
    b0, b2, expect = bits(line[1]), bits(line[2]), bits(line[3])
    A = gen.from_coo(16, 16, [0] * len(acols), acols, [1.0] * len(acols))
    B = gen.from_coo(16, 16, [0] * len(b0) + [2] * len(b2), b0 + b2, [1.0] * (len(b0) + len(b2)))
    TA, TB = oracle.csr_to_tiles(A), oracle.csr_to_tiles(B)
    mask, nnz, matched, contrib = oracle.step2_masks(TA, TB, [0], [0])
    assert [c for c in range(16) if mask[0] >> c & 1] == expect
    assert nnz[0] == len(expect) and matched[0] == 1 and contrib[0] == 1


def test_c1_step_statistics_match_survey():
    gold = read_golden_kv("c1_poisson2d64.txt")
    A = gen.config("C1")
    d = oracle.diagnostics(A, A)
    assert oracle.csr_to_tiles(A).num_tiles == gold["tiles_a"]
    for k in ("tiles_structural", "tiles_c", "pairs_structural", "pairs", "nnz_c", "products"):
        assert d[k] == gold[k], k


@pytest.mark.parametrize("maker", [lambda: gen.config("C1"), lambda: gen.rmat(10), lambda: gen.random_sparse(300, 300, 0.01, 2),
                                   lambda: gen.strip_fem(4, 30, 6)])
def test_algorithm2_masks_equal_tiled_gustavson(maker):
    """Two formulations: Alg 2's OR over matched pairs == O2(O1(A,A)); empty C' tiles <-> nnz 0."""
    A = maker()
    d = oracle.diagnostics(A, A)
    T = oracle.expected_tiles(A, A)
    nonempty = d["cp_nnz"] > 0
    assert nonempty.sum() == T.num_tiles and d["tiles_c"] <= d["tiles_structural"]
    cI = np.repeat(np.arange(T.tm), np.diff(d["cp_ptr"]))[nonempty]
    cJ = d["cp_col"][nonempty]
    assert np.array_equal(cI, T.tile_rows()) and np.array_equal(cJ, T.tile_col)
    assert np.array_equal(d["cp_mask"].reshape(-1, 16)[nonempty].reshape(-1), T.mask)
    assert np.array_equal(d["cp_nnz"][nonempty], np.diff(T.tile_nnz))
    assert d["nnz_c"] == T.nnz


def test_dense_tiles_are_dense_class():
    A = gen.dense_block(32, 32)
    d = oracle.diagnostics(A, A)
    assert d["tiles_c"] == 4 and d["tiles_dense"] == 4 and d["products"] == 32 ** 3


# ------------------------------------------------------------------------------------------
# generators (input side, deterministic)
# ------------------------------------------------------------------------------------------
def test_generators_deterministic_and_chunk_independent():
    a = gen.rmat(11, chunk=1000)
    b = gen.rmat(11, chunk=1 << 22)
    assert np.array_equal(a.rowptr, b.rowptr) and np.array_equal(a.col, b.col) and np.array_equal(a.val, b.val)
    v = gen.position_values(np.array([3]), np.array([5]))
    assert -1.0 <= v[0] < 1.0
    A = gen.config("C1")
    assert A.nnz == 5 * 4096 - 4 * 64
    for i in range(A.m):
        seg = A.col[A.rowptr[i]:A.rowptr[i + 1]]
        assert np.all(np.diff(seg) > 0)


# ------------------------------------------------------------------------------------------
# O6: CSR transpose (for the paper's second workload C = A*A^T)
# ------------------------------------------------------------------------------------------
@pytest.mark.parametrize("m,n,d", [(1, 1, 1.0), (37, 50, 0.1), (64, 17, 0.3), (100, 100, 0.02), (20, 30, 0.0)])
def test_transpose_matches_dense_and_scipy(m, n, d):
    A = gen.random_sparse(m, n, d, seed=m * 7 + n)
    T = oracle.transpose(A)
    assert (T.m, T.n) == (n, m)
    # dense brute force: every entry lands at the mirrored position
    assert np.array_equal(csr_dense(T.m, T.n, T.rowptr, T.col, T.val), csr_dense(A.m, A.n, A.rowptr, A.col, A.val).T)
    # rows of A^T list columns ascending, values carried bitwise (scipy's CSC view of A)
    S = sp.csr_matrix((A.val, A.col, A.rowptr), shape=(m, n)).tocsc()
    S.sort_indices()
    assert np.array_equal(T.rowptr, S.indptr) and np.array_equal(T.col, S.indices)
    assert bitwise_equal_values(T.val, S.data)


def test_transpose_involution_and_product_rule():
    A = gen.random_sparse(48, 40, 0.08, seed=5)
    B = gen.random_sparse(40, 33, 0.1, seed=6)
    TT = oracle.transpose(oracle.transpose(A))
    assert np.array_equal(TT.rowptr, A.rowptr) and np.array_equal(TT.col, A.col) and bitwise_equal_values(TT.val, A.val)
    # (A B)^T = B^T A^T: same structure; values agree within the sum-of-|products| bound
    L = oracle.transpose(oracle.spgemm(A, B))
    R = oracle.spgemm(oracle.transpose(B), oracle.transpose(A))
    assert np.array_equal(L.rowptr, R.rowptr) and np.array_equal(L.col, R.col)
    assert np.allclose(L.val, R.val, rtol=0, atol=1e-12 * np.abs(R.val).max())
    # A A^T is symmetric for any A (structure exactly; values are the same dot products)
    Q = oracle.spgemm(A, oracle.transpose(A))
    QT = oracle.transpose(Q)
    assert np.array_equal(Q.rowptr, QT.rowptr) and np.array_equal(Q.col, QT.col)
    assert np.allclose(Q.val, QT.val, rtol=0, atol=1e-12 * np.abs(Q.val).max())


# ------------------------------------------------------------------------------------------
# O1 in single precision (the paper's Section 4.7 half-in / single-out setup,
# P:3143-3152)
# ------------------------------------------------------------------------------------------
def _with_values(A, vals):
    return gen.CSR(A.m, A.n, A.rowptr, A.col, vals, A.name)


def test_gustavson_f32_exact_on_small_integers():
    """Integers with |sums| < 2^24 are exact in fp32: the f32 loop must equal the fp64 one."""
    rng = np.random.default_rng(5)
    for m, k, n in ((16, 16, 16), (40, 33, 27)):
        A = gen.random_sparse(m, k, 0.3, seed=m + 1)
        B = gen.random_sparse(k, n, 0.3, seed=n + 2)
        A = _with_values(A, rng.integers(-8, 9, A.col.size).astype(np.float64))
        B = _with_values(B, rng.integers(-8, 9, B.col.size).astype(np.float64))
        for fma in (False, True):
            C64 = oracle.spgemm(A, B, fma=fma)
            C32 = oracle.spgemm(A, B, fma=fma, prec="f32")
            assert C32.val.dtype == np.float32
            assert np.array_equal(C32.rowptr, C64.rowptr) and np.array_equal(C32.col, C64.col)
            assert np.array_equal(C32.val.astype(np.float64), C64.val)


def test_gustavson_f32_within_rounding_bound():
    """Random values: |c32 - c64| <= (k+1) * 2^-24 * sum|a*b| per entry (k = products of the
    entry; standard recursive-summation bound with fp32 inputs rounded first), and the fp64
    products of the fp32-rounded inputs bound the abs sums."""
    A = gen.random_sparse(70, 60, 0.15, seed=3)
    B = gen.random_sparse(60, 50, 0.15, seed=4)
    A32 = _with_values(A, A.val.astype(np.float32).astype(np.float64))
    B32 = _with_values(B, B.val.astype(np.float32).astype(np.float64))
    ref = oracle.spgemm(A32, B32)  # exact-input fp64 reference
    ones = oracle.spgemm(_with_values(A, np.ones_like(A.val)), _with_values(B, np.ones_like(B.val)))
    k = ones.val  # products per entry
    for fma in (False, True):
        C32 = oracle.spgemm(A, B, fma=fma, prec="f32")
        assert np.array_equal(C32.col, ref.col)
        err = np.abs(C32.val.astype(np.float64) - ref.val)
        assert np.all(err <= (k + 1) * 2.0 ** -24 * ref.abs + 1e-300)
        assert np.allclose(C32.abs, ref.abs, rtol=1e-15, atol=0)


def test_gustavson_f16_inputs_widen_exactly():
    """Half inputs are widened to fp32 exactly: the f32 product of float16 values
    equals the f32 product of the same values given as float32, and matches the dense fp64 product
    of the half-rounded matrices within the fp32 bound."""
    A = gen.random_sparse(33, 35, 0.2, seed=8)
    B = gen.random_sparse(35, 31, 0.2, seed=9)
    Ah, Bh = _with_values(A, A.val.astype(np.float16)), _with_values(B, B.val.astype(np.float16))
    Af, Bf = _with_values(A, Ah.val.astype(np.float32)), _with_values(B, Bh.val.astype(np.float32))
    Ch = oracle.spgemm(Ah, Bh, fma=True, prec="f32")
    Cf = oracle.spgemm(Af, Bf, fma=True, prec="f32")
    assert np.array_equal(Ch.val, Cf.val)
    D = csr_dense(A.m, A.n, A.rowptr, A.col, Ah.val.astype(np.float64)) @ \
        csr_dense(B.m, B.n, B.rowptr, B.col, Bh.val.astype(np.float64))
    got = csr_dense(Ch.m, Ch.n, Ch.rowptr, Ch.col, Ch.val.astype(np.float64))
    absd = np.abs(csr_dense(A.m, A.n, A.rowptr, A.col, Ah.val.astype(np.float64))) @ \
        np.abs(csr_dense(B.m, B.n, B.rowptr, B.col, Bh.val.astype(np.float64)))
    assert np.all(np.abs(got - D) <= (A.n + 1) * 2.0 ** -24 * absd + 1e-300)


def test_gustavson_f32_accumulates_in_single_precision():
    """Closed form: products 1, 2^-24, 2^-24 summed in ascending k.  In fp32 each 1 + 2^-24 is a
    tie and rounds to even (1.0), so the result is exactly 1.0; in fp64 it is 1 + 2^-23.  A loop
    that accumulated in fp64 and rounded once would give 1 + 2^-23 (the next float above 1)."""
    e = 2.0 ** -12
    A = gen.from_coo(1, 3, [0, 0, 0], [0, 1, 2], [1.0, e, e])
    B = gen.from_coo(3, 1, [0, 1, 2], [0, 0, 0], [1.0, e, e])
    for fma in (False, True):
        assert oracle.spgemm(A, B, fma=fma, prec="f32").val.tolist() == [1.0]
        assert oracle.spgemm(A, B, fma=fma).val.tolist() == [1.0 + 2.0 ** -23]


def test_oracle_omp_equals_single_thread():
    """oracle_omp: the row list split over OpenMP threads, each chunk by the same C
    loop, gives the single-threaded result bit for bit -- including more threads than rows."""
    for A, rows in ((gen.config("C1"), np.arange(4096, dtype=np.int64)),
                    (gen.rmat(9), np.arange(0, 512, 3, dtype=np.int64)),
                    (gen.config("C1"), np.arange(5, dtype=np.int64))):
        ref = oracle.spgemm(A, A, rows=rows)
        for th in (2, 3, 8):
            got = oracle.spgemm(A, A, rows=rows, threads=th)
            assert np.array_equal(got.rowptr, ref.rowptr) and np.array_equal(got.col, ref.col)
            assert np.array_equal(got.val.view(np.int64), ref.val.view(np.int64))
            assert np.array_equal(got.abs, ref.abs)
    full = oracle.spgemm(gen.config("C1"), gen.config("C1"), threads=4)
    assert full.nnz == 51972  # the C1 closed form


def test_c1_golden_statistics_reproduce_with_scipy():
    """The C1 tile statistics in tests/golden/c1_poisson2d64.txt (first measured in the survey) are
    regenerated by a committed scipy-only script that shares nothing with oracle/ or the CUDA path."""
    import subprocess
    import sys

    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, os.path.join(root, "scripts", "golden_c1_stats.py"), "--check"],
                         capture_output=True, text=True, cwd=root)
    assert out.returncode == 0, out.stdout + out.stderr


def test_spmv_pinned_by_dense_matvec():
    """orc_spmv (the helper of the row-sum invariant) against the dense matrix-vector product: exact
    on small integers (no rounding), and within the recursive-summation bound on random values;
    empty rows give 0."""
    rng = np.random.default_rng(11)
    for m, n, dens in ((1, 1, 1.0), (7, 5, 0.5), (40, 33, 0.1), (64, 64, 0.0)):
        A = gen.random_sparse(m, n, dens, seed=m + n)
        D = csr_dense(m, n, A.rowptr, A.col, A.val)
        # integer values: every partial sum is exact in fp64
        Ai = gen.CSR(m, n, A.rowptr, A.col, np.round(A.val * 8.0))
        xi = rng.integers(-5, 6, n).astype(np.float64)
        Di = csr_dense(m, n, Ai.rowptr, Ai.col, Ai.val)
        assert np.array_equal(oracle.spmv(Ai, xi), Di @ xi)
        x = rng.uniform(-1, 1, n)
        y = oracle.spmv(A, x)
        bound = np.abs(D) @ np.abs(x) * (n * np.finfo(np.float64).eps) + 1e-300
        assert np.all(np.abs(y - D @ x) <= bound)
        assert np.all(y[np.diff(A.rowptr) == 0] == 0.0)
