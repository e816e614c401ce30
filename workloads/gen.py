"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This module produces sparse matrices in CSR form (numpy arrays) and nothing else: it
holds none of TileSpGEMM's arithmetic (no tiling, no products, no masks).  Both the
oracle (``oracle/``) and the GPU path (``paper_conf_ppopp_niuljs0022_b200``) consume
what it returns; neither is imported here.

Workloads (the recipe restated in DESIGN.md §3):

* ``C1 poisson2d-64``   5-point Laplacian on a 64x64 grid, lexicographic (x fastest).
* ``C2 stencil27-128``  27-point box stencil on a 128^3 grid (A = T⊗T⊗T, T = tridiag(1,1,1)).
* ``C3 strip-fem-pwtk`` A = (T_1042 ⊗ T_32) ⊗ J_6: 9-point node stencil with dense 6x6 blocks.
* ``C4 rmat-20``        R-MAT scale 20, edge factor 16, (a,b,c,d) = (.45,.15,.15,.25).
* ``C5 rmat-22``        same at scale 22.

Values default to uniform[-1,1) drawn from ``splitmix64(seed_v ^ (i<<32 | j))`` so a value
depends only on its position (i, j), never on generation order.
The paper's own workloads are SuiteSparse matrices (§4.1); these are
synthetic stand-ins with the same structural classes (stencil/FEM, banded, power-law).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

U64 = np.uint64
_M64 = (1 << 64) - 1


@dataclass
class CSR:
    """A CSR matrix on the host: sorted, unique column indices per row."""

    m: int
    n: int
    rowptr: np.ndarray  # int64 [m+1]
    col: np.ndarray  # int32 [nnz]
    val: np.ndarray  # float64 [nnz]
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.rowptr[-1])

    def to_scipy(self):
        import scipy.sparse as sp

        return sp.csr_matrix((self.val, self.col, self.rowptr), shape=(self.m, self.n))

    def transpose(self) -> "CSR":
        """Structural transpose (a data-layout helper for the AAᵀ workload, not method arithmetic)."""
        order = np.lexsort((np.repeat(np.arange(self.m, dtype=np.int64), np.diff(self.rowptr)), self.col))
        rows = np.repeat(np.arange(self.m, dtype=np.int64), np.diff(self.rowptr))[order]
        cols = self.col[order].astype(np.int64)
        counts = np.bincount(cols, minlength=self.n)
        rp = np.zeros(self.n + 1, dtype=np.int64)
        np.cumsum(counts, out=rp[1:])
        return CSR(self.n, self.m, rp, rows.astype(np.int32), self.val[order].copy(), self.name + "^T")


# --------------------------------------------------------------------------------------
# counter-based random numbers
# --------------------------------------------------------------------------------------
def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vectorised splitmix64 finaliser over uint64 arrays (wrapping arithmetic)."""
    z = (x.astype(U64) + U64(0x9E3779B97F4A7C15))
    z = (z ^ (z >> U64(30))) * U64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> U64(27))) * U64(0x94D049BB133111EB)
    return z ^ (z >> U64(31))


def u01(z: np.ndarray) -> np.ndarray:
    """Top 53 bits of a uint64 as a double in [0, 1)."""
    return (z >> U64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


def position_values(rows: np.ndarray, cols: np.ndarray, seed_v: int = 2) -> np.ndarray:
    """uniform[-1,1) value for entry (i, j): splitmix64(seed_v ^ (i<<32 | j))."""
    key = (rows.astype(U64) << U64(32)) | cols.astype(U64)
    with np.errstate(over="ignore"):
        z = splitmix64(key ^ U64(seed_v))
    return 2.0 * u01(z) - 1.0


def _sorted_unique(key: np.ndarray) -> np.ndarray:
    """Sorted distinct values (np.sort + neighbour test; np.unique is hash-based and slow here)."""
    if key.size == 0:
        return key
    s = np.sort(key, kind="stable")
    keep = np.empty(s.size, dtype=bool)
    keep[0] = True
    np.not_equal(s[1:], s[:-1], out=keep[1:])
    return s[keep]


def _finish(m, n, rows, cols, values, seed_v, name, const=None):
    """Build a CSR from row-major-sorted (rows, cols) arrays."""
    rows = np.asarray(rows, dtype=np.int64)
    cols = np.asarray(cols, dtype=np.int64)
    counts = np.bincount(rows, minlength=m) if rows.size else np.zeros(m, dtype=np.int64)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    if values == "random":
        val = position_values(rows, cols, seed_v)
    elif values == "ones":
        val = np.ones(rows.size, dtype=np.float64)
    elif values == "const":
        val = const(rows, cols)
    else:
        raise ValueError(values)
    return CSR(m, n, rp, cols.astype(np.int32), np.ascontiguousarray(val, dtype=np.float64), name)


def _grid_stencil(dims, values="random", seed_v=2, name="", const=None):
    """Kronecker-structured stencil.

    ``dims`` lists (size, offsets) from the slowest to the fastest index; the matrix
    index is the mixed-radix number of the grid coordinate.  Offsets are enumerated
    lexicographically so the emitted columns of each row are already ascending.
    """
    sizes = [d[0] for d in dims]
    n = int(np.prod(sizes))
    strides = [int(np.prod(sizes[i + 1:])) for i in range(len(sizes))]
    idx = np.arange(n, dtype=np.int64)
    coords = [(idx // strides[i]) % sizes[i] for i in range(len(sizes))]
    combos = np.array(np.meshgrid(*[np.asarray(d[1]) for d in dims], indexing="ij")).reshape(len(dims), -1).T
    cols = np.empty((n, combos.shape[0]), dtype=np.int64)
    ok = np.ones((n, combos.shape[0]), dtype=bool)
    for t, off in enumerate(combos):
        c = np.zeros(n, dtype=np.int64)
        v = np.ones(n, dtype=bool)
        for i in range(len(sizes)):
            ci = coords[i] + int(off[i])
            v &= (ci >= 0) & (ci < sizes[i])
            c += ci * strides[i]
        cols[:, t] = c
        ok[:, t] = v
    rows = np.broadcast_to(idx[:, None], cols.shape)[ok]
    return _finish(n, n, rows, cols[ok], values, seed_v, name, const)


# --------------------------------------------------------------------------------------
# the five configurations
# --------------------------------------------------------------------------------------
def poisson2d(g: int = 64, values: str = "random", seed_v: int = 2) -> CSR:
    """C1: 5-point Laplacian on a g x g grid.  values='pinned' gives 4 on the diagonal, -1 off it."""
    if values == "pinned":
        return _grid_stencil([(g, [-1, 0, 1]), (g, [-1, 0, 1])], "const", seed_v, f"poisson2d-{g}",
                             const=lambda r, c: np.where(r == c, 4.0, -1.0))._drop_corners(g)
    return _grid_stencil([(g, [-1, 0, 1]), (g, [-1, 0, 1])], values, seed_v, f"poisson2d-{g}")._drop_corners(g)


def _drop_corners(self: CSR, g: int) -> CSR:
    """Keep only |dx|+|dy| <= 1 entries of a 3x3 box stencil (turns 9-point into 5-point)."""
    rows = np.repeat(np.arange(self.m, dtype=np.int64), np.diff(self.rowptr))
    cols = self.col.astype(np.int64)
    dy = np.abs(rows // g - cols // g)
    dx = np.abs(rows % g - cols % g)
    keep = (dx + dy) <= 1
    rows, cols, val = rows[keep], cols[keep], self.val[keep]
    counts = np.bincount(rows, minlength=self.m)
    rp = np.zeros(self.m + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    return CSR(self.m, self.n, rp, cols.astype(np.int32), val, self.name)


CSR._drop_corners = _drop_corners


def stencil27(g: int = 128, values: str = "random", seed_v: int = 2) -> CSR:
    """C2: 27-point box stencil on a g^3 grid; values='ones' gives A = T⊗T⊗T, T = tridiag(1,1,1)."""
    t = (g, [-1, 0, 1])
    return _grid_stencil([t, t, t], values, seed_v, f"stencil27-{g}")


def strip_fem(nx: int = 32, ny: int = 1042, b: int = 6, values: str = "random", seed_v: int = 2) -> CSR:
    """C3: A = (T_ny ⊗ T_nx) ⊗ J_b, dof fastest, then x, then y (n = ny*nx*b)."""
    return _grid_stencil([(ny, [-1, 0, 1]), (nx, [-1, 0, 1]), (b, list(range(-(b - 1), b)))],
                         values, seed_v, f"strip-fem-{nx}x{ny}x{b}")


def rmat(scale: int, edge_factor: int = 16, abcd=(0.45, 0.15, 0.15, 0.25), seed: int = 1,
         values: str = "random", seed_v: int = 2, chunk: int = 1 << 22) -> CSR:
    """C4/C5: R-MAT graph (directed, no noise, no permutation); duplicates merged, self-loops kept.

    Edge e draws z_w = splitmix64(S ^ (e*16 + w)) for w = 0, 1, ...; level l uses the 16-bit
    field (z_{l//4} >> 16*(l%4)) & 0xFFFF as a uniform in [0,1) (resolution 2^-16), so the
    graph does not depend on the chunk size.  S = splitmix64(seed).
    """
    n = 1 << scale
    ne = edge_factor * n
    a, b, c, _ = abcd
    t1, t2, t3 = (int(round(x * 65536)) for x in (a, a + b, a + b + c))
    S = splitmix64(np.array([seed], dtype=U64))[0]
    keys = []
    with np.errstate(over="ignore"):
        for e0 in range(0, ne, chunk):
            e = np.arange(e0, min(ne, e0 + chunk), dtype=U64)
            r = np.zeros(e.size, dtype=np.int64)
            q = np.zeros(e.size, dtype=np.int64)
            base = e * U64(16)
            z = None
            for lev in range(scale):
                if lev % 4 == 0:
                    z = splitmix64((base + U64(lev // 4)) ^ S)
                x = ((z >> U64(16 * (lev % 4))) & U64(0xFFFF)).astype(np.int64)
                rb = (x >= t2).astype(np.int64)
                cb = (((x >= t1) & (x < t2)) | (x >= t3)).astype(np.int64)
                r = (r << 1) | rb
                q = (q << 1) | cb
            keys.append(r * n + q)
    key = _sorted_unique(np.concatenate(keys))
    rows = key // n
    cols = key % n
    return _finish(n, n, rows, cols, values, seed_v, f"rmat-{scale}")


CONFIGS = {
    "C1": ("poisson2d-64", lambda values="random": poisson2d(64, values)),
    "C2": ("stencil27-128", lambda values="random": stencil27(128, values)),
    "C3": ("strip-fem-pwtk", lambda values="random": strip_fem(32, 1042, 6, values)),
    "C4": ("rmat-20", lambda values="random": rmat(20, values=values)),
    "C5": ("rmat-22", lambda values="random": rmat(22, values=values)),
}


def config(name: str, values: str = "random") -> CSR:
    """Build one of C1..C5 by name."""
    label, fn = CONFIGS[name]
    A = fn(values)
    A.name = label
    return A


# --------------------------------------------------------------------------------------
# test families (edge cases, tiny brute-force inputs)
# --------------------------------------------------------------------------------------
def random_sparse(m: int, n: int, density: float, seed: int = 0, values: str = "random",
                  seed_v: int = 2, empty_rows=(), empty_cols=()) -> CSR:
    """Uniform random structure: each (i, j) present with probability ``density``."""
    rng = np.random.default_rng(seed)
    total = m * n
    k = rng.binomial(total, density) if total else 0
    flat = _sorted_unique(rng.integers(0, max(total, 1), size=k, dtype=np.int64)) if k else np.zeros(0, np.int64)
    rows = flat // max(n, 1)
    cols = flat % max(n, 1)
    keep = ~np.isin(rows, np.asarray(empty_rows, dtype=np.int64)) & ~np.isin(cols, np.asarray(empty_cols, dtype=np.int64))
    return _finish(m, n, rows[keep], cols[keep], values, seed_v, f"random-{m}x{n}-{density}")


def identity(n: int, scale: float = 1.0) -> CSR:
    idx = np.arange(n, dtype=np.int64)
    return _finish(n, n, idx, idx, "const", 0, f"I{n}", const=lambda r, c: np.full(r.size, scale))


def permutation(n: int, seed: int = 0) -> CSR:
    """P with P[i, p[i]] = 1 for a seeded random permutation p."""
    p = np.random.default_rng(seed).permutation(n).astype(np.int64)
    return _finish(n, n, np.arange(n, dtype=np.int64), p, "ones", 0, f"P{n}")


def tridiagonal(n: int, lo: float = -1.0, d: float = 2.0, up: float = -1.0) -> CSR:
    i = np.arange(n, dtype=np.int64)
    rows = np.concatenate([i[1:], i, i[:-1]])
    cols = np.concatenate([i[:-1], i, i[1:]])
    vals = np.concatenate([np.full(n - 1, lo), np.full(n, d), np.full(n - 1, up)])
    order = np.lexsort((cols, rows))
    rows, cols, vals = rows[order], cols[order], vals[order]
    return _finish(n, n, rows, cols, "const", 0, f"tridiag{n}", const=lambda r, c: vals)


def dense_block(m: int, n: int, values: str = "random", seed_v: int = 2) -> CSR:
    """Every entry present (full 256-nnz tiles)."""
    rows = np.repeat(np.arange(m, dtype=np.int64), n)
    cols = np.tile(np.arange(n, dtype=np.int64), m)
    return _finish(m, n, rows, cols, values, seed_v, f"dense{m}x{n}")


def from_coo(m: int, n: int, rows, cols, vals, name: str = "coo") -> CSR:
    """Sort and merge (keep first) a COO triple list into CSR -- used for hand-made edge cases."""
    rows = np.asarray(rows, dtype=np.int64)
    cols = np.asarray(cols, dtype=np.int64)
    vals = np.asarray(vals, dtype=np.float64)
    key = rows * n + cols
    key_u, first = np.unique(key, return_index=True)
    return _finish(m, n, key_u // n, key_u % n, "const", 0, name, const=lambda r, c: vals[first])


def hub(n: int, hub_rows=(0,), hub_cols=(0,), density: float = 0.001, seed: int = 3, values: str = "random") -> CSR:
    """Random background plus fully dense hub rows and columns (load-balance stress)."""
    base = random_sparse(n, n, density, seed, values)
    rows = [np.repeat(np.arange(n, dtype=np.int64), np.diff(base.rowptr))]
    cols = [base.col.astype(np.int64)]
    for h in hub_rows:
        rows.append(np.full(n, h, dtype=np.int64))
        cols.append(np.arange(n, dtype=np.int64))
    for h in hub_cols:
        rows.append(np.arange(n, dtype=np.int64))
        cols.append(np.full(n, h, dtype=np.int64))
    key = _sorted_unique(np.concatenate(rows) * n + np.concatenate(cols))
    return _finish(n, n, key // n, key % n, values, 2, f"hub{n}")


def row_block(A: CSR, r0: int, r1: int) -> CSR:
    """Rows [r0, r1) of A as a (r1-r0) x n CSR (input slicing for sampled checks)."""
    s, e = int(A.rowptr[r0]), int(A.rowptr[r1])
    return CSR(r1 - r0, A.n, (A.rowptr[r0:r1 + 1] - s).copy(), A.col[s:e].copy(), A.val[s:e].copy(), A.name + f"[{r0}:{r1}]")
