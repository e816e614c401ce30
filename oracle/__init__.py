"""CPU oracle for TileSpGEMM -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` leg may import this package.  The product path
(``paper_conf_ppopp_niuljs0022_b200``) never imports it and shares no code with it.

A thin ctypes/numpy layer over ``oracle/tsg_oracle.c`` (plain single-threaded C, fp64,
``-O2 -ffp-contract=off``).  See the C file for the per-function citations into PAPER.md.

Parity status: O1 (Gustavson), O2/O3 (tile format), O4 (C' and Algorithm-2 masks), O5
(products), O6 (CSR transpose, for C = A*A^T) are all pinned by tests/test_oracle_pins.py (closed forms, brute force, invariants,
the paper's Fig 5 mask fact, and two-formulation cross-checks).  Nothing here is "parity
unpinned".
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "tsg_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
TILE = 16


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain C, no fused multiply-add contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fPIC", "-shared", "-std=c11", "-fopenmp",
                               "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None
_i64p = np.ctypeslib.ndpointer(np.int64, flags="C")
_i32p = np.ctypeslib.ndpointer(np.int32, flags="C")
_f64p = np.ctypeslib.ndpointer(np.float64, flags="C")
_f32p = np.ctypeslib.ndpointer(np.float32, flags="C")
_u8p = np.ctypeslib.ndpointer(np.uint8, flags="C")
_u16p = np.ctypeslib.ndpointer(np.uint16, flags="C")


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        i64 = C.c_int64
        L.orc_products.restype = i64
        L.orc_products.argtypes = [i64, _i64p, _i32p, _i64p]
        L.orc_gustavson_rowcounts.argtypes = [i64, i64, _i64p, _i32p, _i64p, _i32p, C.c_void_p, i64, _i64p]
        L.orc_gustavson.argtypes = [i64, i64, _i64p, _i32p, _f64p, _i64p, _i32p, _f64p, C.c_void_p, i64,
                                    _i64p, _i32p, _f64p, C.c_void_p, C.c_int]
        L.orc_gustavson_rowcounts_omp.argtypes = [i64, i64, _i64p, _i32p, _i64p, _i32p, C.c_void_p, i64, _i64p,
                                                  C.c_int]
        L.orc_gustavson_omp.argtypes = [i64, i64, _i64p, _i32p, _f64p, _i64p, _i32p, _f64p, C.c_void_p, i64,
                                        _i64p, _i32p, _f64p, C.c_void_p, C.c_int, C.c_int]
        L.orc_gustavson_f32.argtypes = [i64, i64, _i64p, _i32p, _f32p, _i64p, _i32p, _f32p, C.c_void_p, i64,
                                         _i64p, _i32p, _f32p, C.c_void_p, C.c_int]
        L.orc_csr_to_tiles_count.argtypes = [i64, i64, _i64p, _i32p, _i64p]
        L.orc_csr_to_tiles_fill.argtypes = [i64, i64, _i64p, _i32p, _f64p, _i64p, _i32p, _i64p, _u8p, _u16p,
                                            _u8p, _f64p]
        L.orc_tiles_to_csr.argtypes = [i64, i64, _i64p, _i32p, _i64p, _u8p, _u8p, _f64p, _i64p, _i32p, _f64p]
        L.orc_tile_structural_count.argtypes = [i64, i64, _i64p, _i32p, _i64p, _i32p, _i64p]
        L.orc_tile_structural_fill.argtypes = [i64, i64, _i64p, _i32p, _i64p, _i32p, _i64p, _i32p]
        L.orc_step2_masks.argtypes = [i64, i64, _i64p, _i32p, _u16p, _i64p, _i32p, _u16p, i64, _i64p, _i32p,
                                      _u16p, _i64p, _i64p, _i64p]
        L.orc_spmv.argtypes = [i64, _i64p, _i32p, _f64p, _f64p, _f64p]
        _lib = L
    return _lib


def _chk(rc: int, what: str):
    if rc != 0:
        raise RuntimeError(f"oracle {what} failed with status {rc}")


def _arr(x, dt):
    return np.ascontiguousarray(x, dtype=dt)


@dataclass
class OracleCSR:
    m: int
    n: int
    rowptr: np.ndarray
    col: np.ndarray
    val: np.ndarray
    abs: np.ndarray | None = None

    @property
    def nnz(self):
        return int(self.rowptr[-1])


@dataclass
class OracleTiles:
    """Sparse-tile arrays exactly as Section 3.2 defines them."""

    m: int
    n: int
    tile_ptr: np.ndarray
    tile_col: np.ndarray
    tile_nnz: np.ndarray
    row_ptr: np.ndarray
    mask: np.ndarray
    idx: np.ndarray
    val: np.ndarray

    @property
    def tm(self):
        return (self.m + TILE - 1) // TILE

    @property
    def tn(self):
        return (self.n + TILE - 1) // TILE

    @property
    def num_tiles(self):
        return int(self.tile_ptr[-1])

    @property
    def nnz(self):
        return int(self.tile_nnz[-1])

    def tile_rows(self) -> np.ndarray:
        """tileRowidx: the tile row of every tile (Alg 2 line 2)."""
        return np.repeat(np.arange(self.tm, dtype=np.int64), np.diff(self.tile_ptr))


# ------------------------------------------------------------------------------------------
def products(A, B) -> int:
    """O5: number of intermediate products of A*B (Table 2 caption)."""
    return int(lib().orc_products(A.m, _arr(A.rowptr, np.int64), _arr(A.col, np.int32), _arr(B.rowptr, np.int64)))


def transpose(A) -> OracleCSR:
    """O6: A^T in CSR for the paper's second workload C = A*A^T.

    The definition written out: entry (i, j, v) of A becomes (j, i, v); rows of A^T are filled by
    walking A's rows in ascending i, so every row of A^T lists its columns ascending (a stable
    counting sort by column)."""
    rowptr = np.asarray(A.rowptr, np.int64)
    col = np.asarray(A.col, np.int64)
    val = np.asarray(A.val, np.float64)
    nnz = int(rowptr[-1]) if rowptr.size else 0
    counts = np.zeros(A.n + 1, np.int64)
    for j in col[:nnz]:
        counts[j + 1] += 1
    rpT = np.cumsum(counts)
    cur = rpT[:-1].copy()
    colT = np.empty(nnz, np.int32)
    valT = np.empty(nnz, np.float64)
    for i in range(A.m):
        for p in range(rowptr[i], rowptr[i + 1]):
            j = col[p]
            colT[cur[j]] = i
            valT[cur[j]] = val[p]
            cur[j] += 1
    return OracleCSR(A.n, A.m, rpT, colT, valT)


def spgemm(A, B, fma: bool = False, rows=None, prec: str = "f64", threads: int = 1) -> OracleCSR:
    """O1: C = A*B by Gustavson's row-row Algorithm 1.  ``rows`` selects a subset.

    prec="f32": the same loop in single precision (f3); values are taken as float32
    (a float16 input is widened exactly), the result's val is float32, abs stays fp64.
    threads > 1 (fp64): the row list split over OpenMP threads, each chunk by the same C loop
    (the oracle_omp baseline of SURVEY 8(d); bit-for-bit the single-threaded result)."""
    if A.n != B.m:
        raise ValueError("shape mismatch")
    if prec not in ("f64", "f32"):
        raise ValueError("prec must be 'f64' or 'f32'")
    L = lib()
    vdt = np.float64 if prec == "f64" else np.float32
    Arp, Aci, Av = _arr(A.rowptr, np.int64), _arr(A.col, np.int32), _arr(A.val, vdt)
    Brp, Bci, Bv = _arr(B.rowptr, np.int64), _arr(B.col, np.int32), _arr(B.val, vdt)
    if rows is None:
        R, rp_ptr, nrows = A.m, None, 0
    else:
        rows = _arr(rows, np.int64)
        R, rp_ptr, nrows = rows.size, rows.ctypes.data_as(C.c_void_p), rows.size
    omp = threads > 1 and prec == "f64"
    if omp and rows is None:  # the OpenMP driver splits an explicit row list
        rows = np.arange(A.m, dtype=np.int64)
        R, rp_ptr, nrows = rows.size, rows.ctypes.data_as(C.c_void_p), rows.size
    rowlen = np.zeros(max(R, 1), dtype=np.int64)
    if omp:
        _chk(L.orc_gustavson_rowcounts_omp(A.m, B.n, Arp, Aci, Brp, Bci, rp_ptr, nrows, rowlen, int(threads)),
             "rowcounts")
    else:
        _chk(L.orc_gustavson_rowcounts(A.m, B.n, Arp, Aci, Brp, Bci, rp_ptr, nrows, rowlen), "rowcounts")
    rp = np.zeros(R + 1, dtype=np.int64)
    np.cumsum(rowlen[:R], out=rp[1:])
    nnz = int(rp[-1])
    col = np.zeros(max(nnz, 1), dtype=np.int32)
    val = np.zeros(max(nnz, 1), dtype=vdt)
    ab = np.zeros(max(nnz, 1), dtype=np.float64)
    if omp:
        _chk(L.orc_gustavson_omp(A.m, B.n, Arp, Aci, Av, Brp, Bci, Bv, rp_ptr, nrows, rp, col, val,
                                 ab.ctypes.data_as(C.c_void_p), int(fma), int(threads)), "gustavson")
    else:
        f = L.orc_gustavson if prec == "f64" else L.orc_gustavson_f32
        _chk(f(A.m, B.n, Arp, Aci, Av, Brp, Bci, Bv, rp_ptr, nrows, rp, col, val, ab.ctypes.data_as(C.c_void_p),
               int(fma)), "gustavson")
    return OracleCSR(R, B.n, rp, col[:nnz], val[:nnz], ab[:nnz])


def csr_to_tiles(A) -> OracleTiles:
    """O2: CSR -> sparse tiles (Section 3.2)."""
    L = lib()
    tm = (A.m + TILE - 1) // TILE
    Arp, Aci, Av = _arr(A.rowptr, np.int64), _arr(A.col, np.int32), _arr(A.val, np.float64)
    tp = np.zeros(tm + 1, dtype=np.int64)
    _chk(L.orc_csr_to_tiles_count(A.m, A.n, Arp, Aci, tp), "csr_to_tiles_count")
    nt = int(tp[-1])
    nnz = int(Arp[-1])
    tc = np.zeros(max(nt, 1), np.int32)
    tz = np.zeros(nt + 1, np.int64)
    rp = np.zeros(max(16 * nt, 1), np.uint8)
    mk = np.zeros(max(16 * nt, 1), np.uint16)
    ix = np.zeros(max(nnz, 1), np.uint8)
    vv = np.zeros(max(nnz, 1), np.float64)
    _chk(L.orc_csr_to_tiles_fill(A.m, A.n, Arp, Aci, Av, tp, tc, tz, rp, mk, ix, vv), "csr_to_tiles_fill")
    return OracleTiles(A.m, A.n, tp, tc[:nt], tz, rp[:16 * nt], mk[:16 * nt], ix[:nnz], vv[:nnz])


def tiles_to_csr(T: OracleTiles) -> OracleCSR:
    """O3: sparse tiles -> CSR."""
    L = lib()
    nnz = T.nnz
    rp = np.zeros(T.m + 1, np.int64)
    col = np.zeros(max(nnz, 1), np.int32)
    val = np.zeros(max(nnz, 1), np.float64)
    _chk(L.orc_tiles_to_csr(T.m, T.n, _arr(T.tile_ptr, np.int64), _arr(T.tile_col, np.int32),
                            _arr(T.tile_nnz, np.int64), _pad(T.row_ptr, np.uint8), _pad(T.idx, np.uint8),
                            _pad(T.val, np.float64), rp, col, val), "tiles_to_csr")
    return OracleCSR(T.m, T.n, rp, col[:nnz], val[:nnz])


def _pad(x, dt):
    x = _arr(x, dt)
    return x if x.size else np.zeros(1, dt)


def tile_structural(TA: OracleTiles, TB: OracleTiles):
    """O4a: C' = A'B' on the tile layouts (Section 3.3 step 1).

    Returns (Cp_ptr [tm+1], Cp_col [|C'|]).  C' keeps tiles that may turn out empty.
    """
    L = lib()
    args = (TA.tm, TB.tn, _arr(TA.tile_ptr, np.int64), _pad(TA.tile_col, np.int32),
            _arr(TB.tile_ptr, np.int64), _pad(TB.tile_col, np.int32))
    cp = np.zeros(TA.tm + 1, np.int64)
    _chk(L.orc_tile_structural_count(*args, cp), "structural_count")
    cc = np.zeros(max(int(cp[-1]), 1), np.int32)
    _chk(L.orc_tile_structural_fill(*args, cp, cc), "structural_fill")
    return cp, cc[:int(cp[-1])]


def step2_masks(TA: OracleTiles, TB: OracleTiles, cI, cJ):
    """O4b: Algorithm 2 on the C tiles (cI[t], cJ[t]).

    Returns (mask [16*nc] uint16, nnz [nc], matched pairs [nc], contributing pairs [nc]).
    """
    L = lib()
    cI = _arr(cI, np.int64)
    cJ = _arr(cJ, np.int32)
    nc = cI.size
    mask = np.zeros(max(16 * nc, 1), np.uint16)
    nnz = np.zeros(max(nc, 1), np.int64)
    matched = np.zeros(max(nc, 1), np.int64)
    contrib = np.zeros(max(nc, 1), np.int64)
    _chk(L.orc_step2_masks(TB.tm, TB.tn, _arr(TA.tile_ptr, np.int64), _pad(TA.tile_col, np.int32),
                           _pad(TA.mask, np.uint16), _arr(TB.tile_ptr, np.int64), _pad(TB.tile_col, np.int32),
                           _pad(TB.mask, np.uint16), nc, _pad(cI, np.int64), _pad(cJ, np.int32), mask, nnz,
                           matched, contrib), "step2_masks")
    return mask[:16 * nc], nnz[:nc], matched[:nc], contrib[:nc]


def spmv(A, x) -> np.ndarray:
    y = np.zeros(A.m, np.float64)
    lib().orc_spmv(A.m, _arr(A.rowptr, np.int64), _pad(A.col, np.int32), _pad(A.val, np.float64),
                   _pad(_arr(x, np.float64), np.float64), y)
    return y


# ------------------------------------------------------------------------------------------
# composite diagnostics used by tests and bench (plain compositions of O1..O5)
# ------------------------------------------------------------------------------------------
DENSE_THRESHOLD = 192  # t_nnz = 192 for 16x16 tiles; dense iff nnz >= 192 (reading A7)


def expected_tiles(A, B, fma: bool = False, prec: str = "f64") -> OracleTiles:
    """The exact tile-format C that TileSpGEMM must produce: O2(O1(A, B)) (reading A6).
    prec="f32": O1 in single precision; the tiler moves the float32 values exactly (via fp64)."""
    O = spgemm(A, B, fma=fma, prec=prec)
    T = csr_to_tiles(O)
    if prec == "f32":
        T.val = T.val.astype(np.float32)
    return T


def diagnostics(A, B) -> dict:
    """Step-level facts of Section 3.3 for A*B: |C'|, non-empty tiles, pairs, classes."""
    TA, TB = csr_to_tiles(A), csr_to_tiles(B)
    cp, cc = tile_structural(TA, TB)
    cI = np.repeat(np.arange(TA.tm, dtype=np.int64), np.diff(cp))
    mask, nnz, matched, contrib = step2_masks(TA, TB, cI, cc)
    nonempty = nnz > 0
    return dict(
        tiles_structural=int(cp[-1]),
        tiles_c=int(nonempty.sum()),
        pairs_structural=int(matched.sum()),
        pairs=int(contrib[nonempty].sum()),
        nnz_c=int(nnz.sum()),
        tiles_dense=int((nnz >= DENSE_THRESHOLD).sum()),
        products=products(A, B),
        cp_ptr=cp, cp_col=cc, cp_mask=mask, cp_nnz=nnz, cp_contrib=contrib,
    )
