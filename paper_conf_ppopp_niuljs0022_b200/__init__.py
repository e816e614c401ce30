"""B200-native TileSpGEMM hot path (Niu et al., PPoPP'22) -- Python binding.

Argument marshalling only: every step of the path runs in libtsg.so's sm_100a kernels behind
the C ABI of ``include/tsg.h``.  PyTorch provides device memory (input tensors), the current
stream and process groups; results alias library-owned device memory as torch tensors.

    import paper_conf_ppopp_niuljs0022_b200 as tsg
    A = tsg.csr_to_tiles(rowptr, col, val, (m, n))        # torch CUDA tensors (int64/int32/float64)
    C = tsg.spgemm(A, A)                                 # C = A^2 in the sparse-tile format
    rp, ci, v = tsg.tiles_to_csr(C)                      # back to CSR (torch CUDA tensors)

Names follow the paper: tile_ptr / tile_col / tile_nnz / row_ptr / mask / idx / val (Section 3.2,
PAPER.md P:795-878).
"""
from __future__ import annotations

import ctypes as C
from dataclasses import dataclass

import numpy as np

from . import _lib
from ._lib import TILE, DENSE_NNZ, TsgError  # noqa: F401

__all__ = ["Tiles", "csr_to_tiles", "spgemm", "tiles_to_csr", "slice_rows", "wrap", "TsgError",
           "kernel_launch_count", "workspace_release", "transpose", "partition_tile_rows"]

_DT = {"int64": ("<i8", 8), "int32": ("<i4", 4), "uint8": ("|u1", 1), "uint16": ("<u2", 2), "float64": ("<f8", 8),
       "float32": ("<f4", 4), "float16": ("<f2", 2)}
# tsg_dtype (include/tsg.h) <-> value type names
DTYPES = {0: "float64", 1: "float32", 2: "float16"}
_DTYPE_CODE = {v: k for k, v in DTYPES.items()}


class _DeviceArray:
    """__cuda_array_interface__ over library memory; keeps the owning handle alive."""

    def __init__(self, ptr: int, count: int, dtype: str, owner):
        self._owner = owner
        self.__cuda_array_interface__ = {"shape": (int(count),), "typestr": _DT[dtype][0],
                                         "data": (int(ptr or 0) if count else 0, False), "version": 3,
                                         "strides": None, "stream": None}


def _torch():
    import torch

    return torch


def _stream_ptr(stream=None) -> int:
    torch = _torch()
    s = stream if stream is not None else torch.cuda.current_stream()
    return int(s.cuda_stream)


class _Handle:
    """Owns one tsg_tiles*; destroys it when the last reference (incl. tensor views) goes.

    The arrays are freed stream-ordered on the stream the handle was made on (``stream``, a
    cudaStream_t as int), so a free never overtakes the kernels that wrote them; work on other
    streams that reads them must be ordered before the last reference is dropped (as with
    torch's caching allocator and ``record_stream``)."""

    def __init__(self, ptr: int, stream: int = 0):
        self.ptr = ptr
        self.stream = stream

    def __del__(self):
        if self.ptr:
            try:
                _lib.load().tsg_tiles_destroy(C.c_void_p(self.ptr), C.c_void_p(self.stream or None))
            except Exception:
                pass
            self.ptr = 0


@dataclass
class Tiles:
    """A device-resident matrix in sparse-tile form (tensors alias the library's arrays)."""

    handle: _Handle
    m: int
    n: int
    tile_m: int
    tile_n: int
    num_tiles: int
    nnz: int
    tile_ptr: object
    tile_col: object
    tile_nnz: object
    row_ptr: object
    mask: object
    idx: object
    val: object
    stats: dict | None = None
    dtype: str = "float64"

    @property
    def ptr(self) -> C.c_void_p:
        return C.c_void_p(self.handle.ptr)

    @property
    def shape(self):
        return (self.m, self.n)

    def arrays(self) -> dict:
        return {k: getattr(self, k) for k in ("tile_ptr", "tile_col", "tile_nnz", "row_ptr", "mask", "idx", "val")}

    def space(self) -> dict:
        """Bytes of this matrix in the tile format vs CSR (the paper's Fig 11,
        P:2991-3057).  Tile format: tile_ptr 8(tm+1) + per tile 4 (col) + 8 (nnz offset) + 16
        (row_ptr) + 32 (mask) + per nonzero 1 (idx) + 8 (val); CSR: 8(m+1) row offsets (int64, reading
        A4) + per nonzero 4 (col) + 8 (val)."""
        vb = _DT[self.dtype][1]
        tile = 8 * (self.tile_m + 1) + 8 + 60 * self.num_tiles + (1 + vb) * self.nnz
        csr = 8 * (self.m + 1) + (4 + vb) * self.nnz
        return {"tile_bytes": tile, "csr_bytes": csr, "ratio": tile / csr if csr else float("nan")}

    def copy_to_host(self, out: dict | None = None, stream=None, blocking: bool = True) -> dict:
        """Copy the seven arrays into host buffers (numpy or pinned torch CPU tensors) via the C ABI.
        ``blocking=False``: stream-ordered (tsg_tiles_copy_to_host_async); the buffers are valid once
        ``stream`` has passed the copy, and this matrix must stay alive until then."""
        sizes = {"tile_ptr": (self.tile_m + 1, np.int64), "tile_col": (self.num_tiles, np.int32),
                 "tile_nnz": (self.num_tiles + 1, np.int64), "row_ptr": (16 * self.num_tiles, np.uint8),
                 "mask": (16 * self.num_tiles, np.uint16), "idx": (self.nnz, np.uint8),
                 "val": (self.nnz, getattr(np, self.dtype))}
        if out is None:
            out = {k: np.empty(n, dt) for k, (n, dt) in sizes.items()}
        ptrs = []
        for k in sizes:
            a = out[k]
            ptrs.append(C.c_void_p(a.data_ptr() if hasattr(a, "data_ptr") else a.ctypes.data))
        L = _lib.load()
        fn = L.tsg_tiles_copy_to_host if blocking else L.tsg_tiles_copy_to_host_async
        _lib.check(fn(self.ptr, C.c_void_p(_stream_ptr(stream)), *ptrs))
        return out


def _from_handle(ptr: int, stats=None, stream: int = 0) -> Tiles:
    L = _lib.load()
    h = _Handle(ptr, stream)
    v = _lib.TilesView()
    _lib.check(L.tsg_tiles_get_view(C.c_void_p(ptr), C.byref(v)))
    torch = _torch()

    def t(p, count, dt):
        if count == 0:
            return torch.empty(0, dtype=getattr(torch, dt), device="cuda")
        return torch.as_tensor(_DeviceArray(p, count, dt, h), device="cuda")

    return Tiles(h, v.m, v.n, v.tile_m, v.tile_n, v.num_tiles, v.nnz,
                 t(v.tile_ptr, v.tile_m + 1, "int64"), t(v.tile_col, v.num_tiles, "int32"),
                 t(v.tile_nnz, v.num_tiles + 1, "int64"), t(v.row_ptr, 16 * v.num_tiles, "uint8"),
                 t(v.mask, 16 * v.num_tiles, "uint16"), t(v.idx, v.nnz, "uint8"), t(v.val, v.nnz, DTYPES[v.dtype]),
                 stats, DTYPES[v.dtype])


def _dptr(x, dtype) -> C.c_void_p:
    torch = _torch()
    if not isinstance(x, torch.Tensor) or not x.is_cuda:
        raise TypeError("expected a CUDA torch tensor")
    if x.dtype != dtype or not x.is_contiguous():
        raise TypeError(f"expected a contiguous {dtype} tensor, got {x.dtype}")
    return C.c_void_p(x.data_ptr() if x.numel() else 0)


def csr_to_tiles(row_ptr, col_idx, val, shape, validate: bool = False, stream=None) -> Tiles:
    """CSR -> sparse tiles on the GPU (tsg_csr_to_tiles_typed).

    Device input: torch CUDA tensors (int64 row_ptr, int32 col_idx, float64/float32/float16 val).
    Host input: numpy arrays or CPU torch tensors (pinned for speed) -- copied in by the library.
    The value type is taken from ``val`` (f3: fp32 and fp16 variants).
    """
    torch = _torch()
    m, n = int(shape[0]), int(shape[1])
    L = _lib.load()
    out = C.c_void_p()
    flags = _lib.VALIDATE if validate else 0
    host = not (isinstance(row_ptr, torch.Tensor) and row_ptr.is_cuda)
    if host:
        flags |= _lib.INPUT_HOST
        arrs = []
        vdt = str(val.dtype).replace("torch.", "") if isinstance(val, torch.Tensor) else np.asarray(val).dtype.name
        if vdt not in _DTYPE_CODE:
            raise TypeError(f"unsupported value type {val.dtype} (float64, float32 or float16)")
        for a, dt, tdt in ((row_ptr, np.int64, torch.int64), (col_idx, np.int32, torch.int32),
                           (val, getattr(np, vdt), getattr(torch, vdt))):
            if isinstance(a, torch.Tensor):
                if a.dtype != tdt:
                    if tdt.is_floating_point or not a.dtype.is_floating_point:
                        a = a.to(tdt)
                    else:
                        raise TypeError(f"expected an integer tensor, got {a.dtype}")
                a = a.contiguous()
                arrs.append((a, C.c_void_p(a.data_ptr() if a.numel() else 0)))
            else:
                a = np.ascontiguousarray(a, dtype=dt)
                arrs.append((a, C.c_void_p(a.ctypes.data if a.size else 0)))
        if len(arrs[0][0]) != m + 1:
            raise ValueError(f"row_ptr has {len(arrs[0][0])} entries, expected m + 1 = {m + 1}")
        nnz = int(arrs[0][0][-1]) if m >= 0 and len(arrs[0][0]) else 0
        if len(arrs[1][0]) < nnz or len(arrs[2][0]) < nnz:
            raise ValueError(f"row_ptr[m] = {nnz} exceeds the length of col_idx / val")
        rc = L.tsg_csr_to_tiles_typed(m, n, nnz, arrs[0][1], arrs[1][1], arrs[2][1], _DTYPE_CODE[vdt], flags,
                                      None, C.c_void_p(_stream_ptr(stream)), C.byref(out))
    else:
        nnz = int(col_idx.numel())
        vdt = str(val.dtype).replace("torch.", "")
        if vdt not in _DTYPE_CODE:
            raise TypeError(f"unsupported value type {val.dtype}")
        rc = L.tsg_csr_to_tiles_typed(m, n, nnz, _dptr(row_ptr, torch.int64), _dptr(col_idx, torch.int32),
                                      _dptr(val, val.dtype), _DTYPE_CODE[vdt], flags, None,
                                      C.c_void_p(_stream_ptr(stream)), C.byref(out))
    _lib.check(rc)
    return _from_handle(out.value, stream=_stream_ptr(stream))


def spgemm(A: Tiles, B: Tiles, stats: bool = False, timing: bool = False, products: bool = False,
           structural: bool = False, scan_only: bool = False, list_always: bool = False,
           dense_threshold: int | None = None, sort_only: bool = False, path_general: bool = False,
           path_rows: bool = False, debug_high_offsets: bool = False,
           small_stage: bool | None = None, queue_chunk: int | None = None, stream=None) -> Tiles:
    """C = A*B in the sparse-tile format (tsg_spgemm: steps 1-3 of Section 3.3).

    stats / timing / products / structural: fill ``C.stats`` (one extra blocking read), with CUDA-
    event step times, the intermediate-product count, |C'| of the paper's step 1.  The other
    options select work splits only (the result is the same bit for bit): step-1 modes, the dense
    threshold t_nnz, ``path_general`` (the per-C-tile pipeline even for narrow tile rows), ``path_rows``
    (the fused per-tile-row pipeline wherever every tile row is narrow), ``debug_high_offsets`` (C's
    nonzero offsets carry +2^32 inside the call: a test of the 64-bit offset paths),
    ``queue_chunk`` (per-C-tile work distribution: 0 static, k > 0 k groups per request)."""
    L = _lib.load()
    flags = 0
    if timing:
        flags |= _lib.STATS_TIMING
    if products:
        flags |= _lib.STATS_PRODUCTS
    if structural:
        flags |= _lib.STATS_STRUCTURAL
    if scan_only:
        flags |= _lib.STEP1_SCAN_ONLY
    if list_always:
        flags |= _lib.STEP1_LIST_ALWAYS
    if sort_only:
        flags |= _lib.STEP1_SORT_ONLY
    if path_general:
        flags |= _lib.PATH_GENERAL
    if path_rows:
        flags |= _lib.PATH_ROWS_FORCE
    if debug_high_offsets:
        flags |= _lib.DEBUG_HIGH_OFFSETS
    if small_stage is not None:
        flags |= _lib.SMALL_STAGE_ON if small_stage else _lib.SMALL_STAGE_OFF
    if dense_threshold is not None:
        if not 1 <= dense_threshold <= 257:
            raise ValueError("dense_threshold must be in [1, 257]")
        flags |= dense_threshold << _lib.DENSE_THRESHOLD_SHIFT
    if queue_chunk is not None:
        if not 0 <= queue_chunk <= 14:
            raise ValueError("queue_chunk must be in [0, 14]")
        flags |= (queue_chunk + 1) << _lib.QUEUE_CHUNK_SHIFT
    st = _lib.Stats() if (stats or timing or products or structural) else None
    out = C.c_void_p()
    sp = _stream_ptr(stream)
    rc = L.tsg_spgemm(A.ptr, B.ptr, flags, None, C.c_void_p(sp), C.byref(out),
                      C.byref(st) if st is not None else None)
    _lib.check(rc)
    return _from_handle(out.value, st.as_dict() if st is not None else None, stream=sp)


def transpose(T: Tiles, stream=None) -> Tiles:
    """A^T in the sparse-tile format (tsg_tiles_transpose), e.g. for C = A * A^T."""
    out = C.c_void_p()
    sp = _stream_ptr(stream)
    _lib.check(_lib.load().tsg_tiles_transpose(T.ptr, None, C.c_void_p(sp), C.byref(out)))
    return _from_handle(out.value, stream=sp)


def tiles_to_csr(T: Tiles, stream=None):
    """Sparse tiles -> CSR on the GPU; returns (row_ptr int64, col_idx int32, val of T's dtype) tensors."""
    L = _lib.load()
    torch = _torch()
    rp, ci, v = C.c_void_p(), C.c_void_p(), C.c_void_p()
    nnz = C.c_int64()
    sp = _stream_ptr(stream)
    _lib.check(L.tsg_tiles_to_csr(T.ptr, None, C.c_void_p(sp), C.byref(rp), C.byref(ci),
                                  C.byref(v), C.byref(nnz)))
    owner = _CsrOwner([rp.value, ci.value, v.value], sp)

    def t(p, count, dt):
        if count == 0:
            return torch.empty(0, dtype=getattr(torch, dt), device="cuda")
        return torch.as_tensor(_DeviceArray(p, count, dt, owner), device="cuda")

    return t(rp.value, T.m + 1, "int64"), t(ci.value, nnz.value, "int32"), t(v.value, nnz.value, T.dtype)


class _CsrOwner:
    """Frees the arrays of tsg_tiles_to_csr on the stream that produced them (stream-ordered)."""

    def __init__(self, ptrs, stream: int = 0):
        self.ptrs = ptrs
        self.stream = stream

    def __del__(self):
        try:
            L = _lib.load()
            for p in self.ptrs:
                if p:
                    L.tsg_free(C.c_void_p(p), 0, None, C.c_void_p(self.stream or None))
        except Exception:
            pass


def slice_rows(T: Tiles, tile_row_begin: int, tile_row_end: int, stream=None) -> Tiles:
    """Zero-copy view of tile rows [begin, end) (tsg_tiles_slice_rows).  Keeps T alive."""
    out = C.c_void_p()
    sp = _stream_ptr(stream)
    _lib.check(_lib.load().tsg_tiles_slice_rows(T.ptr, int(tile_row_begin), int(tile_row_end),
                                                C.c_void_p(sp), C.byref(out)))
    V = _from_handle(out.value, stream=sp)
    V.handle.parent = T.handle  # the view borrows T's arrays
    return V


def wrap(m: int, n: int, arrays: dict, keepalive=None) -> Tiles:
    """Borrowing handle over seven torch CUDA tensors laid out as Section 3.2 (tsg_tiles_wrap)."""
    torch = _torch()
    v = _lib.TilesView()
    v.m, v.n = int(m), int(n)
    v.tile_m, v.tile_n = (m + TILE - 1) // TILE, (n + TILE - 1) // TILE
    v.num_tiles = int(arrays["tile_col"].numel())
    v.nnz = int(arrays["val"].numel())
    vdt = str(arrays["val"].dtype).replace("torch.", "")
    if vdt not in _DTYPE_CODE:
        raise TypeError(f"unsupported value type {arrays['val'].dtype}")
    v.dtype = _DTYPE_CODE[vdt]
    for k, dt in (("tile_ptr", torch.int64), ("tile_col", torch.int32), ("tile_nnz", torch.int64),
                  ("row_ptr", torch.uint8), ("mask", torch.uint16), ("idx", torch.uint8), ("val", arrays["val"].dtype)):
        setattr(v, k, _dptr(arrays[k], dt).value)
    out = C.c_void_p()
    _lib.check(_lib.load().tsg_tiles_wrap(C.byref(v), None, C.byref(out)))
    T = _from_handle(out.value)
    T.handle.keep = (arrays, keepalive)
    return T


def partition_tile_rows(A: Tiles, B: Tiles, parts: int, stream=None):
    """Product-balanced cuts of C's tile rows for ``parts`` ranks, computed on the device
    (tsg_partition_tile_rows).  Returns (cuts: numpy int64 [parts + 1], products)."""
    cuts = np.zeros(int(parts) + 1, dtype=np.int64)
    tot = C.c_int64()
    _lib.check(_lib.load().tsg_partition_tile_rows(A.ptr, B.ptr, int(parts), C.c_void_p(_stream_ptr(stream)),
                                                   C.c_void_p(cuts.ctypes.data), C.byref(tot)))
    return cuts, int(tot.value)


def kernel_launch_count() -> int:
    return int(_lib.load().tsg_kernel_launch_count())


def workspace_release(stream=None) -> int:
    """Free this thread's cached scratch arena on the current device (tsg_workspace_release)."""
    return int(_lib.load().tsg_workspace_release(C.c_void_p(_stream_ptr(stream))))
