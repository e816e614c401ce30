"""ctypes declarations of include/tsg.h (argument marshalling only).

The shared library is built in-tree (``make`` / ``__graft_entry__.build()``) as
``paper_conf_ppopp_niuljs0022_b200/libtsg.so``.  If it is missing this module raises: there is
no CPU fallback anywhere in the product path.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TSG_LIBRARY", os.path.join(_HERE, "libtsg.so"))

TILE = 16
DENSE_NNZ = 96  # include/tsg.h TSG_DENSE_NNZ

# flags (include/tsg.h)
INPUT_HOST = 0x1
VALIDATE = 0x2
STATS_TIMING = 0x1
STATS_STRUCTURAL = 0x2
STEP1_SCAN_ONLY = 0x4
STEP1_LIST_ALWAYS = 0x8
STATS_PRODUCTS = 0x10
PATH_GENERAL = 0x20
PATH_ROWS_FORCE = 0x400
DEBUG_HIGH_OFFSETS = 0x800
STEP1_SORT_ONLY = 0x40
SMALL_STAGE_ON = 0x100
SMALL_STAGE_OFF = 0x200
DENSE_THRESHOLD_SHIFT = 16
QUEUE_CHUNK_SHIFT = 25
PATH_TILES, PATH_ROWS = 0, 1  # tsg_stats.path

STATUS = {0: "TSG_OK", 1: "TSG_ERR_INVALID_ARG", 2: "TSG_ERR_SHAPE", 3: "TSG_ERR_UNSORTED",
          4: "TSG_ERR_OVERFLOW", 5: "TSG_ERR_OOM", 6: "TSG_ERR_CUDA", 7: "TSG_ERR_INTERNAL"}


class TsgError(RuntimeError):
    def __init__(self, status: int, detail: str):
        super().__init__(f"{STATUS.get(status, status)}: {detail}")
        self.status = status
        self.name = STATUS.get(status, str(status))


class TilesView(C.Structure):
    _fields_ = [("m", C.c_int64), ("n", C.c_int64), ("tile_m", C.c_int64), ("tile_n", C.c_int64),
                ("num_tiles", C.c_int64), ("nnz", C.c_int64),
                ("tile_ptr", C.c_void_p), ("tile_col", C.c_void_p), ("tile_nnz", C.c_void_p),
                ("row_ptr", C.c_void_p), ("mask", C.c_void_p), ("idx", C.c_void_p), ("val", C.c_void_p),
                ("dtype", C.c_int32)]


class Stats(C.Structure):
    _fields_ = [("products", C.c_int64), ("tiles_structural", C.c_int64), ("tiles_c", C.c_int64),
                ("nnz_c", C.c_int64), ("candidates", C.c_int64), ("pairs", C.c_int64),
                ("tiles_dense", C.c_int64), ("tiles_sparse", C.c_int64), ("kernel_launches", C.c_int64),
                ("step1_list_tiles", C.c_int32), ("host_syncs", C.c_int32),
                ("ms_index", C.c_float), ("ms_step1", C.c_float), ("ms_step2", C.c_float),
                ("ms_alloc", C.c_float), ("ms_step3", C.c_float), ("ms_total", C.c_float),
                ("ms_host_sync", C.c_float), ("ms_host_alloc", C.c_float),
                ("path", C.c_int64), ("step1_big_rows", C.c_int64),
                ("step1_merge_rows", C.c_int64), ("bytes_scratch", C.c_int64), ("bytes_out", C.c_int64)]

    def as_dict(self) -> dict:
        return {f[0]: getattr(self, f[0]) for f in self._fields_}


class Allocator(C.Structure):
    _fields_ = [("alloc", C.c_void_p), ("free", C.c_void_p), ("ctx", C.c_void_p)]


# every symbol the header declares (checked by tests/test_abi.py against include/tsg.h)
SYMBOLS = ["tsg_csr_to_tiles", "tsg_csr_to_tiles_typed", "tsg_spgemm", "tsg_tiles_to_csr", "tsg_tiles_get_view", "tsg_tiles_wrap",
           "tsg_tiles_slice_rows", "tsg_tiles_copy_to_host", "tsg_tiles_copy_to_host_async", "tsg_tiles_destroy", "tsg_free",
           "tsg_status_string", "tsg_last_error", "tsg_abi_version", "tsg_kernel_launch_count",
           "tsg_workspace_release", "tsg_tiles_transpose", "tsg_partition_tile_rows"]

_lib = None


def load():
    """Load libtsg.so (raises ImportError when it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"libtsg.so not found at {LIB_PATH}; run `make` or __graft_entry__.build() "
                          "(the CUDA path has no fallback)")
    L = C.CDLL(LIB_PATH)
    i64, vp, u32 = C.c_int64, C.c_void_p, C.c_uint32
    pp = C.POINTER(C.c_void_p)
    L.tsg_csr_to_tiles.restype = C.c_int
    L.tsg_csr_to_tiles.argtypes = [i64, i64, i64, vp, vp, vp, u32, vp, vp, pp]
    L.tsg_csr_to_tiles_typed.restype = C.c_int
    L.tsg_csr_to_tiles_typed.argtypes = [i64, i64, i64, vp, vp, vp, C.c_int32, u32, vp, vp, pp]
    L.tsg_spgemm.restype = C.c_int
    L.tsg_spgemm.argtypes = [vp, vp, u32, vp, vp, pp, C.POINTER(Stats)]
    L.tsg_tiles_to_csr.restype = C.c_int
    L.tsg_tiles_to_csr.argtypes = [vp, vp, vp, pp, pp, pp, C.POINTER(i64)]
    L.tsg_tiles_get_view.restype = C.c_int
    L.tsg_tiles_get_view.argtypes = [vp, C.POINTER(TilesView)]
    L.tsg_tiles_wrap.restype = C.c_int
    L.tsg_tiles_wrap.argtypes = [C.POINTER(TilesView), vp, pp]
    L.tsg_tiles_slice_rows.restype = C.c_int
    L.tsg_tiles_slice_rows.argtypes = [vp, i64, i64, vp, pp]
    L.tsg_tiles_copy_to_host.restype = C.c_int
    L.tsg_tiles_copy_to_host.argtypes = [vp, vp, vp, vp, vp, vp, vp, vp, vp]
    L.tsg_tiles_copy_to_host_async.restype = C.c_int
    L.tsg_tiles_copy_to_host_async.argtypes = [vp, vp, vp, vp, vp, vp, vp, vp, vp]
    L.tsg_tiles_destroy.restype = None
    L.tsg_tiles_destroy.argtypes = [vp, vp]
    L.tsg_free.restype = None
    L.tsg_free.argtypes = [vp, C.c_size_t, vp, vp]
    L.tsg_status_string.restype = C.c_char_p
    L.tsg_status_string.argtypes = [C.c_int]
    L.tsg_last_error.restype = C.c_char_p
    L.tsg_last_error.argtypes = []
    L.tsg_abi_version.restype = C.c_int
    L.tsg_kernel_launch_count.restype = i64
    L.tsg_tiles_transpose.restype = C.c_int
    L.tsg_tiles_transpose.argtypes = [vp, vp, vp, pp]
    L.tsg_partition_tile_rows.restype = C.c_int
    L.tsg_partition_tile_rows.argtypes = [vp, vp, i64, vp, vp, C.POINTER(i64)]
    L.tsg_workspace_release.restype = C.c_size_t
    L.tsg_workspace_release.argtypes = [vp]
    _lib = L
    return L


def check(status: int):
    if status != 0:
        detail = load().tsg_last_error().decode(errors="replace")
        raise TsgError(status, detail)
