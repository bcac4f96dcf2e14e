"""ctypes declarations of include/sptrsv.h (argument marshalling only).

Loading fails loudly if the in-tree CUDA library is missing: there is no CPU
fallback anywhere in this package.
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libsptrsv_b200.so")

# enums (must match include/sptrsv.h)
SUCCESS = 0
STATUS_NAMES = {0: "SUCCESS", 1: "INVALID_VALUE", 2: "NOT_TRIANGULAR", 3: "UNSORTED", 4: "ZERO_PIVOT",
                5: "NOT_SUPPORTED", 6: "ALLOC", 7: "CUDA", 8: "DEADLOCK"}
R64F, R32F = 0, 1
LOWER, UPPER = 0, 1
COL_MAJOR, ROW_MAJOR = 0, 1
VARIANTS = {"REC": 0, "COL": 1, "ROW": 2}
SELECTORS = {"PAPER": 0, "B200": 1}
KERNELS = ["COMPLETELY_PARALLEL", "LEVEL_SET", "SYNC_FREE", "NEAR_SERIAL",
           "SCALAR_CSR", "SCALAR_DCSR", "VECTOR_CSR", "VECTOR_DCSR"]
FORMATS = ["DIAG", "CSR", "DCSR"]
IMPLS = ["TRI_DIAG", "TRI_LEVELSET", "TRI_SYNCFREE", "TRI_CHAIN", "SQ_SCALAR", "SQ_VECTOR", "TRI_SUPERNODE", "TRI_PIPE", "SQ_ADAPT"]
ARRAY_IN_DEGREE, ARRAY_LEVEL_PTR, ARRAY_DCSR_ROWS = 0, 1, 2

EXPORTS = ["sptrsv_opts_default", "sptrsv_analyse", "sptrsv_solve", "sptrsv_solve_transposed", "sptrsv_free", "sptrsv_plan_info",
           "sptrsv_plan_segments", "sptrsv_plan_perm", "sptrsv_plan_levels", "sptrsv_plan_seg_array",
           "sptrsv_plan_matrix", "sptrsv_plan_hash", "sptrsv_set_profiling", "sptrsv_seg_times", "sptrsv_status_string",
           "sptrsv_last_error", "sptrsv_version"]


DEV_ALLOC = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
DEV_FREE = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p)


class Opts(ctypes.Structure):
    _fields_ = [("variant", ctypes.c_int32), ("depth", ctypes.c_int32), ("min_block_rows", ctypes.c_int64),
                ("reorder", ctypes.c_int32), ("selector", ctypes.c_int32), ("force_tri_impl", ctypes.c_int32),
                ("force_sq_impl", ctypes.c_int32), ("host_only", ctypes.c_int32), ("sm_count", ctypes.c_int32),
                ("threads", ctypes.c_int32), ("device", ctypes.c_int32), ("transpose", ctypes.c_int32),
                ("max_nrhs", ctypes.c_int32), ("graphs", ctypes.c_int32), ("analysis", ctypes.c_int32),
                ("reserved", ctypes.c_int32 * 4),
                ("dev_alloc", DEV_ALLOC), ("dev_free", DEV_FREE), ("alloc_ctx", ctypes.c_void_p)]


class PlanInfo(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int32), ("depth", ctypes.c_int32), ("nseg", ctypes.c_int32),
                ("variant", ctypes.c_int32), ("dtype", ctypes.c_int32), ("fill", ctypes.c_int32),
                ("reorder", ctypes.c_int32), ("selector", ctypes.c_int32), ("nnz", ctypes.c_int64),
                ("min_block_rows", ctypes.c_int64), ("sm_count", ctypes.c_int32),
                ("launches_per_solve", ctypes.c_int32), ("analyse_ms", ctypes.c_double),
                ("device_bytes", ctypes.c_int64), ("depth_rule", ctypes.c_int32),
                ("analysis", ctypes.c_int32)]


class SegInfo(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("row0", ctypes.c_int32), ("row1", ctypes.c_int32),
                ("col0", ctypes.c_int32), ("col1", ctypes.c_int32), ("nnz", ctypes.c_int64),
                ("nlevels", ctypes.c_int32), ("nnz_per_row", ctypes.c_int32), ("empty_rows", ctypes.c_int32),
                ("kernel", ctypes.c_int32), ("format", ctypes.c_int32), ("impl", ctypes.c_int32),
                ("max_level_rows", ctypes.c_int32)]


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(
            f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
            "(nvcc, sm_100a). There is no CPU fallback.")
    L = ctypes.CDLL(LIB_PATH)
    vp, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
    L.sptrsv_opts_default.restype = None
    L.sptrsv_opts_default.argtypes = [ctypes.POINTER(Opts)]
    L.sptrsv_analyse.restype = ctypes.c_int
    L.sptrsv_analyse.argtypes = [i32, i64, vp, vp, vp, ctypes.c_int, ctypes.c_int, ctypes.POINTER(Opts), vp,
                                 ctypes.POINTER(vp)]
    L.sptrsv_solve.restype = ctypes.c_int
    L.sptrsv_solve.argtypes = [vp, vp, i64, vp, i64, i32, ctypes.c_int, vp]
    L.sptrsv_solve_transposed.restype = ctypes.c_int
    L.sptrsv_solve_transposed.argtypes = [vp, vp, i64, vp, i64, i32, ctypes.c_int, vp]
    L.sptrsv_free.restype = ctypes.c_int
    L.sptrsv_free.argtypes = [vp]
    L.sptrsv_plan_info.restype = ctypes.c_int
    L.sptrsv_plan_info.argtypes = [vp, ctypes.POINTER(PlanInfo)]
    L.sptrsv_plan_segments.restype = ctypes.c_int
    L.sptrsv_plan_segments.argtypes = [vp, ctypes.POINTER(SegInfo), i32, ctypes.POINTER(i32)]
    L.sptrsv_plan_perm.restype = ctypes.c_int
    L.sptrsv_plan_perm.argtypes = [vp, vp]
    L.sptrsv_plan_levels.restype = ctypes.c_int
    L.sptrsv_plan_levels.argtypes = [vp, vp]
    L.sptrsv_plan_seg_array.restype = ctypes.c_int
    L.sptrsv_plan_seg_array.argtypes = [vp, i32, i32, vp, i64, ctypes.POINTER(i64)]
    L.sptrsv_plan_matrix.restype = ctypes.c_int
    L.sptrsv_plan_matrix.argtypes = [vp, vp, vp, vp]
    L.sptrsv_plan_hash.restype = ctypes.c_int
    L.sptrsv_plan_hash.argtypes = [vp, ctypes.POINTER(ctypes.c_uint64)]
    L.sptrsv_set_profiling.restype = ctypes.c_int
    L.sptrsv_set_profiling.argtypes = [vp, i32]
    L.sptrsv_seg_times.restype = ctypes.c_int
    L.sptrsv_seg_times.argtypes = [vp, ctypes.POINTER(ctypes.c_float), i32, ctypes.POINTER(i32)]
    L.sptrsv_status_string.restype = ctypes.c_char_p
    L.sptrsv_status_string.argtypes = [ctypes.c_int]
    L.sptrsv_last_error.restype = ctypes.c_char_p
    L.sptrsv_last_error.argtypes = []
    L.sptrsv_version.restype = ctypes.c_char_p
    L.sptrsv_version.argtypes = []
    _lib = L
    return L


class SptrsvError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        self.status_name = STATUS_NAMES.get(status, str(status))
        detail = lib().sptrsv_last_error().decode(errors="replace")
        super().__init__(f"{where}: SPTRSV_ERROR_{self.status_name}: {detail}")


def check(status: int, where: str) -> None:
    if status != SUCCESS:
        raise SptrsvError(status, where)
