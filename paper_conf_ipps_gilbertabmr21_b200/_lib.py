"""ctypes declarations for libhec.so (include/hec.h).  Argument marshalling only."""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# HEC_LIB_PATH: an alternative build of libhec.so (A/B timing of kernel variants)
LIB_PATH = os.environ.get("HEC_LIB_PATH") or os.path.join(_HERE, "libhec.so")

HEC_OK, HEC_EINVAL, HEC_ENOMEM, HEC_ECUDA, HEC_EOVERFLOW = 0, -1, -2, -3, -4
STOP_CUTOFF, STOP_DISCARD, STOP_STALL, STOP_MAX_LEVELS = 0, 1, 2, 3
MAP_METHODS = {"hec": 0, "hec3": 1, "hem": 2}  # HEC_MAP_HEC / HEC_MAP_HEC3 / HEC_MAP_HEM
BUILD_METHODS = {"hash": 0, "sort": 1, "one_end": 2, "auto": 3}  # HEC_BUILD_*

# Every symbol include/hec.h declares (checked by tests/test_abi.py).
EXPORTS = [
    "hec_last_error", "hec_ctx_create", "hec_ctx_destroy", "hec_ctx_set_validate",
    "hec_ctx_set_stream", "hec_ctx_last_stats", "hec_prio", "hec_find_mapping",
    "hec_find_mapping_prio", "build_coarse_graph", "hec_csr_view", "hec_csr_free",
    "coarsen_hierarchy", "hec_hierarchy_levels", "hec_hierarchy_level",
    "hec_hierarchy_stop_reason", "hec_hierarchy_discarded_n_c", "hec_hierarchy_rounds",
    "hec_hierarchy_free", "hec_debug_heavy", "hec_debug_roots", "hec_build_rows_count",
    "hec_build_rows_write", "hec_heavy_range", "hec_mapping_from_heavy", "hec_balance_rows",
    "hec_ctx_set_profiling", "hec_ctx_profile_reset", "hec_ctx_profile",
    "hec_ctx_launches", "hec_find_mapping_dist", "build_coarse_graph_dist", "hec_csr_dist_slice",
    "coarsen_hierarchy_dist", "hec_find_mapping_method", "hec_find_mapping_method_prio", "coarsen_hierarchy_ex",
    "hec_spectral_bisection", "build_coarse_graph_ex",
]


class HecGraph(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("col", ctypes.c_void_p),
                ("wgt", ctypes.c_void_p), ("vwgt", ctypes.c_void_p)]


class HecStats(ctypes.Structure):
    _fields_ = [("rounds", ctypes.c_int32), ("fallback", ctypes.c_int32),
                ("n_c", ctypes.c_int64), ("nnz_c", ctypes.c_int64),
                ("huge_rows", ctypes.c_int64), ("dense_rows", ctypes.c_int64)]


class HecSpectralOpts(ctypes.Structure):
    _fields_ = [("max_iter", ctypes.c_int64), ("tol", ctypes.c_double), ("seed", ctypes.c_uint64)]


class HecPhaseTime(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char * 24), ("ms", ctypes.c_double), ("calls", ctypes.c_int64),
                ("bytes", ctypes.c_double), ("level", ctypes.c_int32)]


ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
# int allgather(const void *send, void *recv, size_t bytes, stream, void *user)
ALLGATHER_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p,
                                ctypes.c_void_p)


class HecComm(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int32), ("world", ctypes.c_int32), ("allgather", ALLGATHER_FN),
                ("user", ctypes.c_void_p)]
FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p)

_L = None


def load():
    """Load libhec.so.  Fails loudly: there is no fallback implementation."""
    global _L
    if _L is not None:
        return _L
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"libhec.so not built ({LIB_PATH}); run `make hec` "
                           "or __graft_entry__.build()")
    L = ctypes.CDLL(LIB_PATH)
    p, i64, i32, u64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_uint64
    G = ctypes.POINTER(HecGraph)
    sig = {
        "hec_last_error": (ctypes.c_char_p, []),
        "hec_ctx_create": (i32, [p, ALLOC_FN, FREE_FN, p, ctypes.POINTER(p)]),
        "hec_ctx_destroy": (None, [p]),
        "hec_ctx_set_validate": (i32, [p, i32]),
        "hec_ctx_set_stream": (i32, [p, p]),
        "hec_ctx_last_stats": (i32, [p, ctypes.POINTER(HecStats)]),
        "hec_prio": (u64, [u64, i32, i64]),
        "hec_find_mapping": (i32, [p, G, u64, i32, p, ctypes.POINTER(i64)]),
        "hec_find_mapping_prio": (i32, [p, G, p, p, ctypes.POINTER(i64)]),
        "build_coarse_graph": (i32, [p, G, p, i64, ctypes.POINTER(p)]),
        "hec_csr_view": (i32, [p, G]),
        "hec_csr_free": (None, [p]),
        "coarsen_hierarchy": (i32, [p, G, i64, u64, i64, i32, ctypes.POINTER(p)]),
        "hec_hierarchy_levels": (i32, [p]),
        "hec_hierarchy_level": (i32, [p, i32, G, ctypes.POINTER(p), ctypes.POINTER(i64)]),
        "hec_hierarchy_stop_reason": (i32, [p]),
        "hec_hierarchy_discarded_n_c": (i64, [p]),
        "hec_hierarchy_rounds": (i32, [p, i32]),
        "hec_hierarchy_free": (None, [p]),
        "hec_debug_heavy": (i32, [p, G, p]),
        "hec_debug_roots": (i32, [p, G, p, u64, i32, p, ctypes.POINTER(i32)]),
        "hec_build_rows_count": (i32, [p, G, p, i64, i64, i64, p, ctypes.POINTER(i64)]),
        "hec_build_rows_write": (i32, [p, i64, p, p, p, p]),
        "hec_heavy_range": (i32, [p, G, i64, i64, p]),
        "hec_mapping_from_heavy": (i32, [p, G, p, u64, i32, i64, i64, p, ctypes.POINTER(i64)]),
        "hec_balance_rows": (i32, [p, G, p, i64, i32, ctypes.POINTER(i64)]),
        "hec_ctx_set_profiling": (i32, [p, i32]),
        "hec_ctx_profile_reset": (i32, [p]),
        "hec_ctx_profile": (i32, [p, ctypes.POINTER(HecPhaseTime), i32, ctypes.POINTER(i32)]),
        "hec_ctx_launches": (i64, [p]),
        "hec_find_mapping_dist": (i32, [p, G, u64, i32, ctypes.POINTER(HecComm), p, ctypes.POINTER(i64)]),
        "build_coarse_graph_dist": (i32, [p, G, p, i64, ctypes.POINTER(HecComm), i32, ctypes.POINTER(p)]),
        "hec_csr_dist_slice": (i32, [p, ctypes.POINTER(i64), ctypes.POINTER(i64), ctypes.POINTER(i64),
                                     ctypes.POINTER(i64)]),
        "coarsen_hierarchy_dist": (i32, [p, G, i64, u64, i64, i32, ctypes.POINTER(HecComm), i64, ctypes.POINTER(p)]),
        "hec_find_mapping_method": (i32, [p, G, i32, u64, i32, p, ctypes.POINTER(i64)]),
        "hec_find_mapping_method_prio": (i32, [p, G, i32, p, p, ctypes.POINTER(i64)]),
        "coarsen_hierarchy_ex": (i32, [p, G, i64, u64, i64, i32, i32, i32, ctypes.POINTER(p)]),
        "build_coarse_graph_ex": (i32, [p, G, p, i64, i32, ctypes.POINTER(p)]),
        "hec_spectral_bisection": (i32, [p, G, p, ctypes.POINTER(HecSpectralOpts), p, p, ctypes.POINTER(i64),
                                         ctypes.POINTER(i64)]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _L = L
    return L


class HecError(RuntimeError):
    def __init__(self, code: int, what: str):
        msg = load().hec_last_error().decode(errors="replace")
        super().__init__(f"{what} failed (code {code}): {msg}")
        self.code = code


def check(rc: int, what: str):
    if rc != HEC_OK:
        raise HecError(rc, what)
