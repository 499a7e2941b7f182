"""ctypes declarations of include/gamma.h (argument marshalling only).

Loads the in-tree ``libgamma.so``.  There is no fallback: if the library is
missing or cannot be loaded, importing raises ``ImportError``.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
# GAMMA_LIB_VARIANT=<tag>: an in-tree A/B build (build.py tag=...), libgamma_<tag>.so
LIB_PATH = os.path.join(HERE, f"libgamma_{os.environ['GAMMA_LIB_VARIANT']}.so"
                        if os.environ.get("GAMMA_LIB_VARIANT") else "libgamma.so")

GAMMA_OK = 0
GAMMA_E_INVAL = -1
GAMMA_E_NOMEM = -2
GAMMA_E_CUDA = -3
GAMMA_E_OVERFLOW = -4
GAMMA_E_UNSUPPORTED = -5

GAMMA_FLAG_TIME_KERNELS = 0x1
GAMMA_FLAG_NO_FUSE = 0x2
GAMMA_FLAG_SPILL = 0x4
GAMMA_FLAG_DEBUG_NOSTAGE = 0x8
GAMMA_FLAG_NO_BITMAP = 0x10
GAMMA_FLAG_NO_SPLIT = 0x20
GAMMA_FLAG_DEBUG_SPLIT_ALL = 0x40
GAMMA_FLAG_COUNT_SORT_BUILD = 0x80
GAMMA_FLAG_FPM_INSTANCES = 0x100
GAMMA_FLAG_TWO_PASS = 0x200
GAMMA_FLAG_SM_EDGE_JOIN = 0x400
GAMMA_FLAG_HOST_DAG = 0x800

ALLOC_FN = C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p)
FREE_FN = C.CFUNCTYPE(None, C.c_void_p, C.c_void_p)
ALLREDUCE_FN = C.CFUNCTYPE(C.c_int32, C.POINTER(C.c_uint64), C.c_size_t, C.c_void_p)
ALLTOALL_FN = C.CFUNCTYPE(C.c_int32, C.c_void_p, C.c_void_p, C.c_uint64, C.c_void_p)


class gamma_ctx_desc(C.Structure):
    _fields_ = [
        ("device", C.c_int32), ("rank", C.c_int32), ("world", C.c_int32),
        ("stream", C.c_void_p),
        ("dev_alloc", ALLOC_FN), ("dev_free", FREE_FN), ("alloc_user", C.c_void_p),
        ("allreduce_sum_u64", ALLREDUCE_FN), ("coll_user", C.c_void_p),
        ("hbm_budget_bytes", C.c_uint64), ("host_spill_bytes", C.c_uint64),
        ("flags", C.c_uint32),
        ("alltoall_u32", ALLTOALL_FN),
        ("dag_cache_bytes", C.c_uint64),
    ]


class gamma_graph_info(C.Structure):
    _fields_ = [("n", C.c_uint32), ("m", C.c_uint64), ("max_degree", C.c_uint32),
                ("max_out_degree", C.c_uint32), ("device_bytes", C.c_uint64), ("build_ms", C.c_double)]


class gamma_pattern(C.Structure):
    _fields_ = [("nv", C.c_uint32), ("ne", C.c_uint32), ("edges", C.POINTER(C.c_uint32)),
                ("labels", C.POINTER(C.c_uint32)), ("induced", C.c_int32)]


class gamma_plan_info(C.Structure):
    _fields_ = [("nv", C.c_uint32), ("order", C.c_uint32 * 8), ("backward_mask", C.c_uint32 * 8),
                ("less_mask", C.c_uint32 * 8), ("greater_mask", C.c_uint32 * 8), ("aut", C.c_uint64)]


class gamma_fpm_pattern(C.Structure):
    _fields_ = [("nv", C.c_uint32), ("ne", C.c_uint32), ("labels", C.c_uint32 * 8),
                ("edges", (C.c_uint8 * 2) * 8), ("support", C.c_uint64),
                ("instances", C.c_uint64)]


class gamma_fpm_result(C.Structure):
    _fields_ = [("n", C.c_uint64), ("pats", C.POINTER(gamma_fpm_pattern))]


MAX_KC = 16
MAX_LEVELS = 34


class gamma_run_stats(C.Structure):
    _fields_ = [
        ("n_classes", C.c_uint32),
        ("name", (C.c_char * 32) * MAX_KC),
        ("launches", C.c_uint64 * MAX_KC),
        ("ms", C.c_double * MAX_KC),
        ("alg_bytes", C.c_uint64 * MAX_KC),
        ("level_entries", C.c_uint64 * MAX_LEVELS),
        ("list_elems", C.c_uint64), ("chunks", C.c_uint64), ("retries", C.c_uint64),
        ("spilled_bytes", C.c_uint64), ("total_launches", C.c_uint64), ("wall_ms", C.c_double),
    ]


# (name, restype, argtypes) -- every entry point declared in include/gamma.h
SIGNATURES = [
    ("gamma_abi_version", C.c_int32, []),
    ("gamma_last_error", C.c_char_p, []),
    ("gamma_ctx_create", C.c_int32, [C.POINTER(gamma_ctx_desc), C.POINTER(C.c_void_p)]),
    ("gamma_ctx_destroy", None, [C.c_void_p]),
    ("gamma_ctx_trim", C.c_int32, [C.c_void_p]),
    ("gamma_load_edges", C.c_int32, [C.c_void_p, C.c_uint32, C.c_void_p, C.c_void_p, C.c_uint64,
                                     C.c_void_p, C.POINTER(C.c_void_p)]),
    ("gamma_load_csr", C.c_int32, [C.c_void_p, C.c_uint32, C.c_void_p, C.c_void_p, C.c_void_p,
                                   C.POINTER(C.c_void_p)]),
    ("gamma_graph_free", None, [C.c_void_p]),
    ("gamma_graph_get_info", C.c_int32, [C.c_void_p, C.POINTER(gamma_graph_info)]),
    ("gamma_graph_copy_csr", C.c_int32, [C.c_void_p, C.c_int, C.c_void_p, C.c_void_p]),
    ("gamma_kclique", C.c_int32, [C.c_void_p, C.c_uint32, C.POINTER(C.c_uint64)]),
    ("gamma_kclique_multi", C.c_int32, [C.c_void_p, C.c_uint32, C.c_void_p, C.c_void_p]),
    ("gamma_kclique_roots", C.c_int32, [C.c_void_p, C.c_uint32, C.c_uint64, C.c_void_p, C.c_void_p]),
    ("gamma_pattern_plan", C.c_int32, [C.POINTER(gamma_pattern), C.POINTER(gamma_plan_info)]),
    ("gamma_match", C.c_int32, [C.c_void_p, C.POINTER(gamma_pattern), C.POINTER(C.c_uint64),
                                C.POINTER(C.c_uint64)]),
    ("gamma_match_batch", C.c_int32, [C.c_void_p, C.c_uint32, C.POINTER(gamma_pattern), C.c_void_p,
                                      C.c_void_p]),
    ("gamma_fpm", C.c_int32, [C.c_void_p, C.c_uint32, C.c_uint64, C.POINTER(C.POINTER(gamma_fpm_result))]),
    ("gamma_fpm_result_free", None, [C.POINTER(gamma_fpm_result)]),
    ("gamma_get_stats", C.c_int32, [C.c_void_p, C.POINTER(gamma_run_stats)]),
]

_lib = None


def load(path: str = LIB_PATH):
    """Load libgamma.so and declare every entry point.  Raises ImportError."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"libgamma.so not built at {path}: run `python paper_conf_icde_hu0o23_b200/build.py` "
                          "(there is no CPU fallback)")
    try:
        lib = C.CDLL(path)
    except OSError as e:
        raise ImportError(f"cannot load {path}: {e}") from e
    for name, res, args in SIGNATURES:
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    _lib = lib
    return lib
