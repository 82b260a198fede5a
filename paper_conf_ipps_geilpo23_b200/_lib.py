"""ctypes binding of libmce_b200.so (include/mce.h).  Marshalling only.

The library is built in-tree (paper_conf_ipps_geilpo23_b200/libmce_b200.so)
by `build()` / __graft_entry__.build().  There is no fallback: if the library
is missing or cannot load, every call raises.
"""

from __future__ import annotations

import ctypes
import os
import subprocess

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libmce_b200.so")
CSRC = os.path.join(_HERE, "csrc")
HEADER = os.path.join(os.path.dirname(_HERE), "include", "mce.h")

MCE_OK = 0
STATUS = {0: "MCE_OK", 1: "MCE_ERR_INVALID", 2: "MCE_ERR_CUDA", 3: "MCE_ERR_NOMEM", 4: "MCE_ERR_BUDGET",
          5: "MCE_ERR_STATE", 6: "MCE_ERR_SYNC"}
WHERE_HOST, WHERE_DEVICE = 0, 1
ORIENT = {"degeneracy": 0, "degree": 1, "degeneracy_det": 2}
HEURISTIC = {"none": 0, "single_degree": 1, "single_core": 2, "multi_degree": 3, "multi_core": 4}
BOUND = {"size": 0, "color": 1}

BOUND_SYNC = ctypes.CFUNCTYPE(ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, ctypes.POINTER(ctypes.c_int32),
                              ctypes.c_void_p)


class Options(ctypes.Structure):
    _fields_ = [
        ("orientation", ctypes.c_int32),
        ("heuristic", ctypes.c_int32),
        ("heuristic_runs", ctypes.c_int64),
        ("bound", ctypes.c_int32),
        ("lower_bound", ctypes.c_int32),
        ("window", ctypes.c_int64),
        ("budget_bytes", ctypes.c_int64),
        ("max_cliques", ctypes.c_int64),
        ("shard_rank", ctypes.c_int32),
        ("shard_count", ctypes.c_int32),
        ("bound_sync", BOUND_SYNC),
        ("bound_sync_user", ctypes.c_void_p),
        ("verbose", ctypes.c_int32),
        ("legacy_roots", ctypes.c_int32),
        ("no_fused_levels", ctypes.c_int32),
        ("no_clique_shortcut", ctypes.c_int32),
        ("no_fused_expand", ctypes.c_int32),
        ("shard_depth", ctypes.c_int32),
        ("no_overlap", ctypes.c_int32),
        ("no_reroot", ctypes.c_int32),
        ("no_smem_expand", ctypes.c_int32),
        ("no_root_colour", ctypes.c_int32),
    ]


class MCEError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


def build(force: bool = False, jobs: int = 8) -> str:
    """Compile the CUDA sources for sm_100a with nvcc (make in csrc/)."""
    cmd = ["make", "-C", CSRC, f"-j{jobs}"]
    if force:
        subprocess.check_call(["make", "-C", CSRC, "clean"])
    subprocess.check_call(cmd)
    return LIB_PATH


EXPORTS = [
    "mce_default_options", "mce_load_csr", "mce_graph_free", "mce_graph_clear_cache", "mce_preprocess", "mce_set_order", "mce_set_core", "mce_heuristic", "mce_enumerate",
    "mce_find_one", "mce_result_info", "mce_result_cliques", "mce_result_levels", "mce_result_timing",
    "mce_result_free", "mce_empty_cache", "mce_last_error", "mce_version",
]

_lib = None


def lib():
    """Load libmce_b200.so (raises if it is missing: no CPU fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run paper_conf_ipps_geilpo23_b200._lib.build() "
                          "(or __graft_entry__.build()); there is no CPU fallback")
    L = ctypes.CDLL(LIB_PATH)
    vp, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
    p32, p64 = ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_int64)
    L.mce_default_options.restype = None
    L.mce_default_options.argtypes = [ctypes.POINTER(Options)]
    L.mce_load_csr.restype = i32
    L.mce_load_csr.argtypes = [i32, i64, vp, vp, i32, i32, vp, ctypes.POINTER(vp)]
    L.mce_graph_free.restype = None
    L.mce_graph_free.argtypes = [vp]
    L.mce_graph_clear_cache.restype = i32
    L.mce_graph_clear_cache.argtypes = [vp]
    L.mce_preprocess.restype = i32
    L.mce_preprocess.argtypes = [vp, i32, vp, vp, i32, p32]
    L.mce_set_order.restype = i32
    L.mce_set_order.argtypes = [vp, i32, vp, i32]
    L.mce_set_core.restype = i32
    L.mce_set_core.argtypes = [vp, vp, vp, i32]
    L.mce_heuristic.restype = i32
    L.mce_heuristic.argtypes = [vp, i32, i64, p32, vp, p32, vp]
    L.mce_enumerate.restype = i32
    L.mce_enumerate.argtypes = [vp, ctypes.POINTER(Options), ctypes.POINTER(vp)]
    L.mce_find_one.restype = i32
    L.mce_find_one.argtypes = [vp, i64, ctypes.POINTER(Options), ctypes.POINTER(vp)]
    L.mce_result_info.restype = i32
    L.mce_result_info.argtypes = [vp, p32, p64, p64, p32]
    L.mce_result_cliques.restype = i32
    L.mce_result_cliques.argtypes = [vp, vp, i32]
    L.mce_result_levels.restype = i32
    L.mce_result_levels.argtypes = [vp, p64, i32, p32]
    L.mce_result_timing.restype = i32
    L.mce_result_timing.argtypes = [vp, ctypes.POINTER(ctypes.c_double), i32]
    L.mce_result_free.restype = None
    L.mce_result_free.argtypes = [vp]
    L.mce_empty_cache.restype = i32
    L.mce_empty_cache.argtypes = [i32]
    L.mce_last_error.restype = ctypes.c_char_p
    L.mce_last_error.argtypes = []
    L.mce_version.restype = ctypes.c_char_p
    L.mce_version.argtypes = []
    _lib = L
    return L


def check(status: int):
    if status != MCE_OK:
        raise MCEError(status, lib().mce_last_error().decode(errors="replace"))
