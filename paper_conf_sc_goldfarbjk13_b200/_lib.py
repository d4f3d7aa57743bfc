"""ctypes declarations of libtt.so (the C ABI in include/tt.h).

Argument marshalling only.  The library is loaded from the package directory
(built in-tree by ``build.py``); if it is missing this module raises -- there
is no fallback implementation.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
# TT_LIB=checked loads the bounds-checked build (build.py --checked,
# tt_check.cuh): the same C ABI with device-side asserts
LIB_PATH = os.path.join(HERE, "libtt_checked.so" if os.environ.get("TT_LIB") == "checked" else "libtt.so")

TT_OK = 0
STATUS = {0: "TT_OK", -1: "TT_ERR_INVALID_ARG", -2: "TT_ERR_CUDA", -3: "TT_ERR_OOM",
          -4: "TT_ERR_TREE_TOO_DEEP", -5: "TT_ERR_KIND_MISMATCH", -6: "TT_ERR_UNSUPPORTED"}
KIND_OCT, KIND_KD, KIND_VP, KIND_NN = 1, 2, 3, 4
MODE = {"auto": 0, "lockstep": 1, "L": 1, "independent": 2, "N": 2}
MEM_HOST, MEM_DEVICE = 0, 1
VARIANT = {"autoropes": 0, "recursive": 1, "stack": 2, "split": 3, "groups": 4, "ropes": 5}
MAX_HEIGHT, MAX_DIM, MAX_K = 48, 16, 32
BH_POINTS_PER_LANE = 2
TILE_POINTS = {"oct": 32 * BH_POINTS_PER_LANE, "kd": 32, "vp": 32, "nn": 32}  # points per warp tile (tt_stats warp_*)


class TTError(RuntimeError):
    def __init__(self, status: int, where: str, cuda: int = 0):
        msg = f"{where}: {STATUS.get(status, status)}"
        if cuda:
            msg += f" (cudaError {cuda})"
        super().__init__(msg)
        self.status = status


class tt_tree_desc(C.Structure):
    _fields_ = [
        ("kind", C.c_int32), ("dim", C.c_int32), ("height", C.c_int32), ("leaf_size", C.c_int32),
        ("n_nodes", C.c_int64), ("n_points", C.c_int64),
        ("first_child", C.c_void_p), ("skip", C.c_void_p), ("level", C.c_void_p),
        ("pbegin", C.c_void_p), ("pcount", C.c_void_p),
        ("split_dim", C.c_void_p), ("split", C.c_void_p), ("lo", C.c_void_p), ("hi", C.c_void_p),
        ("com", C.c_void_p), ("body", C.c_void_p),
        ("root_center", C.c_double * 3), ("root_side", C.c_double),
        ("in_child", C.c_void_p), ("out_child", C.c_void_p),
        ("r_in_max", C.c_void_p), ("r_out_min", C.c_void_p),
        ("tree_order", C.c_void_p), ("points", C.c_void_p),
    ]


class tt_tree_info(C.Structure):
    _fields_ = [
        ("kind", C.c_int32), ("dim", C.c_int32), ("dim_padded", C.c_int32), ("height", C.c_int32),
        ("n_nodes", C.c_int64), ("n_points", C.c_int64),
        ("top_levels", C.c_int32), ("top_count", C.c_int32),
        ("device_bytes", C.c_int64), ("device_blob", C.c_void_p),
    ]


class tt_stats(C.Structure):
    _fields_ = [("visits", C.c_void_p), ("warp_fetches", C.c_void_p), ("warp_steps", C.c_void_p),
                ("warp_mode", C.c_void_p), ("visit_hash", C.c_void_p), ("visit_set", C.c_void_p),
                ("point_tests", C.c_void_p)]


class tt_traverse_opts(C.Structure):
    _fields_ = [("mode", C.c_int32), ("auto_min_depth", C.c_int32), ("order", C.c_void_p),
                ("stats", C.c_void_p), ("block_threads", C.c_int32), ("ctas_per_sm", C.c_int32),
                ("variant", C.c_int32), ("switch_below", C.c_int32)]


# name -> (restype, argtypes); every function declared in include/tt.h
P, I32, I64, F, D, SZ = C.c_void_p, C.c_int32, C.c_int64, C.c_float, C.c_double, C.c_size_t
SIGNATURES = {
    "tt_build_kd": (I32, [P, I64, I32, I32, I32, P]),
    "tt_build_oct": (I32, [P, I64, P]),
    "tt_build_vp": (I32, [P, I64, I32, I32, P]),
    "tt_build_nn": (I32, [P, I64, I32, I32, P]),
    "tt_host_tree_free": (None, [P]),
    "tt_host_tree_desc": (I32, [P, P]),
    "tt_tree_pack_size": (I32, [P, P]),
    "tt_tree_pack": (I32, [P, P, SZ]),
    "tt_tree_from_blob": (I32, [P, SZ, I32, P, P]),
    "tt_tree_upload": (I32, [P, P, P]),
    "tt_build_oct_device": (I32, [P, I64, P, P]),
    "tt_build_oct_device_order": (I32, [P, I64, P, P, P]),
    "tt_build_kd_device": (I32, [P, I64, I32, I32, I32, P, P]),
    "tt_build_vp_device": (I32, [P, I64, I32, I32, P, P]),
    "tt_build_nn_device": (I32, [P, I64, I32, I32, P, P]),
    "tt_tree_download": (I32, [P, P, SZ]),
    "tt_tree_copy_blob": (I32, [P, P, SZ, I32, P]),
    "tt_kick_drift": (I32, [P, P, P, I64, F, F, P]),
    "tt_kick_drift_permuted": (I32, [P, P, P, P, P, I64, F, F, P, P, P, P]),
    "tt_tree_free": (I32, [P]),
    "tt_tree_get_info": (I32, [P, P]),
    "tt_sort_points": (I32, [P, P, I64, I32, P, P, P]),
    "tt_schedule_tiles": (I32, [P, P, I64, I32, P, P, P]),
    "tt_traverse_bh": (I32, [P, P, P, I64, F, F, P, P, P]),
    "tt_traverse_pc": (I32, [P, P, I64, I32, F, P, P, P]),
    "tt_traverse_knn": (I32, [P, P, I64, I32, I32, P, P, P, P]),
    "tt_traverse_vp": (I32, [P, P, I64, I32, P, P, P, P]),
    "tt_traverse_nn": (I32, [P, P, I64, I32, P, P, P, P]),
    "tt_diag_chase": (I32, [P, I64, I32, I64, I32, P, P]),
    "tt_diag_l2read": (I32, [P, I64, I32, P, P]),
    "tt_status_string": (C.c_char_p, [I32]),
    "tt_last_cuda_error": (I32, []),
    "tt_build_info": (C.c_char_p, []),
}

_lib = None


def load():
    """Load libtt.so (raises if it has not been built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'` "
                              "(no CPU fallback exists)")
        L = C.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def check(status: int, where: str):
    if status != TT_OK:
        cuda = load().tt_last_cuda_error() if status == -2 else 0
        raise TTError(status, where, cuda)
