"""ctypes binding of libspgemm.so (include/spgemm.h).  Argument marshalling only.

The product path has NO fallback: if the shared library is missing or the device is not
sm_100, calls raise.  Every step of the SpGEMM runs in the library's CUDA kernels.
"""
from __future__ import annotations

import ctypes
import os
from ctypes import POINTER, c_char_p, c_float, c_int, c_int32, c_int64, c_size_t, c_void_p

_HERE = os.path.dirname(os.path.abspath(__file__))
# SPGEMM_LIB: an alternative build of the same library (diagnostics: kernel variants side by side)
LIB_PATH = os.environ.get("SPGEMM_LIB") or os.path.join(_HERE, "libspgemm.so")

SPGEMM_F32, SPGEMM_F64 = 0, 1
MAX_GROUPS = 24

STATUS = {
    0: "SPGEMM_OK", 1: "SPGEMM_ERR_INVALID_ARG", 2: "SPGEMM_ERR_BAD_STATE", 3: "SPGEMM_ERR_OOM",
    4: "SPGEMM_ERR_CUDA", 5: "SPGEMM_ERR_INDEX_OVERFLOW", 6: "SPGEMM_ERR_NOT_SUPPORTED",
    7: "SPGEMM_ERR_INVALID_INPUT",
}

OPTIONS = {
    "sym_min_group": 0, "num_min_group": 1, "sym_fill_limit": 2, "streams": 3,
    "validate": 4, "lanes": 5, "workspace_budget": 6, "timing": 7, "long_row": 8, "range_hash": 9,
    "cluster": 10, "cluster_fill_limit": 11, "flat": 12, "graphs": 13, "range_warp": 14,
    "range_min_nprod": 15, "bitmap_rank": 16, "rank_acc": 17, "tiny": 18, "rank_l1_pct": 19, "rank_l1_pct_sym": 20,
    "batch": 21, "esc_pct": 22, "esc_groups": 23, "small": 24, "wsort": 25, "rank_big_sym": 26, "rank_big_shared": 27, "rank_mid": 28, "rank_gout": 29, "rank_big_max": 31,
}

# spgemm_kernel_t (include/spgemm.h): kernel family that ran each group
KERNELS = {0: "none", 1: "hash", 2: "rank", 3: "range", 4: "cluster", 5: "global", 6: "rank_big", 7: "tiny", 8: "batch", 9: "esc", 10: "wsort"}

# Group ids of the range-row kernels (spgemm_internal.cuh kSymRange / kNumRange).
SYM_RANGE_GROUP = 12
NUM_RANGE_GROUP = 14

# Symbols declared in include/spgemm.h (tests check the .so exports all of them).
EXPORTS = [
    "spgemm_create", "spgemm_symbolic", "spgemm_numeric", "spgemm_destroy",
    "spgemm_status_string", "spgemm_last_error", "spgemm_set_option", "spgemm_get_stats",
    "spgemm_group_bounds", "spgemm_get_grouping", "spgemm_row_partition", "spgemm_version",
]

ALLOC_FN = ctypes.CFUNCTYPE(c_void_p, c_size_t, c_void_p, c_void_p)
FREE_FN = ctypes.CFUNCTYPE(None, c_void_p, c_size_t, c_void_p, c_void_p)


class Allocator(ctypes.Structure):
    _fields_ = [("alloc", ALLOC_FN), ("free", FREE_FN), ("ctx", c_void_p)]


G = MAX_GROUPS


class Stats(ctypes.Structure):
    _fields_ = [
        ("m", c_int64), ("k", c_int64), ("n", c_int64), ("nnz_a", c_int64), ("nnz_b", c_int64),
        ("nnz_c", c_int64), ("nprod", c_int64), ("max_row_nprod", c_int64), ("max_row_nnz", c_int64),
        ("n_sym_groups", c_int32), ("n_num_groups", c_int32),
        ("sym_rows", c_int64 * G), ("num_rows", c_int64 * G),
        ("sym_nprod", c_int64 * G), ("num_nprod", c_int64 * G),
        ("sym_nnza", c_int64 * G), ("num_nnza", c_int64 * G),
        ("num_nnzc", c_int64 * G),
        ("sym_overflow_rows", c_int64),
        ("sym_group_ms", c_float * G), ("num_group_ms", c_float * G),
        ("setup_ms", c_float), ("symbolic_ms", c_float), ("scan_ms", c_float), ("numeric_ms", c_float),
        ("kernel_launches_symbolic", c_int64), ("kernel_launches_numeric", c_int64),
        ("workspace_bytes", c_int64), ("workspace_peak_bytes", c_int64),
        ("sym_overflow2_rows", c_int64), ("graph_replays", c_int64),
        ("sym_kernel", c_int32 * G), ("num_kernel", c_int32 * G),
    ]

    def to_dict(self) -> dict:
        out = {}
        for name, typ in self._fields_:
            v = getattr(self, name)
            out[name] = list(v) if isinstance(v, ctypes.Array) else v
        return out


_LIB = None


def load() -> ctypes.CDLL:
    """Load libspgemm.so; raise loudly when it was not built (no CPU fallback exists)."""
    global _LIB
    if _LIB is not None:
        return _LIB
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: build it with "
                           "`python -m paper_conf_icpp_nagasakanm17_b200.build` (there is no CPU fallback)")
    lib = ctypes.CDLL(LIB_PATH)
    H = c_void_p
    P = c_void_p
    lib.spgemm_create.argtypes = [POINTER(c_void_p), c_int, c_void_p, POINTER(Allocator)]
    lib.spgemm_symbolic.argtypes = [H, c_int64, c_int64, c_int64, P, P, P, P, P, POINTER(c_int64), POINTER(c_int64)]
    lib.spgemm_numeric.argtypes = [H, c_int, P, P, P, P]
    lib.spgemm_destroy.argtypes = [H]
    lib.spgemm_status_string.argtypes = [c_int]
    lib.spgemm_status_string.restype = c_char_p
    lib.spgemm_last_error.argtypes = [H]
    lib.spgemm_last_error.restype = c_char_p
    lib.spgemm_set_option.argtypes = [H, c_int, c_int64]
    lib.spgemm_get_stats.argtypes = [H, POINTER(Stats)]
    lib.spgemm_group_bounds.argtypes = [c_int, POINTER(c_int64), POINTER(c_int32)]
    lib.spgemm_get_grouping.argtypes = [H, c_int, P, P, P]
    lib.spgemm_row_partition.argtypes = [H, c_int64, c_int64, P, P, P, c_int32, P]
    lib.spgemm_version.argtypes = []
    lib.spgemm_version.restype = c_char_p
    for f in ("spgemm_create", "spgemm_symbolic", "spgemm_numeric", "spgemm_destroy", "spgemm_set_option",
              "spgemm_get_stats", "spgemm_group_bounds", "spgemm_get_grouping", "spgemm_row_partition"):
        getattr(lib, f).restype = c_int
    _LIB = lib
    return lib


class SpgemmError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


def check(status: int, handle=None, what: str = "") -> None:
    if status != 0:
        detail = ""
        if handle is not None:
            detail = (load().spgemm_last_error(handle) or b"").decode(errors="replace")
        raise SpgemmError(status, f"{what} {detail}".strip())


def group_bounds(phase: int):
    arr = (c_int64 * MAX_GROUPS)()
    n = c_int32()
    check(load().spgemm_group_bounds(phase, arr, ctypes.byref(n)), None, "spgemm_group_bounds")
    return [int(arr[i]) for i in range(n.value)]
