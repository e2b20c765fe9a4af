"""ctypes declarations of include/sampleselect.h (marshalling only).

Loading fails loudly: there is no fallback if libsampleselect.so is missing
or a CUDA device is unusable.
"""
from __future__ import annotations

import ctypes
import os
import threading

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SS_LIB") or os.path.join(_PKG, "libsampleselect.so")

SS_FLOAT32, SS_FLOAT64, SS_INT32, SS_INT64 = 0, 1, 2, 3
SS_MAX_LEVELS = 32
ABLATION_MODES = {"shared": 0, "shared_wa": 1, "shared_fig6": 2, "global": 3, "global_wa": 4}
STATUS = {0: "SS_OK", 1: "SS_ERR_INVALID_ARGUMENT", 2: "SS_ERR_CUDA",
          3: "SS_ERR_OUT_OF_MEMORY", 4: "SS_ERR_NCCL", 5: "SS_ERR_INTERNAL"}

# every symbol include/sampleselect.h declares
EXPORTS = [
    "ss_create", "ss_destroy", "ss_get_config", "ss_set_config", "ss_last_stats", "ss_profile_totals",
    "ss_last_error", "ss_status_string", "ss_abi_version",
    "ss_select", "ss_select_host", "ss_approx_select", "ss_approx_select_host", "ss_select_upper", "ss_select_multi",
    "ss_step_sample", "ss_step_tree", "ss_step_count", "ss_step_count_ablation", "ss_quickselect", "ss_step_filter",
    "ss_step_search", "ss_step_keys_to_values", "ss_oracle_offset",
    "ss_nccl_unique_id", "ss_comm_init", "ss_local_group_create", "ss_local_group_destroy", "ss_comm_init_local",
    "ss_select_sharded", "ss_select_f32", "ss_select_f64", "ss_select_i32", "ss_select_i64", "ss_approx_select_f32",
]


class SSConfig(ctypes.Structure):
    _fields_ = [("b_exact", ctypes.c_int32), ("sample_size", ctypes.c_int32),
                ("base_case", ctypes.c_int32), ("ctas_per_sm", ctypes.c_int32),
                ("profile", ctypes.c_int32), ("b_deep", ctypes.c_int32),
                ("classify", ctypes.c_int32), ("seed", ctypes.c_uint64),
                ("fused_filter", ctypes.c_int32), ("spec_z", ctypes.c_float),
                ("spec_min_n", ctypes.c_int64), ("spec_max_frac", ctypes.c_float),
                ("shard_gather_log2", ctypes.c_int32), ("directed", ctypes.c_int32),
                ("upper_onepass", ctypes.c_int32)]


class SSStats(ctypes.Structure):
    _fields_ = [("levels", ctypes.c_int32), ("equality_exit", ctypes.c_int32),
                ("n_level", ctypes.c_int64 * SS_MAX_LEVELS),
                ("bucket", ctypes.c_int32 * SS_MAX_LEVELS),
                ("bytes_algorithmic", ctypes.c_double),
                ("launches", ctypes.c_int32),
                ("h2d_bytes", ctypes.c_int64), ("d2h_bytes", ctypes.c_int64),
                ("ms_kernel", (ctypes.c_float * 3) * SS_MAX_LEVELS),
                ("tl_us", ((ctypes.c_float * 2) * 3) * SS_MAX_LEVELS),
                ("lut_ctas", ctypes.c_int32), ("lut_marker", ctypes.c_int32),
                ("spec_levels", ctypes.c_int32), ("fused_levels", ctypes.c_int32),
                ("upper_greater", ctypes.c_int64), ("ms_upper_gather", ctypes.c_float),
                ("ms_quick", ctypes.c_float), ("incomplete_rounds", ctypes.c_int32),
                ("shard_levels", ctypes.c_int32), ("shard_ranks", ctypes.c_int32),
                ("workspace_bytes", ctypes.c_int64), ("upper_onepass", ctypes.c_int32),
                ("pad_", ctypes.c_int32)]


class SSError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


_lock = threading.Lock()
_lib = None


def lib() -> ctypes.CDLL:
    """Load libsampleselect.so (raises if it was not built)."""
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        if not os.path.exists(LIB_PATH):
            raise ImportError(
                f"{LIB_PATH} not found: build it with `python -m paper_conf_ipps_ribizela19_b200.build` "
                "(there is no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        vp, i32, i64, u64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64
        pctx = ctypes.POINTER(vp)
        st = ctypes.c_int
        L.ss_create.argtypes = [ctypes.c_int, pctx]
        L.ss_destroy.argtypes = [vp]
        L.ss_destroy.restype = None
        L.ss_get_config.argtypes = [vp, ctypes.POINTER(SSConfig)]
        L.ss_set_config.argtypes = [vp, ctypes.POINTER(SSConfig)]
        L.ss_last_stats.argtypes = [vp, ctypes.POINTER(SSStats)]
        L.ss_profile_totals.argtypes = [vp, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(i64),
                                        ctypes.POINTER(i64), ctypes.POINTER(i64), i32]
        L.ss_last_error.argtypes = [vp]
        L.ss_last_error.restype = ctypes.c_char_p
        L.ss_status_string.argtypes = [st]
        L.ss_status_string.restype = ctypes.c_char_p
        L.ss_abi_version.argtypes = []
        L.ss_select.argtypes = [vp, st, vp, i64, i64, vp, vp]
        L.ss_select_host.argtypes = [vp, st, vp, i64, i64, vp, vp]
        L.ss_approx_select.argtypes = [vp, st, vp, i64, i64, i32, vp, ctypes.POINTER(i64), vp]
        L.ss_approx_select_host.argtypes = [vp, st, vp, i64, i64, i32, vp, ctypes.POINTER(i64), vp]
        L.ss_select_upper.argtypes = [vp, st, vp, i64, i64, vp, vp, vp]
        L.ss_quickselect.argtypes = [vp, st, vp, i64, i64, vp, ctypes.POINTER(i64), i32, ctypes.POINTER(i32), vp]
        L.ss_select_multi.argtypes = [vp, st, vp, i64, i32, ctypes.POINTER(i64), vp, vp]
        L.ss_step_sample.argtypes = [vp, st, vp, i64, i32, i64, i64, vp, vp]
        L.ss_step_tree.argtypes = [vp, st, vp, i32, i32, i32, vp, vp, vp, vp]
        L.ss_step_count.argtypes = [vp, st, vp, i64, vp, i32, vp, vp, vp]
        L.ss_step_count_ablation.argtypes = [vp, st, vp, i64, vp, i32, i32, vp, vp]
        L.ss_step_filter.argtypes = [vp, st, vp, i64, vp, i32, vp, vp, vp]
        L.ss_step_search.argtypes = [vp, vp, i32, i64, vp, vp, vp]
        L.ss_step_keys_to_values.argtypes = [vp, st, vp, i64, vp, vp]
        L.ss_oracle_offset.argtypes = [st, vp, i64]
        L.ss_nccl_unique_id.argtypes = [ctypes.c_char_p]
        L.ss_comm_init.argtypes = [vp, ctypes.c_char_p, ctypes.c_int, ctypes.c_int]
        L.ss_local_group_create.argtypes = [ctypes.c_int, pctx]
        L.ss_local_group_destroy.argtypes = [vp]
        L.ss_local_group_destroy.restype = None
        L.ss_comm_init_local.argtypes = [vp, vp, ctypes.c_int]
        L.ss_select_sharded.argtypes = [vp, st, vp, i64, i64, vp, vp]
        for name in ("ss_select_f32", "ss_select_f64", "ss_select_i32", "ss_select_i64"):
            getattr(L, name).argtypes = [vp, i64, i64, vp]
        L.ss_approx_select_f32.argtypes = [vp, i64, i64, i32, vp, ctypes.POINTER(i64)]
        L.ss_oracle_offset.restype = i64
        for name in EXPORTS:
            if name not in ("ss_destroy", "ss_last_error", "ss_status_string", "ss_abi_version",
                            "ss_oracle_offset", "ss_local_group_destroy"):
                getattr(L, name).restype = st
        _lib = L
        return _lib
