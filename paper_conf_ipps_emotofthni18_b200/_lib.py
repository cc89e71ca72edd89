"""ctypes loader for libsat.so (the C ABI of include/sat.h).  Argument marshalling only.

The library is built in-tree by ``__graft_entry__.build()`` / ``python build_native.py``.  There is
no fallback: if libsat.so is missing or fails to load, importing the binding raises.
"""
from __future__ import annotations

import ctypes
import os
from pathlib import Path

_HERE = Path(__file__).resolve().parent
# SAT_LIB may point at an instrumented build (libsat_stats.so, tools/stats.py); never a fallback.
LIB_PATH = Path(os.environ["SAT_LIB"]) if os.environ.get("SAT_LIB") else _HERE / "libsat.so"

SAT_OK = 0
SAT_INT32, SAT_FLOAT32 = 0, 1
STATUS_NAMES = {
    0: "SAT_OK", 1: "SAT_ERR_INVALID_VALUE", 2: "SAT_ERR_MISALIGNED", 3: "SAT_ERR_UNSUPPORTED",
    4: "SAT_ERR_OUT_OF_MEMORY", 5: "SAT_ERR_CUDA", 6: "SAT_ERR_NCCL",
}

# every symbol declared in include/sat.h (checked by tests/test_abi.py against the header)
EXPORTS = (
    "sat_compute_i32", "sat_compute_f32", "sat_compute_u8", "sat_compute_f32_f64", "sat_compute_moments_f32", "sat_compute", "sat_compute_host", "sat_compute_batched", "sat_compute_batched_u8", "sat_box_sum", "sat_rect_sums",
    "sat_strip_colsum",
    "sat_carry_prefix", "sat_comm_get_unique_id", "sat_comm_init", "sat_comm_destroy", "sat_compute_sharded",
    "sat_chain_create", "sat_chain_export", "sat_chain_connect", "sat_chain_connect_local", "sat_chain_destroy",
    "sat_compute_chained",
    "sat_query_plan", "sat_set_tuning", "sat_set_max_ctas", "sat_num_variants", "sat_variant_info", "sat_debug_tile_order", "sat_debug_occupy", "sat_debug_stats", "sat_debug_trace",
    "sat_debug_workspace", "sat_release_stream_workspace", "sat_release_workspaces", "sat_status_string", "sat_last_error_detail", "sat_version",
)


class SatPlan(ctypes.Structure):
    _fields_ = [
        ("tile_rows", ctypes.c_int32), ("tile_cols", ctypes.c_int32), ("tma", ctypes.c_int32),
        ("ctas", ctypes.c_int32), ("tiles", ctypes.c_int64), ("aux_bytes", ctypes.c_int64),
        ("variant", ctypes.c_int32), ("order", ctypes.c_int32), ("family", ctypes.c_int32),
        ("reserved", ctypes.c_int32),
    ]


class SatWsInfo(ctypes.Structure):
    _fields_ = [("tile_rows", ctypes.c_int32), ("tile_cols", ctypes.c_int32), ("R", ctypes.c_int32),
                ("C", ctypes.c_int32), ("words", ctypes.c_int64)]


class SatError(RuntimeError):
    def __init__(self, status: int, fn: str, detail: str):
        self.status = status
        super().__init__(f"{fn} -> {STATUS_NAMES.get(status, status)}: {detail}")


_vp, _i64, _i32, _int = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_int


def _declare(lib):
    sig = {
        "sat_compute_i32": [_vp, _vp, _i64, _i64, _i64, _vp],
        "sat_compute_f32": [_vp, _vp, _i64, _i64, _i64, _vp],
        "sat_compute": [_int, _vp, _vp, _i64, _i64, _i64, _vp, _vp],
        "sat_compute_u8": [_vp, _i64, _vp, _i64, _i64, _i64, _vp],
        "sat_compute_f32_f64": [_vp, _i64, _vp, _i64, _i64, _i64, _vp],
        "sat_compute_moments_f32": [_vp, _i64, _vp, _i64, _i64, _i64, _vp],
        "sat_compute_host": [_int, _vp, _vp, _i64, _i64, _i64, _vp],
        "sat_compute_batched": [_int, _vp, _vp, _i64, _i64, _i64, _i64, _i64, _vp],
        "sat_compute_batched_u8": [_vp, _i64, _i64, _vp, _i64, _i64, _i64, _i64, _i64, _vp],
        "sat_box_sum": [_int, _vp, _vp, _i64, _i64, _i64, _i64, _i64, _vp],
        "sat_rect_sums": [_int, _vp, _i64, _i64, _i64, _vp, _i64, _vp, _vp],
        "sat_strip_colsum": [_int, _vp, _vp, _i64, _i64, _i64, _vp],
        "sat_carry_prefix": [_int, _vp, _int, _int, _i64, _vp, _vp],
        "sat_comm_get_unique_id": [ctypes.c_char_p],
        "sat_comm_init": [ctypes.POINTER(_vp), ctypes.c_char_p, _int, _int],
        "sat_comm_destroy": [_vp],
        "sat_compute_sharded": [_vp, _int, _vp, _vp, _i64, _i64, _i64, _vp],
        "sat_chain_create": [_int, _int, _i64, ctypes.POINTER(_vp)],
        "sat_chain_export": [_vp, ctypes.c_char_p],
        "sat_chain_connect": [_vp, ctypes.c_char_p],
        "sat_chain_connect_local": [ctypes.POINTER(_vp), _int],
        "sat_chain_destroy": [_vp],
        "sat_compute_chained": [_vp, _int, _vp, _vp, _i64, _i64, _i64, _vp],
        "sat_query_plan": [_int, _i64, _i64, _i64, _vp, _vp, ctypes.POINTER(SatPlan)],
        "sat_set_tuning": [_int, _int, _int],
        "sat_set_max_ctas": [_int],
        "sat_num_variants": [],
        "sat_variant_info": [_int, ctypes.POINTER(_i32), ctypes.POINTER(_i32)],
        "sat_debug_tile_order": [_i64, _i64, _int, _vp, _vp],
        "sat_debug_occupy": [_int, _i64, _i64, _vp],
        "sat_debug_stats": [_vp, _int, ctypes.POINTER(_int), ctypes.POINTER(_int)],
        "sat_debug_trace": [_vp, _i64, ctypes.POINTER(_i64)],
        "sat_debug_workspace": [_vp, _vp, _i64, ctypes.POINTER(SatWsInfo)],
        "sat_release_stream_workspace": [_vp],
        "sat_release_workspaces": [],
        "sat_status_string": [_int],
        "sat_last_error_detail": [],
        "sat_version": [],
    }
    for name, args in sig.items():
        f = getattr(lib, name, None)
        if f is None:
            if not os.environ.get("SAT_LIB"):
                raise ImportError(f"{LIB_PATH} lacks {name}: rebuild it (python build_native.py)")
            continue  # an older tuning build named by SAT_LIB: only the calls it has
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = _int
    lib.sat_status_string.restype = ctypes.c_char_p
    lib.sat_last_error_detail.restype = ctypes.c_char_p


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not LIB_PATH.exists():
            raise ImportError(f"{LIB_PATH} is missing: build it with `python build_native.py` "
                              "or `python -c 'import __graft_entry__ as g; g.build()'` (no fallback exists)")
        l = ctypes.CDLL(str(LIB_PATH))
        _declare(l)
        _lib = l
    return _lib


def check(status: int, fn: str) -> None:
    if status != SAT_OK:
        raise SatError(status, fn, lib().sat_last_error_detail().decode(errors="replace"))
