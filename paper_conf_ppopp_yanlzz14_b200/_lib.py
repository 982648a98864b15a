"""ctypes declarations of include/yaspmv.h (argument marshalling only).

Loads the in-tree ``libyaspmv.so`` built by ``make`` / ``__graft_entry__.build()``.
There is no fallback: if the library is missing, importing the package raises.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# YASPMV_LIB_PATH: development override (A/B builds of the same sources); default in-tree
LIB_PATH = os.environ.get("YASPMV_LIB_PATH") or os.path.join(_HERE, "libyaspmv.so")

# status codes / enums (yaspmv.h)
OK, EINVAL, ENOMEM, ECUDA, EUNSUPPORTED = 0, 1, 2, 3, 4
F32, F64 = 0, 1
COL_AUTO, COL_U16, COL_I32, COL_DELTA16 = 0, 1, 2, 3
EMPTY_AUTO, EMPTY_FILLER, EMPTY_MAP = 0, 1, 2
KEEP_HOST, DROP_CSR, GPU_ENCODE, TICKET_IDS, NO_PDL, FORCE_HANDOFF = 1, 2, 4, 8, 16, 32
ARR = {"flags": 0, "col": 1, "col_delta": 2, "val0": 3, "val1": 4, "val2": 5, "val3": 6,
       "seg_row": 7, "zero_rows": 8, "cta_seg0": 9, "fre": 10,
       # panel-sliced BCCOO+ band stream
       "band_flags": 11, "band_col16": 12, "band_val": 13, "band_panel_blk0": 14, "band_slice_ptr": 15,
       "band_stop_ptr": 16, "band_first_row": 17, "band_tile_rank": 18, "band_far_col": 19, "band_far_blk0": 20}
FAR_SEPARATE, FAR_IN_PANEL = 1, 2  # yaspmv_params.band_far (include/yaspmv.h)
PANEL_BT, PANEL_BC = 16, 32  # band stream tile: 16 blocks x 32 threads (csrc/panel.hpp PANEL_BT, PANEL_WT)

MAX_RANKS = 8  # YASPMV_MAX_RANKS
IPC_HANDLE_BYTES = 64

# every symbol include/yaspmv.h declares (checked by tests/test_abi.py)
EXPORTED = ["yaspmv_build_csr", "yaspmv_build_coo", "yaspmv_free", "yaspmv_spmv", "yaspmv_spmv_host",
            "yaspmv_tune", "yaspmv_reencode", "yaspmv_get_info", "yaspmv_export", "yaspmv_export_device",
            "yaspmv_nrm2sq", "yaspmv_nrm2sq_scratch_bytes", "yaspmv_export_device_range", "yaspmv_scale", "yaspmv_last_error",
            "yaspmv_version", "yaspmv_launches_per_spmv", "yaspmv_spmv_host_async", "yaspmv_host_sync",
            "yaspmv_spmv_power", "yaspmv_launches_per_power_step", "yaspmv_tune_ex",
            "yaspmv_comm_create", "yaspmv_comm_ipc_handle", "yaspmv_comm_open_ipc", "yaspmv_comm_connect_local",
            "yaspmv_comm_x", "yaspmv_comm_begin", "yaspmv_power_step_fused", "yaspmv_comm_wait",
            "yaspmv_comm_norm2_device", "yaspmv_comm_seq", "yaspmv_comm_check", "yaspmv_launches_per_fused_step",
            "yaspmv_comm_free", "yaspmv_debug_spin_tile", "yaspmv_profile_begin", "yaspmv_profile_end",
            "yaspmv_comm_mc_supported", "yaspmv_comm_mc_create", "yaspmv_comm_mc_import",
            "yaspmv_comm_mc_add_device", "yaspmv_comm_mc_bind", "yaspmv_comm_mc_active", "yaspmv_comm_mc_release", "yaspmv_l2_persist",
            # include/yaspmv_ablation.h
            "yaspmv_ablation_spmv", "yaspmv_ablation_tree", "yaspmv_ablation_tree_scratch_bytes"]


class Params(ctypes.Structure):
    _fields_ = [("block_h", ctypes.c_int32), ("block_w", ctypes.c_int32), ("slices", ctypes.c_int32),
                ("thread_tile", ctypes.c_int32), ("cta_size", ctypes.c_int32), ("col_mode", ctypes.c_int32),
                ("empty_mode", ctypes.c_int32), ("flags", ctypes.c_int32), ("result_cache", ctypes.c_int32),
                ("tiles_per_cta", ctypes.c_int32), ("band", ctypes.c_int32), ("panel_rows", ctypes.c_int32),
                ("slice_width", ctypes.c_int32), ("band_col0", ctypes.c_int32), ("band_far", ctypes.c_int32)]

    def as_dict(self):
        return {k: int(getattr(self, k)) for k, _ in self._fields_}


class Info(ctypes.Structure):
    _fields_ = [("m", ctypes.c_int64), ("n", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("MB", ctypes.c_int64), ("NB", ctypes.c_int64), ("SW", ctypes.c_int64),
                ("nnzb", ctypes.c_int64), ("nnzb_pad", ctypes.c_int64), ("ntiles", ctypes.c_int64),
                ("n_stops", ctypes.c_int64), ("n_filler", ctypes.c_int64), ("n_zero_rows", ctypes.c_int64),
                ("format_bytes", ctypes.c_int64), ("alg_bytes", ctypes.c_int64),
                ("footprint_bytes", ctypes.c_int64), ("params", Params), ("dtype", ctypes.c_int32),
                ("device", ctypes.c_int32), ("has_seg_row", ctypes.c_int32), ("regs_per_thread", ctypes.c_int32),
                ("build_seconds", ctypes.c_double), ("tune_seconds", ctypes.c_double),
                ("tune_candidates", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("band_blocks", ctypes.c_int64), ("band_blocks_pad", ctypes.c_int64), ("band_panels", ctypes.c_int64),
                ("band_slices", ctypes.c_int64), ("band_stops", ctypes.c_int64),
                ("band_format_bytes", ctypes.c_int64), ("band_far_blocks_pad", ctypes.c_int64)]

    def as_dict(self):
        d = {}
        for k, _ in self._fields_:
            v = getattr(self, k)
            d[k] = v.as_dict() if isinstance(v, Params) else v
        return d


class YaspmvError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"yaspmv status {status}: {msg}")
        self.status = status


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `make -C {_HERE}` or __graft_entry__.build() "
                          "(there is no CPU fallback)")
    lib = ctypes.CDLL(LIB_PATH)
    vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
    H = ctypes.c_void_p  # opaque handle
    sig = {
        "yaspmv_build_csr": ([i64, i64, vp, vp, vp, ctypes.c_int, ctypes.POINTER(Params), i32, ctypes.POINTER(H)],
                             ctypes.c_int),
        "yaspmv_build_coo": ([i64, i64, i64, vp, vp, vp, ctypes.c_int, ctypes.POINTER(Params), i32,
                              ctypes.POINTER(H)], ctypes.c_int),
        "yaspmv_free": ([H], None),
        "yaspmv_spmv": ([H, vp, vp, vp], ctypes.c_int),
        "yaspmv_spmv_host": ([H, vp, vp, vp], ctypes.c_int),
        "yaspmv_tune": ([H, vp, ctypes.POINTER(Params)], ctypes.c_int),
        "yaspmv_tune_ex": ([H, vp, ctypes.POINTER(Params), i32], ctypes.c_int),
        "yaspmv_ablation_spmv": ([H, i32, vp, vp, vp], ctypes.c_int),
        "yaspmv_ablation_tree": ([vp, vp, vp, vp, vp, i64, vp, vp, i64, ctypes.c_int, vp, i64, vp], ctypes.c_int),
        "yaspmv_ablation_tree_scratch_bytes": ([i64], i64),
        "yaspmv_reencode": ([H, ctypes.POINTER(Params)], ctypes.c_int),
        "yaspmv_get_info": ([H, ctypes.POINTER(Info)], ctypes.c_int),
        "yaspmv_export": ([H, i32, vp, i64, ctypes.POINTER(i64)], ctypes.c_int),
        "yaspmv_export_device": ([H, i32, vp, i64, ctypes.POINTER(i64)], ctypes.c_int),
        "yaspmv_export_device_range": ([H, i32, i64, i64, vp, i64, ctypes.POINTER(i64)], ctypes.c_int),
        "yaspmv_nrm2sq": ([vp, i64, ctypes.c_int, vp, vp, vp], ctypes.c_int),
        "yaspmv_nrm2sq_scratch_bytes": ([i64], i64),
        "yaspmv_scale": ([vp, vp, i64, ctypes.c_int, vp, vp], ctypes.c_int),
        "yaspmv_last_error": ([], ctypes.c_char_p),
        "yaspmv_version": ([], ctypes.c_char_p),
        "yaspmv_launches_per_spmv": ([H], i32),
        "yaspmv_spmv_host_async": ([H, vp, vp, vp], ctypes.c_int),
        "yaspmv_host_sync": ([H], ctypes.c_int),
        "yaspmv_spmv_power": ([H, vp, vp, vp, vp, vp], ctypes.c_int),
        "yaspmv_launches_per_power_step": ([H], i32),
        "yaspmv_comm_create": ([i32, i32, i32, i64, ctypes.c_int, i32, ctypes.POINTER(H)], ctypes.c_int),
        "yaspmv_comm_ipc_handle": ([H, vp, i64], ctypes.c_int),
        "yaspmv_comm_open_ipc": ([H, vp, i64], ctypes.c_int),
        "yaspmv_comm_connect_local": ([H, ctypes.POINTER(H), i32], ctypes.c_int),
        "yaspmv_comm_x": ([H, i32], vp),
        "yaspmv_comm_begin": ([H], ctypes.c_int),
        "yaspmv_power_step_fused": ([H, H, vp], ctypes.c_int),
        "yaspmv_comm_wait": ([H, vp], ctypes.c_int),
        "yaspmv_comm_norm2_device": ([H], vp),
        "yaspmv_comm_seq": ([H], i64),
        "yaspmv_comm_check": ([H], ctypes.c_int),
        "yaspmv_launches_per_fused_step": ([H], i32),
        "yaspmv_comm_free": ([H], None),
        "yaspmv_comm_mc_supported": ([i32], i32),
        "yaspmv_comm_mc_create": ([H, ctypes.POINTER(i64)], ctypes.c_int),
        "yaspmv_comm_mc_import": ([H, i64, i64], ctypes.c_int),
        "yaspmv_comm_mc_add_device": ([H], ctypes.c_int),
        "yaspmv_comm_mc_bind": ([H], ctypes.c_int),
        "yaspmv_comm_mc_active": ([H], i32),
        "yaspmv_comm_mc_release": ([H], ctypes.c_int),
        "yaspmv_l2_persist": ([i32, i64, ctypes.POINTER(i64)], ctypes.c_int),
        "yaspmv_debug_spin_tile": ([], i64),
        "yaspmv_profile_begin": ([H], ctypes.c_int),
        "yaspmv_profile_end": ([H, vp, i32, ctypes.POINTER(i64)], ctypes.c_int),
    }
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    return lib


lib = _load()


def check(status: int) -> None:
    if status != OK:
        raise YaspmvError(status, lib.yaspmv_last_error().decode())
