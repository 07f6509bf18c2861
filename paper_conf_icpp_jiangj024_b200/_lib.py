"""ctypes declarations of libgd.so (include/gd.h).  Argument marshalling only.

The library is REQUIRED: importing this module raises if libgd.so is missing or does not
load.  There is no fallback path of any kind.
"""
from __future__ import annotations

import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libgd.so")
GD_MAX_HOPS = 8
GD_MAX_FANOUT = 256

STATUS = {0: "GD_OK", 1: "GD_ERR_INVALID", 2: "GD_ERR_OOM", 3: "GD_ERR_CUDA", 4: "GD_ERR_CAPACITY",
          5: "GD_ERR_DEVICE"}
DEV_BITS = {0x1: "GD_DEV_BAD_ID", 0x2: "GD_DEV_DUP_SEED", 0x4: "GD_DEV_UNDERFLOW", 0x8: "GD_DEV_STANDBY_DRY"}

# every entry point include/gd.h declares (checked by tests/test_abi.py)
EXPORTS = ["gd_last_error", "gd_version", "gd_graph_create", "gd_graph_destroy", "gd_sample_bounds", "gd_sample",
           "gd_buffer_init", "gd_buffer_destroy", "gd_extract", "gd_buffer_release", "gd_check_device_status",
           "gd_buffer_snapshot", "gd_buffer_set_state", "gd_buffer_side_stream", "gd_buffer_timing",
           "gd_buffer_timing_read", "gd_graph_timing", "gd_graph_timing_read", "gd_graph_sampler", "gd_buffer_config", "gd_buffer_stage_mode",
           "gd_buffer_peer_attach", "gd_buffer_peer_export_ipc", "gd_buffer_peer_attach_ipc", "gd_buffer_peer_stats",
           "gd_sage_create", "gd_sage_destroy", "gd_sage_step", "gd_sage_grads", "gd_sage_apply_sgd", "gd_sage_get",
           "gd_workspace_create", "gd_workspace_destroy", "gd_sample_ws", "gd_buffer_init_mod", "gd_debug_umma_gemm",
           "gd_buffer_policy_read"]


class GdError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class SampleOutC(ctypes.Structure):
    _fields_ = [("n_id", ctypes.c_void_p),
                ("rowptr", ctypes.c_void_p * GD_MAX_HOPS),
                ("col", ctypes.c_void_p * GD_MAX_HOPS),
                ("eid", ctypes.c_void_p * GD_MAX_HOPS),
                ("sizes", ctypes.c_void_p)]


_vp = ctypes.c_void_p
_i64 = ctypes.c_int64
_i32 = ctypes.c_int32
_st = ctypes.c_int


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `python tools/build_native.py` "
                          "(or __graft_entry__.build()); there is no non-CUDA fallback")
    L = ctypes.CDLL(LIB_PATH)
    L.gd_last_error.restype = ctypes.c_char_p
    L.gd_last_error.argtypes = []
    L.gd_version.restype = ctypes.c_int
    L.gd_graph_create.argtypes = [_vp, _vp, _i64, _i64, ctypes.c_int, ctypes.c_int, ctypes.POINTER(_vp)]
    L.gd_graph_destroy.argtypes = [_vp]
    L.gd_sample_bounds.argtypes = [_i64, _vp, _i32, _i64, _i64, _vp, _vp]
    L.gd_sample.argtypes = [_vp, _vp, _i64, _vp, _i32, ctypes.c_uint64, ctypes.c_uint32,
                            ctypes.POINTER(SampleOutC), _vp]
    L.gd_workspace_create.argtypes = [_vp, ctypes.POINTER(_vp)]
    L.gd_workspace_destroy.argtypes = [_vp]
    L.gd_sample_ws.argtypes = [_vp, _vp, _vp, _i64, _vp, _i32, ctypes.c_uint64, ctypes.c_uint32,
                               ctypes.POINTER(SampleOutC), _vp]
    L.gd_buffer_init.argtypes = [_vp, _i64, _i64, _i64, _i32, _i64, ctypes.c_int, ctypes.c_int, ctypes.POINTER(_vp)]
    L.gd_buffer_init_mod.argtypes = [_vp, _i64, _i64, _i64, _i64, _i32, _i64, ctypes.c_int, ctypes.c_int,
                                     ctypes.POINTER(_vp)]
    L.gd_buffer_destroy.argtypes = [_vp]
    L.gd_extract.argtypes = [_vp, _vp, _vp, _i64, _vp, _vp, _vp, _vp, _vp]
    L.gd_buffer_release.argtypes = [_vp, _vp, _vp, _i64, _vp]
    L.gd_check_device_status.argtypes = [_vp, ctypes.POINTER(ctypes.c_uint32)]
    L.gd_buffer_snapshot.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, ctypes.POINTER(_i64)]
    L.gd_buffer_set_state.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _i64]
    L.gd_buffer_side_stream.argtypes = [_vp]
    L.gd_buffer_side_stream.restype = _vp
    _dp = ctypes.POINTER(ctypes.c_double)
    L.gd_buffer_timing.argtypes = [_vp, ctypes.c_int]
    L.gd_buffer_timing_read.argtypes = [_vp, _dp, ctypes.POINTER(_i64)]
    L.gd_buffer_config.argtypes = [_vp, ctypes.c_int, ctypes.c_double, ctypes.c_int, ctypes.c_int]
    L.gd_buffer_stage_mode.argtypes = [_vp, ctypes.c_int]
    L.gd_buffer_policy_read.argtypes = [_vp, _dp, _i32]
    L.gd_buffer_peer_attach.argtypes = [_vp, ctypes.c_int, ctypes.POINTER(_vp)]
    L.gd_buffer_peer_export_ipc.argtypes = [_vp, ctypes.c_void_p, ctypes.c_int64]
    L.gd_buffer_peer_attach_ipc.argtypes = [_vp, ctypes.c_int, ctypes.c_void_p]
    L.gd_buffer_peer_stats.argtypes = [_vp, ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64)]
    L.gd_sage_create.argtypes = [_i32, _vp, _vp, _vp, _vp, ctypes.c_int, ctypes.POINTER(_vp)]
    L.gd_sage_destroy.argtypes = [_vp]
    L.gd_sage_step.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _vp, _vp]
    L.gd_sage_grads.argtypes = [_vp, ctypes.POINTER(_vp), ctypes.POINTER(_i64)]
    L.gd_sage_apply_sgd.argtypes = [_vp, ctypes.c_float, ctypes.c_float, _vp]
    L.gd_sage_get.argtypes = [_vp, _i32, _i32, _vp, _i64]
    L.gd_debug_umma_gemm.argtypes = [_i32, _vp, _i64, _vp, _i64, _vp, _i64, _i32, _i32, _vp, _vp, _i64, _i64, _i32,
                                     _i32, _i32, _i32, _vp]
    L.gd_graph_timing.argtypes = [_vp, ctypes.c_int]
    L.gd_graph_sampler.argtypes = [_vp, ctypes.c_int]
    L.gd_graph_timing_read.argtypes = [_vp, _dp, ctypes.POINTER(_i64)]
    for name in EXPORTS:
        if name not in ("gd_last_error", "gd_version", "gd_buffer_side_stream"):
            getattr(L, name).restype = _st
    return L


lib = _load()


def check(status: int):
    if status != 0:
        raise GdError(status, lib.gd_last_error().decode())
