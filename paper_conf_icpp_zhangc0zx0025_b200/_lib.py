"""ctypes declarations of libwinrs.so (include/winrs.h, include/winrs_debug.h).

Argument marshalling only.  The library is loaded from the package directory
(built in-tree by tools/build.py / __graft_entry__.build()); if it is missing
every call raises — there is no fallback implementation.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# WINRS_LIB selects another in-tree build of the same library (an A/B kernel
# variant from `tools/build.py --variant TAG`, e.g. libwinrs_TAG.so).
LIB_PATH = os.path.join(_HERE, os.environ.get("WINRS_LIB", "libwinrs.so"))

WINRS_OK = 0
STATUS = {0: "WINRS_OK", 1: "WINRS_ERR_INVALID_ARG", 2: "WINRS_ERR_UNSUPPORTED",
          3: "WINRS_ERR_WORKSPACE", 4: "WINRS_ERR_CUDA", 5: "WINRS_ERR_HOST_ALLOC"}
DTYPES = {"f32": 0, "f16": 1, "bf16": 2}


class WinrsError(RuntimeError):
    def __init__(self, status: int, what: str = ""):
        self.status = status
        super().__init__(f"{what}: {STATUS.get(status, status)}")


class DeviceT(ctypes.Structure):
    _fields_ = [("num_sms", ctypes.c_int), ("cc_major", ctypes.c_int), ("cc_minor", ctypes.c_int)]


class PlanInfoT(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int) for n in
                ("N", "C", "H", "W", "K", "R", "S", "pad", "dtype", "Ho", "Wo",
                 "alpha0", "n0", "r0", "k0", "alpha1", "n1", "r1", "k1", "masked_cols",
                 "z_hat", "Z", "seg_h", "seg_w", "bands", "seg_cols",
                 "tile_k0", "tile_c0", "tile_k1", "tile_c1")] + [
        ("ctas_main", ctypes.c_longlong), ("ctas_resid", ctypes.c_longlong),
        ("ctas_reduce", ctypes.c_longlong), ("csplit", ctypes.c_int), ("workspace_bytes", ctypes.c_size_t),
        ("direct_flops", ctypes.c_double), ("ewm_flops", ctypes.c_double),
        ("D", ctypes.c_int), ("T", ctypes.c_int), ("Do", ctypes.c_int)]


# (name, restype, argtypes) of every exported symbol, in header order.
_i, _p, _s = ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t
SYMBOLS = [
    ("winrs_plan", _i, [_i] * 8 + [_i, ctypes.POINTER(_p)]),
    ("winrs_plan_for_device", _i, [_i] * 8 + [_i, ctypes.POINTER(DeviceT), ctypes.POINTER(_p)]),
    ("winrs_plan3d", _i, [_i] * 10 + [_i, ctypes.POINTER(_p)]),
    ("winrs_plan3d_for_device", _i, [_i] * 10 + [_i, ctypes.POINTER(DeviceT), ctypes.POINTER(_p)]),
    ("winrs_plan_info", _i, [_p, ctypes.POINTER(PlanInfoT)]),
    ("winrs_workspace_bytes", _s, [_p]),
    ("winrs_bfc", _i, [_p, _p, _p, _p, _p, _p]),
    ("winrs_bfc_strided", _i, [_p, _p, _p, ctypes.c_longlong, _p, _p, _p]),
    ("winrs_bfc_host", _i, [_p, _p, _p, _p, _p, _p, _p, _p, _p]),
    ("winrs_plan_destroy", None, [_p]),
    ("winrs_status_string", ctypes.c_char_p, [_i]),
    ("winrs_version", ctypes.c_char_p, []),
    ("winrs_launch_count", _i, [_p]),
    ("winrs_conv_plan", _i, [_i] * 9 + [_i, ctypes.POINTER(_p)]),
    ("winrs_conv_plan_for_device", _i, [_i] * 9 + [_i, ctypes.POINTER(DeviceT), ctypes.POINTER(_p)]),
    ("winrs_conv_workspace_bytes", _s, [_p]),
    ("winrs_conv_bfc_plan", _i, [_p, ctypes.POINTER(_p)]),
    ("winrs_conv_launch_count", _i, [_p]),
    ("winrs_fc", _i, [_p, _p, _p, _p, _p, _p]),
    ("winrs_bdc", _i, [_p, _p, _p, _p, _p, _p]),
    ("winrs_conv_plan_destroy", None, [_p]),
    ("winrs_ipc_alloc", _i, [_s, ctypes.POINTER(_p), ctypes.c_char_p]),
    ("winrs_ipc_open", _i, [ctypes.c_char_p, ctypes.POINTER(_p)]),
    ("winrs_ipc_close", _i, [_p]),
    ("winrs_ipc_free", _i, [_p]),
    ("winrs_allreduce_flag_bytes", _s, []),
    ("winrs_bfc_allreduce", _i, [_p, _p, _p, _p, _p, ctypes.POINTER(_p), ctypes.POINTER(_p), ctypes.POINTER(_p),
                                 _i, _i, ctypes.c_uint, _p]),
    # winrs_debug.h
    ("winrs_debug_emulate", _i, [_p, _p, _p, _p]),
    ("winrs_debug_transform", _i, [_i, _i, _i, _i, _p, _p]),
    ("winrs_debug_kernel_count", _i, []),
    ("winrs_debug_kernel_name", ctypes.c_char_p, [_i]),
    ("winrs_debug_plan_kernel", ctypes.c_char_p, [_p]),
    ("winrs_debug_plan_model_us", ctypes.c_double, [_p]),
]

_lib = None


def lib():
    """Load libwinrs.so (raises if it was not built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} not found: build it with `python tools/build.py` "
                               "(there is no non-CUDA fallback)")
        L = ctypes.CDLL(LIB_PATH)
        for name, res, args in SYMBOLS:
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def check(status: int, what: str):
    if status != WINRS_OK:
        raise WinrsError(status, what)
