"""ctypes binding of include/fmmfft.h — argument marshalling only; every step of the FMM-FFT
runs inside libfmmfft.so. There is deliberately NO fallback: if the shared library is missing
or fails to load, importing this module raises."""
from __future__ import annotations

import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("FMMFFT_LIB") or os.path.join(_PKG, "libfmmfft.so")   # FMMFFT_LIB: a tuning build

SUCCESS, INVALID_VALUE, UNSUPPORTED, ALLOC_FAILED, CUDA_ERROR, NCCL_ERROR, NOT_INITIALIZED = range(7)
STATUS_NAMES = ["SUCCESS", "INVALID_VALUE", "UNSUPPORTED", "ALLOC_FAILED", "CUDA_ERROR", "NCCL_ERROR",
                "NOT_INITIALIZED"]
C64, C128 = 0, 1
FLAG_VIRTUAL, FLAG_PROFILE, FLAG_DEBUG, FLAG_INVERSE, FLAG_DIRECT, FLAG_REAL, FLAG_VIRTUAL_NCCL = 1, 2, 4, 8, 16, 32, 64

# every symbol include/fmmfft.h declares (checked by tests/test_abi.py)
EXPORTS = [
    "fmmfft_get_unique_id", "fmmfft_comm_init", "fmmfft_comm_destroy", "fmmfft_plan", "fmmfft_plan_ex",
    "fmmfft_execute", "fmmfft_execute_host", "fmmfft_destroy", "fmmfft_get_info", "fmmfft_stage_times",
    "fmmfft_stage_name", "fmmfft_debug_buffer", "fmmfft_last_error", "fmmfft_version", "fmmfft_autotune",
]


class Info(ctypes.Structure):
    _fields_ = [("N", ctypes.c_longlong), ("P", ctypes.c_int), ("G", ctypes.c_int), ("B", ctypes.c_int),
                ("Q", ctypes.c_int), ("M_L", ctypes.c_int), ("L", ctypes.c_int), ("precision", ctypes.c_int),
                ("M", ctypes.c_longlong), ("level_gather", ctypes.c_int), ("n_stages", ctypes.c_int),
                ("workspace_bytes", ctypes.c_size_t), ("kernels_per_execute", ctypes.c_int),
                ("variant", ctypes.c_uint), ("top_level", ctypes.c_int)]


class Tune(ctypes.Structure):
    _fields_ = [("P", ctypes.c_int), ("B", ctypes.c_int), ("Q", ctypes.c_int), ("M_L", ctypes.c_int),
                ("ms", ctypes.c_float), ("error", ctypes.c_double), ("candidates", ctypes.c_int)]


class FmmfftError(RuntimeError):
    def __init__(self, status: int, msg: str):
        self.status = status
        name = STATUS_NAMES[status] if 0 <= status < len(STATUS_NAMES) else str(status)
        super().__init__(f"fmmfft {name}: {msg}")


def _load() -> ctypes.CDLL:
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built: run `python -m paper_conf_sc_cecka17_b200.build` "
                          "(there is no CPU fallback)")
    lib = ctypes.CDLL(LIB_PATH, mode=ctypes.RTLD_GLOBAL)
    vp, i, ll, u, st = ctypes.c_void_p, ctypes.c_int, ctypes.c_longlong, ctypes.c_uint, ctypes.c_int
    sig = {
        "fmmfft_get_unique_id": (st, [ctypes.c_char_p]),
        "fmmfft_comm_init": (st, [i, i, ctypes.c_char_p]),
        "fmmfft_comm_destroy": (st, []),
        "fmmfft_plan": (st, [ctypes.POINTER(vp), ll, i, i, i, i, i]),
        "fmmfft_plan_ex": (st, [ctypes.POINTER(vp), ll, i, i, i, i, i, i, u]),
        "fmmfft_execute": (st, [vp, vp, vp, vp]),
        "fmmfft_execute_host": (st, [vp, vp, vp, vp]),
        "fmmfft_destroy": (st, [vp]),
        "fmmfft_get_info": (st, [vp, ctypes.POINTER(Info)]),
        "fmmfft_stage_times": (st, [vp, ctypes.POINTER(ctypes.c_float), i, ctypes.POINTER(i)]),
        "fmmfft_stage_name": (ctypes.c_char_p, [i]),
        "fmmfft_debug_buffer": (st, [vp, i, i, i, ctypes.POINTER(vp), ctypes.POINTER(ctypes.c_size_t)]),
        "fmmfft_last_error": (ctypes.c_char_p, []),
        "fmmfft_version": (ctypes.c_char_p, []),
        "fmmfft_autotune": (st, [ll, i, i, ctypes.c_double, i, ctypes.POINTER(Tune)]),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype, f.argtypes = res, args
    return lib


lib = _load()


def check(status: int) -> None:
    if status != SUCCESS:
        raise FmmfftError(status, lib.fmmfft_last_error().decode())
