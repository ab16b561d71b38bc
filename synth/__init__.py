"""Seeded synthetic inputs (host numpy generator + device twin in synth.cu).

See synth/synth.py for the generator definition.  ``device_fill_f16`` /
``device_fill_f32`` write generator elements straight into device memory (given
as an integer pointer) with values bit-identical to ``synth.fill_f16`` /
``synth.fill_f32``.
"""
from __future__ import annotations

import ctypes
import os

from .synth import *  # noqa: F401,F403
from .synth import scales_for, weight_sigma

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def lib() -> ctypes.CDLL:
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libsqsynth.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build()")
        L = ctypes.CDLL(path)
        for name in ("synth_fill_f16", "synth_fill_f32"):
            fn = getattr(L, name)
            fn.restype = ctypes.c_int
            fn.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64,
                           ctypes.c_float, ctypes.c_float, ctypes.c_int, ctypes.c_void_p]
        L.synth_fill_f32_host.restype = None
        L.synth_fill_f32_host.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64,
                                          ctypes.c_float, ctypes.c_float, ctypes.c_int]
        _LIB = L
    return _LIB


def device_fill_f16(ptr: int, seed: int, start: int, count: int, sigma: float, outliers: bool, stream: int = 0) -> None:
    s, so = scales_for(sigma, outliers)
    rc = lib().synth_fill_f16(ptr, seed, start, count, float(s), float(so), int(outliers), stream)
    if rc != 0:
        raise RuntimeError(f"synth_fill_f16 failed: cuda error {rc}")


def device_fill_f32(ptr: int, seed: int, start: int, count: int, sigma: float, outliers: bool, stream: int = 0) -> None:
    s, so = scales_for(sigma, outliers)
    rc = lib().synth_fill_f32(ptr, seed, start, count, float(s), float(so), int(outliers), stream)
    if rc != 0:
        raise RuntimeError(f"synth_fill_f32 failed: cuda error {rc}")


def device_weight_f16(ptr: int, seed: int, n: int, k: int, stream: int = 0) -> None:
    device_fill_f16(ptr, seed, 0, n * k, weight_sigma(k), True, stream)
