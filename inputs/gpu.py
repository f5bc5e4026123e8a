"""ctypes loader for inputs/libktiler_inputs.so (device twin of inputs/synth.py).

Fills caller-owned device memory (a torch uint8 CUDA tensor) with the same bytes
inputs.synth would produce.  No KTILER arithmetic lives here.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import synth

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libktiler_inputs.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `python __graft_entry__.py build` (or build()) first")
        L = ctypes.CDLL(path)
        L.ktin_gen_uniform.argtypes = [ctypes.c_void_p] + [ctypes.c_int64] * 8 + [ctypes.c_uint64, ctypes.c_void_p]
        L.ktin_gen_uniform.restype = ctypes.c_int
        L.ktin_gen_scene.argtypes = [ctypes.c_void_p] + [ctypes.c_int64] * 5 + [ctypes.c_uint64,
                                                                                 ctypes.POINTER(ctypes.c_int32),
                                                                                 ctypes.c_void_p]
        L.ktin_gen_scene.restype = ctypes.c_int
        _LIB = L
    return _LIB


def fill(kind: str, seed: int, dst_ptr: int, pitch: int, frame_stride: int, W: int, H: int,
         y0: int = 0, rows: int | None = None, f0: int = 0, F: int = 1, stream: int = 0) -> None:
    """Write rows [y0, y0+rows) of frames [f0, f0+F) of image ``kind(seed)`` (global size W x H)
    to dst (row pitch ``pitch`` bytes, frame stride ``frame_stride`` bytes)."""
    rows = H - y0 if rows is None else rows
    if kind == "uniform":
        rc = lib().ktin_gen_uniform(dst_ptr, pitch, frame_stride, W, H, y0, rows, f0, F, seed & synth.M64, stream)
        if rc:
            raise RuntimeError(f"ktin_gen_uniform: cuda error {rc}")
        return
    if kind != "scene":
        raise ValueError(kind)
    for f in range(F):
        s = seed + f0 + f
        rects = np.asarray(synth.scene_rects(s, W, H), dtype=np.int32).reshape(-1)
        rc = lib().ktin_gen_scene(dst_ptr + f * frame_stride, pitch, W, H, y0, rows, s & synth.M64,
                                  rects.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)), stream)
        if rc:
            raise RuntimeError(f"ktin_gen_scene: cuda error {rc}")
