"""Seeded, counter-based synthetic input generator (shared test/bench module).

This module is the ONLY code shared between the CUDA path's tests/bench and
the CPU oracle harness.  It holds none of the summed-area-table arithmetic: it
maps a pixel coordinate (seed, image, y, x) to an input value.  The numpy
implementation below and the C/CUDA implementation in ``satgen.h`` compute the
same function (checked by ``tests/test_satgen.py``).

Value recipe: 8u = top 8 bits of the hash; 32f =
top 24 bits * 2^-24 in [0, 1); 64f = top 53 bits * 2^-53 in [0, 1); the 64f
"dyadic24" mode uses the 32f mapping widened to double; "const" fills a value.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

KIND_U8, KIND_F32, KIND_F64 = 0, 1, 2
MODE_UNIFORM, MODE_DYADIC24, MODE_CONST = 0, 1, 2

KIND_OF_DTYPE = {np.dtype(np.uint8): KIND_U8, np.dtype(np.float32): KIND_F32,
                 np.dtype(np.float64): KIND_F64}
DTYPE_OF_KIND = {KIND_U8: np.uint8, KIND_F32: np.float32, KIND_F64: np.float64}

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libsatgen.so")

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def _mix64(z: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = z + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def bits(seed: int, img, y, x) -> np.ndarray:
    """64-bit hash of (seed, img, y, x); broadcasting numpy arrays allowed."""
    P = np.uint64(0x100000001B3)
    with np.errstate(over="ignore"):
        k = np.uint64(0xCBF29CE484222325) ^ np.uint64(seed)
        k = (k * P) ^ np.asarray(img, dtype=np.uint64)
        k = (k * P) ^ np.asarray(y, dtype=np.uint64)
        k = (k * P) ^ np.asarray(x, dtype=np.uint64)
    return _mix64(k)


def generate(kind: int, H: int, W: int, seed: int = 0, img: int = 0, y0: int = 0,
             mode: int = MODE_UNIFORM, value: float = 0.0) -> np.ndarray:
    """Return an H x W numpy image of the given kind (numpy reference path)."""
    dt = DTYPE_OF_KIND[kind]
    if mode == MODE_CONST:
        return np.full((H, W), value, dtype=dt)
    ys = np.arange(y0, y0 + H, dtype=np.uint64)[:, None]
    xs = np.arange(W, dtype=np.uint64)[None, :]
    b = bits(seed, img, ys, xs)
    if kind == KIND_U8:
        return (b >> np.uint64(56)).astype(np.uint8)
    if kind == KIND_F32:
        return ((b >> np.uint64(40)).astype(np.float32) * np.float32(1.0 / 16777216.0)).astype(np.float32)
    if mode == MODE_DYADIC24:
        return (b >> np.uint64(40)).astype(np.float64) * (1.0 / 16777216.0)
    return (b >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


_lib = None


def lib():
    """ctypes handle of libsatgen.so (built by __graft_entry__.build())."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH)
        i64, u64, dbl, vp = ctypes.c_int64, ctypes.c_uint64, ctypes.c_double, ctypes.c_void_p
        L.satgen_fill_device.argtypes = [ctypes.c_int, ctypes.c_int, u64, dbl, vp, i64, i64, i64,
                                         i64, i64, i64, i64, vp]
        L.satgen_fill_device.restype = ctypes.c_int
        L.satgen_fill_host.argtypes = [ctypes.c_int, ctypes.c_int, u64, dbl, vp, i64, i64, i64,
                                       i64, i64, i64, i64]
        L.satgen_fill_host.restype = ctypes.c_int
        _lib = L
    return _lib


def fill_host(arr: np.ndarray, seed: int = 0, img0: int = 0, y0: int = 0,
              mode: int = MODE_UNIFORM, value: float = 0.0) -> np.ndarray:
    """Fill a host numpy array [..., H, W] (last dim contiguous) via the C generator."""
    kind = KIND_OF_DTYPE[arr.dtype]
    H, W = arr.shape[-2], arr.shape[-1]
    batch = int(np.prod(arr.shape[:-2])) if arr.ndim > 2 else 1
    assert arr.strides[-1] == arr.itemsize
    img_stride = arr.strides[-3] if arr.ndim > 2 else H * arr.strides[-2]
    rc = lib().satgen_fill_host(kind, mode, seed, value, arr.ctypes.data, H, W, arr.strides[-2],
                                batch, img_stride, img0, y0)
    if rc != 0:
        raise RuntimeError(f"satgen_fill_host failed ({rc})")
    return arr


def fill_device(t, seed: int = 0, img0: int = 0, y0: int = 0, mode: int = MODE_UNIFORM,
                value: float = 0.0, stream=None):
    """Fill a CUDA torch tensor [..., H, W] on its current stream (device generator)."""
    import torch

    kinds = {torch.uint8: KIND_U8, torch.float32: KIND_F32, torch.float64: KIND_F64}
    kind = kinds[t.dtype]
    H, W = t.shape[-2], t.shape[-1]
    batch = 1
    for d in t.shape[:-2]:
        batch *= d
    es = t.element_size()
    assert t.stride(-1) == 1
    img_stride = t.stride(-3) * es if t.dim() > 2 else H * t.stride(-2) * es
    s = stream if stream is not None else torch.cuda.current_stream(t.device)
    rc = lib().satgen_fill_device(kind, mode, seed, value, t.data_ptr(), H, W, t.stride(-2) * es,
                                  batch, img_stride, img0, y0, s.cuda_stream)
    if rc != 0:
        raise RuntimeError(f"satgen_fill_device failed (cudaError {rc})")
    return t
