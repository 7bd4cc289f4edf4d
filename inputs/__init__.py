"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NO scan arithmetic.  It only defines a counter-based generator so that
both sides see bit-identical inputs (the input recipe):

    h(seed, idx) = splitmix64_mix(seed + (idx + 1) * 0x9E3779B97F4A7C15)      (mod 2^64)

i.e. element ``idx`` is the ``idx``-th output of the reference splitmix64 stream started
from state ``seed`` (for seed 0 the stream begins 0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4,
0x06C45D188009454F -- checked in tests/test_inputs.py).  ``idx`` is the GLOBAL element
index g*N + i (plus a rank offset when sharded), so a problem's values do not depend on
how it is split.

Distributions (each maps the 64-bit h to one 32-bit element with integer ops and exact
conversions only):
    i32     (int32)(uint32)h                 full range, wraps on add (PAPER.md:237 ints)
    u32     (uint32)h
    f32u    (float)(h >> 40) * 2^-24          U[0,1), exact
    f32s    (float)((h >> 39) - 2^24) * 2^-24 U[-1,1), exact
    small   (int32)(h % 2001) - 1000           small ints, no overflow in moderate N
    iota    (idx % row_len) + 1 as int32      the 1..N closed-form input (north_star)
    iotaf   (idx % row_len) + 1 as float32

The device twin is ``inputs/gen.cu`` (built into ``inputs/libinputs.so``); it implements
the same formulas and is checked bit-for-bit against this module in tests/test_gpu_*.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

GAMMA = np.uint64(0x9E3779B97F4A7C15)
M1 = np.uint64(0xBF58476D1CE4E5B9)
M2 = np.uint64(0x94D049BB133111EB)

DISTS = {"i32": 0, "u32": 1, "f32u": 2, "f32s": 3, "small": 4, "iota": 5, "iotaf": 6}
DIST_DTYPE = {"i32": np.int32, "u32": np.uint32, "f32u": np.float32, "f32s": np.float32,
              "small": np.int32, "iota": np.int32, "iotaf": np.float32}

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libinputs.so")


def splitmix64(seed: int, idx: np.ndarray) -> np.ndarray:
    """Counter-based splitmix64: the idx-th output of the stream with initial state seed."""
    with np.errstate(over="ignore"):
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + (idx.astype(np.uint64) + np.uint64(1)) * GAMMA
        z = (z ^ (z >> np.uint64(30))) * M1
        z = (z ^ (z >> np.uint64(27))) * M2
        z = z ^ (z >> np.uint64(31))
    return z


def generate(dist: str, count: int, seed: int, offset: int = 0, row_len: int = 0,
             chunk: int = 1 << 22) -> np.ndarray:
    """Host generator: elements offset .. offset+count-1 of distribution ``dist``."""
    dt = DIST_DTYPE[dist]
    out = np.empty(count, dt)
    for s in range(0, count, chunk):
        e = min(count, s + chunk)
        idx = np.arange(offset + s, offset + e, dtype=np.uint64)
        if dist in ("iota", "iotaf"):
            v = (idx % np.uint64(row_len)) + np.uint64(1)
            out[s:e] = v.astype(np.int64).astype(dt)
            continue
        h = splitmix64(seed, idx)
        if dist == "i32":
            out[s:e] = (h & np.uint64(0xFFFFFFFF)).astype(np.uint32).view(np.int32)
        elif dist == "u32":
            out[s:e] = (h & np.uint64(0xFFFFFFFF)).astype(np.uint32)
        elif dist == "f32u":
            out[s:e] = (h >> np.uint64(40)).astype(np.float32) * np.float32(2.0 ** -24)
        elif dist == "f32s":
            v = (h >> np.uint64(39)).astype(np.int64) - (1 << 24)
            out[s:e] = v.astype(np.float32) * np.float32(2.0 ** -24)
        elif dist == "small":
            out[s:e] = ((h % np.uint64(2001)).astype(np.int64) - 1000).astype(np.int32)
        else:
            raise ValueError(dist)
    return out


_dlib = None


def device_lib():
    """ctypes handle to the device generator (raises if it was not built)."""
    global _dlib
    if _dlib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError("inputs/libinputs.so missing: run __graft_entry__.build()")
        lib = ctypes.CDLL(LIB_PATH)
        lib.inputs_fill.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint64,
                                    ctypes.c_int64, ctypes.c_int, ctypes.c_int64, ctypes.c_void_p]
        lib.inputs_fill.restype = ctypes.c_int
        _dlib = lib
    return _dlib


def fill_device(tensor, dist: str, seed: int, offset: int = 0, row_len: int = 0, stream=None):
    """Fill a CUDA tensor (torch) in place with the same values ``generate`` would give."""
    import torch
    if stream is None:
        stream = torch.cuda.current_stream(tensor.device).cuda_stream
    rc = device_lib().inputs_fill(ctypes.c_void_p(tensor.data_ptr()), tensor.numel(), seed & (2**64 - 1),
                                  offset, DISTS[dist], row_len, ctypes.c_void_p(stream))
    if rc != 0:
        raise RuntimeError("inputs_fill failed with cuda error %d" % rc)
    return tensor
