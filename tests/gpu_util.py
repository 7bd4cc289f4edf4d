"""Helpers for the -m gpu parity tests: move seeded inputs to the device, run the CUDA path
through the C-ABI (via the thin binding), compare with the oracle element by element."""
from __future__ import annotations

import numpy as np
import torch

import inputs
import oracle

TORCH = {"i32": torch.int32, "u32": torch.uint32, "f32": torch.float32}
NP = {"i32": np.int32, "u32": np.uint32, "f32": np.float32}
DIST = {"i32": "i32", "u32": "u32", "f32": "f32s"}
COMBOS = [("add", "i32"), ("add", "u32"), ("add", "f32"), ("max", "i32"), ("max", "u32"), ("max", "f32")]
F32_TOL = 1e-5          # north_star: |err_i| <= 1e-5 * sum_{k<=i} |x_k|


def to_device(x: np.ndarray) -> torch.Tensor:
    t = torch.from_numpy(np.ascontiguousarray(x).view(np.int32)).cuda()
    return t.view(TORCH[{np.dtype(np.int32): "i32", np.dtype(np.uint32): "u32",
                         np.dtype(np.float32): "f32"}[x.dtype]])


def to_host(t: torch.Tensor, dtype) -> np.ndarray:
    return t.view(torch.int32).cpu().numpy().view(dtype)


def device_inputs(dist: str, count: int, seed: int, offset: int = 0, row_len: int = 0) -> torch.Tensor:
    dt = {np.int32: torch.int32, np.uint32: torch.uint32, np.float32: torch.float32}[inputs.DIST_DTYPE[dist]]
    t = torch.empty(count, dtype=torch.int32, device="cuda")
    inputs.fill_device(t, dist, seed, offset, row_len)
    return t.view(dt)


def assert_parity(got: np.ndarray, x: np.ndarray, op: str, kind: str, label: str = "") -> None:
    """Bit-exact for integer add/max and f32 max; north_star tolerance for f32 add."""
    if x.dtype == np.float32 and op == "add":
        ref, sabs = oracle.scan(x, op, kind, with_abs=True)
        err = np.abs(got.astype(np.float64) - ref)
        bad = err > F32_TOL * sabs
        if bad.any():
            i = np.argwhere(bad)[0]
            raise AssertionError("%s f32 add mismatch at %s: got %r ref %r sabs %r (%d bad)" % (
                label, tuple(i), got[tuple(i)], ref[tuple(i)], sabs[tuple(i)], int(bad.sum())))
    else:
        ref = oracle.scan(x, op, kind)
        if not np.array_equal(got, ref):
            bad = got != ref
            i = np.argwhere(bad)[0]
            raise AssertionError("%s mismatch at %s: got %r ref %r (%d bad)" % (
                label, tuple(i), got[tuple(i)], ref[tuple(i)], int(bad.sum())))


def spin_lib():
    """Build (once, in-tree, nvcc for sm_100a) and load tests/c/libspin.so, the SM-occupying
    spin kernel of tests/test_gpu_safety.py (test infrastructure, not the product)."""
    import ctypes
    import os
    import subprocess
    here = os.path.join(os.path.dirname(os.path.abspath(__file__)), "c")
    src, so = os.path.join(here, "spin.cu"), os.path.join(here, "libspin.so")
    if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
        tmp = so + ".tmp%d" % os.getpid()
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O2",
                               "-Xcompiler", "-fPIC", "-shared", "-o", tmp, src])
        os.replace(tmp, so)
    lib = ctypes.CDLL(so)
    lib.spin_launch.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_ulonglong, ctypes.c_void_p]
    lib.spin_launch.restype = ctypes.c_int
    return lib
