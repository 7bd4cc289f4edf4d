"""CPU oracle for the batched scan -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package.  The product package
``paper_conf_ipps_dieguezadnm18_b200`` never imports it, and the two share no code.

The arithmetic lives in ``oracle_scan.c`` (plain sequential loops following PAPER.md:29
[§1], the scan definition, over the batch of PAPER.md:96 [§2.1]); this module only
marshals numpy arrays into it.  ``oracle/ref.py`` is an independent pure-Python twin for
tiny brute-force cases.

Parity status of each function (pins are in tests/test_oracle.py):
  scan(..., 'add', int)   pinned: Fig. 1 worked example, closed form i(i+1)/2 mod 2^32,
                          itertools/numpy brute force, linearity, last element = total.
  scan(..., 'max', *)     pinned: numpy maximum.accumulate, monotonicity, idempotence.
  scan(..., 'add', f32)   pinned: exact rational (fractions) sums on small inputs within
                          N*2^-53*sum|x|, closed form for 1..N while exact in fp64.
  sabs (|x| prefix)       pinned: numpy cumsum(|x|) per problem (G >= 3, reset at every
                          problem start), exclusive = sum over k < i (element 0 is 0),
                          one-shot and StreamAdd (tests/test_oracle.py, test_sabs_*).
  exclusive kind          pinned: excl[0] = identity, excl[i] = incl[i-1].
  totals()                pinned: equals the last element of the inclusive scan and a
                          brute-force sum.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle_scan.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

OPS = ("add", "max")
DTYPES = {"i32": np.int32, "u32": np.uint32, "f32": np.float32}


def build(force: bool = False) -> str:
    """Compile oracle_scan.c with plain gcc -O2 (no -ffast-math: IEEE adds)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            P = ctypes.c_void_p
            I = ctypes.c_int64
            for name in ("oracle_scan_add_u32", "oracle_scan_max_i32", "oracle_scan_max_u32",
                         "oracle_scan_max_f32"):
                fn = getattr(lib, name)
                fn.argtypes = [P, P, I, I, ctypes.c_int]
                fn.restype = None
            lib.oracle_scan_add_f32.argtypes = [P, P, P, I, I, ctypes.c_int]
            lib.oracle_scan_add_f32.restype = None
            lib.oracle_total_add_u32.argtypes = [P, P, I, I]
            lib.oracle_total_add_f32.argtypes = [P, P, I, I]
            lib.oracle_stream_add_u32.argtypes = [P, P, I, P, ctypes.c_int]
            lib.oracle_stream_add_f32.argtypes = [P, P, P, I, P, P, ctypes.c_int]
            _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def _as2d(x: np.ndarray, N: int | None):
    x = np.ascontiguousarray(x)
    if x.ndim == 1:
        if N is None:
            N = x.shape[0]
        G = x.shape[0] // N if N else 0
    else:
        G, N = x.shape
    return x, int(N), int(G)


def scan(x: np.ndarray, op: str, kind: str = "inclusive", N: int | None = None,
         with_abs: bool = False):
    """Sequential scan of every row of ``x`` (shape (G, N), or flat with row length N).

    Returns an array of the same shape: int32/uint32/float32 for the exact cases and
    float64 (unrounded fp64 prefix) for f32 add.  With ``with_abs`` (f32 add only) also
    returns the prefix of |x| used by the north_star tolerance.
    """
    if op not in OPS:
        raise ValueError(op)
    if kind not in ("inclusive", "exclusive"):
        raise ValueError(kind)
    excl = 1 if kind == "exclusive" else 0
    shape = x.shape
    x, N, G = _as2d(x, N)
    lib = _load()
    dt = x.dtype
    if dt == np.float32 and op == "add":
        out = np.empty(x.shape, np.float64)
        sabs = np.empty(x.shape, np.float64) if with_abs else None
        lib.oracle_scan_add_f32(_ptr(x), _ptr(out), _ptr(sabs) if with_abs else None, N, G, excl)
        out = out.reshape(shape)
        return (out, sabs.reshape(shape)) if with_abs else out
    if with_abs:
        raise ValueError("with_abs only applies to f32 add")
    out = np.empty(x.shape, dt)
    if op == "add" and dt in (np.int32, np.uint32):
        lib.oracle_scan_add_u32(_ptr(x), _ptr(out), N, G, excl)
    elif op == "max" and dt == np.int32:
        lib.oracle_scan_max_i32(_ptr(x), _ptr(out), N, G, excl)
    elif op == "max" and dt == np.uint32:
        lib.oracle_scan_max_u32(_ptr(x), _ptr(out), N, G, excl)
    elif op == "max" and dt == np.float32:
        lib.oracle_scan_max_f32(_ptr(x), _ptr(out), N, G, excl)
    else:
        raise ValueError("unsupported dtype %s" % dt)
    return out.reshape(shape)


def totals(x: np.ndarray, N: int | None = None) -> np.ndarray:
    """Per-problem add-reduction (u32 wrapping for ints, fp64 for f32)."""
    x, N, G = _as2d(x, N)
    lib = _load()
    if x.dtype == np.float32:
        out = np.empty(G, np.float64)
        lib.oracle_total_add_f32(_ptr(x), _ptr(out), N, G)
    else:
        out = np.empty(G, np.uint32)
        lib.oracle_total_add_u32(_ptr(x), _ptr(out), N, G)
    return out


def identity(op: str, dtype) -> float | int:
    """Reading R2: identity element used for exclusive element 0."""
    dtype = np.dtype(dtype)
    if op == "add":
        return 0
    if dtype == np.int32:
        return -(2 ** 31)
    if dtype == np.uint32:
        return 0
    return float("-inf")


class StreamAdd:
    """Streaming oracle for ONE long add-scan fed chunk by chunk (oracle_stream_add_*).

    ``feed(chunk)`` returns the reference of that chunk (u32 bits for ints; fp64 prefix and
    the |x| prefix for f32), continuing the running value from the previous chunk.
    """

    def __init__(self, dtype, kind: str = "inclusive"):
        self.dtype = np.dtype(dtype)
        self.excl = 1 if kind == "exclusive" else 0
        self.acc_u = np.zeros(1, np.uint32)
        self.acc_d = np.zeros(1, np.float64)
        self.acc_a = np.zeros(1, np.float64)

    def feed(self, x: np.ndarray):
        x = np.ascontiguousarray(x)
        lib = _load()
        n = x.shape[0]
        if self.dtype == np.float32:
            y = np.empty(n, np.float64)
            a = np.empty(n, np.float64)
            lib.oracle_stream_add_f32(_ptr(x), _ptr(y), _ptr(a), n, _ptr(self.acc_d), _ptr(self.acc_a), self.excl)
            return y, a
        y = np.empty(n, np.uint32)
        lib.oracle_stream_add_u32(_ptr(x), _ptr(y), n, _ptr(self.acc_u), self.excl)
        return y.view(self.dtype)
