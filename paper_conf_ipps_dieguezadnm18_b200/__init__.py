"""B200-native batched and sharded scan (prefix sum) -- Python binding.

Diéguez, Amor, Doallo, Nukada, Matsuoka, "Efficient Solving of Scan Primitive on Multi-GPU
Systems" (IPDPS 2018 workshops).  The operation is the scan of PAPER.md:29 [§1] over a
batch of G problems of N elements (PAPER.md:96 [§2.1]); problems larger than one GPU are
split across GPUs (PAPER.md:191-205 [§4]; see ``multi.py``).

This module only marshals torch tensors into the C-ABI of ``libscanb200.so``
(include/scan_b200.h).  Torch provides device memory and streams; every step of the scan
runs in the library's sm_100a kernels.  There is no CPU fallback.
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

from . import _lib
from ._lib import ALGOS, KINDS, OPS, ScanError, check

__all__ = ["scan", "scan_host", "shard_totals", "shard_scan", "workspace_bytes", "ScanError",
           "DTYPES", "plan", "autotune", "autotune_clear"]

DTYPES = {torch.int32: 0, torch.uint32: 1, torch.float32: 2}
_NP_DTYPES = {np.dtype(np.int32): 0, np.dtype(np.uint32): 1, np.dtype(np.float32): 2}


def _shape(x: torch.Tensor):
    if x.dim() == 1:
        return x.shape[0], 1
    if x.dim() == 2:
        return x.shape[1], x.shape[0]
    raise ValueError("expected (N,) or (G, N), got %s" % (tuple(x.shape),))


def _dtype(x: torch.Tensor) -> int:
    try:
        return DTYPES[x.dtype]
    except KeyError:
        raise TypeError("dtype %s not supported (int32, uint32, float32)" % x.dtype) from None


def _stream(x: torch.Tensor, stream) -> int:
    if stream is None:
        stream = torch.cuda.current_stream(x.device)
    return stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)


def _require_cuda(*ts: torch.Tensor) -> None:
    for t in ts:
        if not t.is_cuda:
            raise ValueError("tensors must live on a CUDA device (no CPU fallback)")
        if not t.is_contiguous():
            raise ValueError("tensors must be contiguous (row-major, stride N)")


def scan(x: torch.Tensor, op: str = "add", kind: str = "inclusive", out: torch.Tensor | None = None,
         algo: str = "auto", param: int = -1, workspace: torch.Tensor | None = None,
         stream=None) -> torch.Tensor:
    """Scan each row of ``x`` ((G, N) or (N,)) into ``out`` (may be ``x`` itself).

    Calls ``scan_batch_ex`` on the current (or given) stream; asynchronous.
    """
    if out is None:
        out = torch.empty_like(x)
    _require_cuda(x, out)
    if out.shape != x.shape or out.dtype != x.dtype:
        raise ValueError("out must match x in shape and dtype")
    N, G = _shape(x)
    ws_ptr, ws_bytes = (None, 0)
    if workspace is not None:
        ws_ptr, ws_bytes = workspace.data_ptr(), workspace.numel() * workspace.element_size()
    with torch.cuda.device(x.device):
        rc = _lib.lib.scan_batch_ex(x.data_ptr(), out.data_ptr(), N, G, OPS[op], _dtype(x),
                                    KINDS[kind], ALGOS[algo], param, ws_ptr, ws_bytes,
                                    _stream(x, stream))
    check("scan_batch_ex", rc)
    return out


def workspace_bytes(N: int, G: int, op: str, dtype: torch.dtype, algo: str = "auto", param: int = -1) -> int:
    return int(_lib.lib.scan_workspace_bytes(N, G, OPS[op], DTYPES[dtype], ALGOS[algo], param))


def scan_host(x: np.ndarray, op: str = "add", kind: str = "inclusive",
              out: np.ndarray | None = None) -> np.ndarray:
    """End-to-end scan of a HOST array (numpy, (G, N) or (N,)) through ``scan_batch_host``:
    the library pipelines host->device copies, the device scan and device->host copies.
    Synchronous.  Pinned host memory (e.g. ``torch.empty(..., pin_memory=True).numpy()``)
    lets the copies overlap."""
    if x.dtype not in _NP_DTYPES:
        raise TypeError("dtype %s not supported" % x.dtype)
    if not x.flags.c_contiguous:
        raise ValueError("x must be C-contiguous")
    if out is None:
        out = np.empty_like(x)
    if out.shape != x.shape or out.dtype != x.dtype or not out.flags.c_contiguous:
        raise ValueError("out must match x")
    N, G = (x.shape[0], 1) if x.ndim == 1 else (x.shape[1], x.shape[0])
    rc = _lib.lib.scan_batch_host(x.ctypes.data, out.ctypes.data, N, G, OPS[op],
                                  _NP_DTYPES[x.dtype], KINDS[kind])
    check("scan_batch_host", rc)
    return out


def shard_totals(x_local: torch.Tensor, op: str = "add", totals: torch.Tensor | None = None,
                 workspace: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """Stage 1 + 2 on this rank's portion of every problem; returns ``totals`` (G int64
    slots: the 32-bit value in the low half, or the fp64 bits for f32 add)."""
    N, G = _shape(x_local)
    if totals is None:
        totals = torch.empty(G, dtype=torch.int64, device=x_local.device)
    _require_cuda(x_local, totals)
    ws_ptr, ws_bytes = (None, 0)
    if workspace is not None:
        ws_ptr, ws_bytes = workspace.data_ptr(), workspace.numel() * workspace.element_size()
    with torch.cuda.device(x_local.device):
        rc = _lib.lib.scan_shard_totals(x_local.data_ptr(), N, G, OPS[op], _dtype(x_local),
                                        totals.data_ptr(), ws_ptr, ws_bytes, _stream(x_local, stream))
    check("scan_shard_totals", rc)
    return totals


def shard_scan(x_local: torch.Tensor, all_totals: torch.Tensor, rank: int, ngpu: int,
               op: str = "add", kind: str = "inclusive", out: torch.Tensor | None = None,
               workspace: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """Stage 3 on this rank's portion: carry = totals of ranks < rank, then the chunk
    prefixes kept by ``shard_totals`` (same workspace / stream)."""
    if out is None:
        out = torch.empty_like(x_local)
    _require_cuda(x_local, out, all_totals)
    N, G = _shape(x_local)
    ws_ptr, ws_bytes = (None, 0)
    if workspace is not None:
        ws_ptr, ws_bytes = workspace.data_ptr(), workspace.numel() * workspace.element_size()
    with torch.cuda.device(x_local.device):
        rc = _lib.lib.scan_shard_scan(x_local.data_ptr(), out.data_ptr(), N, G, OPS[op],
                                      _dtype(x_local), KINDS[kind], all_totals.data_ptr(), rank, ngpu,
                                      ws_ptr, ws_bytes, _stream(x_local, stream))
    check("scan_shard_scan", rc)
    return out


ALGO_NAMES = {v: k for k, v in ALGOS.items()}
KERNEL_NAMES = {"lookback": "lookback_*_kernel (decoupled look-back)",
                "cascade_cta": "chunk_scan_kernel (one CTA per problem, cascade)",
                "cascade_warp": "warp_cascade_kernel (one warp per problem, cascade)",
                "three_stage": "chunk_reduce + aux_scan + chunk_scan kernels",
                "packed_warp": "packed_warp_kernel (k short problems per warp, segmented)",
                "cluster": "cluster_scan_kernel (one thread-block cluster per problem, DSMEM aggregates)",
                "fused": "fused_grid_kernel (three stages in one cooperative launch, tiles in registers)"}


def plan(x: torch.Tensor, out: torch.Tensor | None = None, op: str = "add",
         kind: str = "inclusive") -> tuple[str, int]:
    """The (algo, param) that algo='auto' picks for this tensor, op and kind (scan_plan_ex)."""
    N, G = _shape(x)
    a, pr = ctypes.c_int(0), ctypes.c_int64(0)
    with torch.cuda.device(x.device):
        check("scan_plan_ex", _lib.lib.scan_plan_ex(N, G, OPS[op], _dtype(x), KINDS[kind], x.data_ptr(),
                                                    (out if out is not None else x).data_ptr(),
                                                    ctypes.byref(a), ctypes.byref(pr)))
    return ALGO_NAMES[a.value], pr.value


def autotune(x: torch.Tensor, op: str = "add", kind: str = "inclusive", out: torch.Tensor | None = None,
             stream=None) -> tuple[str, int, float]:
    """Time every kernel family / parameter that takes this shape on x -> out (out is
    overwritten, must not be x) and make the fastest the AUTO choice for (device, N, G,
    alignment, op, dtype, kind) in this process (scan_autotune, the automated form of the paper's K search,
    PAPER.md:183).  Synchronous.  Returns (algo, param, microseconds per call)."""
    if out is None:
        out = torch.empty_like(x)
    _require_cuda(x, out)
    N, G = _shape(x)
    a, pr, us = ctypes.c_int(0), ctypes.c_int64(0), ctypes.c_float(0.0)
    with torch.cuda.device(x.device):
        rc = _lib.lib.scan_autotune(x.data_ptr(), out.data_ptr(), N, G, OPS[op], _dtype(x), KINDS[kind],
                                    _stream(x, stream), ctypes.byref(a), ctypes.byref(pr), ctypes.byref(us))
    check("scan_autotune", rc)
    return ALGO_NAMES[a.value], pr.value, us.value


def autotune_clear() -> None:
    """Forget every tuned choice (AUTO falls back to the static dispatch rules)."""
    check("scan_autotune_clear", _lib.lib.scan_autotune_clear())


def abi_version() -> int:
    return int(_lib.lib.scan_abi_version())
