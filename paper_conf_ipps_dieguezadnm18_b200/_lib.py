"""ctypes binding of libscanb200.so -- argument marshalling only.

Every entry point here forwards to the C-ABI declared in include/scan_b200.h; all scan
arithmetic runs in the library's CUDA kernels.  There is no CPU fallback: if the shared
library is missing or fails to load, importing this module raises.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libscanb200.so")

# enum values of include/scan_b200.h
OPS = {"add": 0, "max": 1}
KINDS = {"inclusive": 0, "exclusive": 1}
ALGOS = {"auto": 0, "lookback": 1, "cascade_cta": 2, "cascade_warp": 3, "three_stage": 4, "packed_warp": 5, "cluster": 6,
         "fused": 7}
STATUS = {0: "SCAN_OK", 1: "SCAN_ERR_INVALID_ARG", 2: "SCAN_ERR_UNSUPPORTED", 3: "SCAN_ERR_CUDA",
          4: "SCAN_ERR_NCCL", 5: "SCAN_ERR_NO_MEMORY", 6: "SCAN_ERR_NO_DEVICE"}

# every symbol include/scan_b200.h declares (checked by tests/test_abi.py)
EXPORTS = ("scan_status_string", "scan_abi_version", "scan_batch", "scan_workspace_bytes",
           "scan_batch_ex", "scan_batch_host", "scan_shard_totals", "scan_shard_scan",
           "scan_shard_workspace_bytes", "scan_debug_trace", "scan_plan", "scan_plan_ex", "scan_comm_create_nccl",
           "scan_comm_get_unique_id", "scan_comm_init_rank", "scan_comm_destroy", "scan_batch_multi",
           "scan_comm_create_peer", "scan_comm_peer_handle", "scan_comm_peer_open", "scan_autotune",
           "scan_autotune_clear")
PEER_HANDLE_BYTES = 128
SHARD = {"problems": 0, "elements": 1}


class ScanError(RuntimeError):
    def __init__(self, fn: str, code: int):
        super().__init__("%s failed: %s" % (fn, STATUS.get(code, code)))
        self.code = code


def _load() -> ctypes.CDLL:
    if not os.path.exists(LIB_PATH):
        raise ImportError("libscanb200.so not built (run __graft_entry__.build()); "
                          "there is no CPU fallback")
    lib = ctypes.CDLL(LIB_PATH)
    P, I64, I, SZ = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_size_t
    sig = {
        "scan_status_string": ([I], ctypes.c_char_p),
        "scan_abi_version": ([], I),
        "scan_batch": ([P, P, I64, I64, I, I, I, P], I),
        "scan_workspace_bytes": ([I64, I64, I, I, I, I64], SZ),
        "scan_batch_ex": ([P, P, I64, I64, I, I, I, I, I64, P, SZ, P], I),
        "scan_batch_host": ([P, P, I64, I64, I, I, I], I),
        "scan_shard_totals": ([P, I64, I64, I, I, P, P, SZ, P], I),
        "scan_shard_scan": ([P, P, I64, I64, I, I, I, P, I, I, P, SZ, P], I),
        "scan_shard_workspace_bytes": ([I64, I64], SZ),
        "scan_debug_trace": ([P, I64], I),
        "scan_plan": ([I64, I64, P, P, P, P], I),
        "scan_plan_ex": ([I64, I64, I, I, I, P, P, P, P], I),
        "scan_comm_create_nccl": ([P, I, I, P], I),
        "scan_comm_get_unique_id": ([P], I),
        "scan_comm_init_rank": ([P, I, I, P], I),
        "scan_comm_destroy": ([P], I),
        "scan_batch_multi": ([P, P, I64, I64, I, I, I, P, I, P, I], I),
        "scan_comm_create_peer": ([I, I, I64, P], I),
        "scan_comm_peer_handle": ([P, P], I),
        "scan_comm_peer_open": ([P, P], I),
        "scan_autotune": ([P, P, I64, I64, I, I, I, P, P, P, P], I),
        "scan_autotune_clear": ([], I),
    }
    for name, (args, res) in sig.items():
        fn = getattr(lib, name)
        fn.argtypes = args
        fn.restype = res
    return lib


lib = _load()


# look-back kernel variants of the library (scan_lookback.cu: lookback_variant_valid)
LOOKBACK_VARIANTS = (0, 1, 2, 3, 10)


def check(fn: str, code: int) -> None:
    if code != 0:
        raise ScanError(fn, code)
