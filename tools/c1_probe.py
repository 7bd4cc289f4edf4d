"""configs[0] latency: device time per call (CUDA graph of 50 calls) for every kernel choice."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
from paper_conf_ipps_dieguezadnm18_b200 import _lib
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from bench import device_time
for N in (1 << 20, 1 << 22):
    x = torch.empty(N, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32", 1)
    y = torch.empty_like(x)
    s = torch.cuda.Stream()
    cands = [("lookback", v) for v in range(_lib.lib_num_lookback_variants())] + [("three_stage", 0), ("three_stage", 1), ("three_stage", 2)]
    for algo, prm in cands:
        us = device_time(lambda: sb.scan(x, "add", out=y, algo=algo, param=prm, stream=s), s, 50) * 1e3
        print("N=2^%d %-12s %d  %7.2f us" % (N.bit_length() - 1, algo, prm, us), flush=True)
