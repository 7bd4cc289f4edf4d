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
    cands = [("lookback", v) for v in (1, 2, 3, 10)] + [("three_stage", k) for k in (0, 1, 2, 3, 4, 6, 8)]
    for algo, prm in cands:
        us = device_time(lambda: sb.scan(x, "add", out=y, algo=algo, param=prm, stream=s), s, 50) * 1e3
        print("N=2^%d %-12s %d  %7.2f us" % (N.bit_length() - 1, algo, prm, us), flush=True)
    # floors / context on the same harness: a plain device copy of the same bytes and
    # torch.cumsum (CUB DeviceScan underneath)
    z = torch.empty(N, dtype=torch.int64, device="cuda")
    for name, fn in [("torch copy_", lambda: y.copy_(x)),
                     ("torch cumsum(int32->int32)", lambda: torch.cumsum(x, 0, dtype=torch.int32, out=y)),
                     ("empty kernel (zero_ 1 elem)", lambda: y[:1].zero_())]:
        with torch.cuda.stream(s):
            us = device_time(fn, s, 50) * 1e3
        print("N=2^%d %-28s %7.2f us" % (N.bit_length() - 1, name, us), flush=True)
