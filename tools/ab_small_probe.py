"""Latency-bound shapes for A/B of library builds: G = 1, N = 2^10 .. 2^21 and a few small
batches, us per call (CUDA graph of back-to-back calls).  One JSON line.

    python tools/ab_small_probe.py
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402
from tools.paper_sweep import device_ms  # noqa: E402

x = torch.empty(1 << 22, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 5)
y = torch.empty_like(x)
row = {}
for n in range(10, 22):
    N = 1 << n
    row["g1_2e%d" % n] = round(device_ms(lambda: sb.scan(x[:N], "add", out=y[:N])) * 1e3, 2)
for G, N in ((16, 4096), (64, 8192), (100, 8192), (8, 32768)):
    xv, yv = x[:G * N].view(G, N), y[:G * N].view(G, N)
    row["G%d_N%d" % (G, N)] = round(device_ms(lambda: sb.scan(xv, "add", out=yv)) * 1e3, 2)
print(json.dumps(row), flush=True)
