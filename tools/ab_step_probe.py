"""Short A/B probe of the shapes the bench reports: the configs[1] step (four back-to-back
scans of G = 4096 x N = 2^14: i32 / f32, inclusive / exclusive; events around 50 steps, best
of 5), configs[0] (CUDA graph of back-to-back calls), one problem of 2^24 / 2^25 / 2^26 and a
ragged batch.  One JSON line.  Use with tools/ab_libs.sh.

    python tools/ab_step_probe.py
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402
from tools.paper_sweep import device_ms, peak  # noqa: E402

G, N = 4096, 1 << 14
xi = torch.empty(G * N, dtype=torch.int32, device="cuda")
inputs.fill_device(xi, "i32", 2)
xf = torch.empty(G * N, dtype=torch.int32, device="cuda")
inputs.fill_device(xf, "f32u", 3)
xi, xf = xi.view(G, N), xf.view(torch.float32).view(G, N)
yi, yf = torch.empty_like(xi), torch.empty_like(xf)


def step():
    sb.scan(xi, "add", "inclusive", out=yi)
    sb.scan(xi, "add", "exclusive", out=yi)
    sb.scan(xf, "add", "inclusive", out=yf)
    sb.scan(xf, "add", "exclusive", out=yf)


best = None
for _ in range(5):
    for _ in range(3):
        step()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(50):
        step()
    e1.record()
    torch.cuda.synchronize()
    t = e0.elapsed_time(e1) / 50
    best = t if best is None else min(best, t)
row = {"c2_ms_per_step": round(best, 5), "c2_Gelem_s": round(4 * G * N / (best * 1e-3) / 1e9, 1),
       "c2_frac": round(4 * 8.0 * G * N / (best * 1e-3) / 1e9 / peak, 4)}
x = torch.empty(1 << 26, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 4)
y = torch.empty_like(x)
row["c1_us"] = round(device_ms(lambda: sb.scan(x[:1 << 20], "add", out=y[:1 << 20])) * 1e3, 2)
for n in (22, 24, 25, 26):
    ms = device_ms(lambda: sb.scan(x[:1 << n], "add", out=y[:1 << n]), reps=10)
    row["g1_2e%d_us" % n] = round(ms * 1e3, 2)
    row["g1_2e%d_frac" % n] = round(8.0 * (1 << n) / (ms * 1e-3) / 1e9 / peak, 4)
xv, yv = x[:2048 * 16384].view(2048, 16384), y[:2048 * 16384].view(2048, 16384)
row["G2048_N2e14_us"] = round(device_ms(lambda: sb.scan(xv, "add", out=yv), reps=10) * 1e3, 2)
print(json.dumps(row), flush=True)
