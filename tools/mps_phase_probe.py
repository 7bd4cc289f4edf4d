"""Scan-MPS at W = 1: 2^28 int32 as G = 2^28/N problems, the sharded
two-pass pipeline's phases timed separately (Stage 1+2 = scan_shard_totals, Stage 3 =
scan_shard_scan) next to the single-pass AUTO scan of the same batch; us per call from
CUDA-graph replays, frac of the measured copy at 4 B/elem (Stage 1+2), 8 B/elem (Stage 3).

    python tools/mps_phase_probe.py [n ...]      # default 13 16 20 28
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

T = 1 << 28
x = torch.empty(T, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 11)
y = torch.empty_like(x)
for n in [int(a) for a in sys.argv[1:]] or [13, 16, 20, 28]:
    N = 1 << n
    G = T // N
    xv, yv = x.view(G, N), y.view(G, N)
    tot = sb.shard_totals(xv, "add")
    allt = tot.view(1, G).clone()
    ms1 = device_ms(lambda: sb.shard_totals(xv, "add", totals=tot), reps=10)
    ms3 = device_ms(lambda: sb.shard_scan(xv, allt, 0, 1, "add", "inclusive", out=yv), reps=10)
    msa = device_ms(lambda: sb.scan(xv, "add", out=yv), reps=10)
    print(json.dumps({"n": n, "G": G, "stage12_us": round(ms1 * 1e3, 1),
                      "stage12_frac_4B": round(4.0 * T / (ms1 * 1e-3) / 1e9 / peak, 3),
                      "stage3_us": round(ms3 * 1e3, 1), "stage3_frac_8B": round(8.0 * T / (ms3 * 1e-3) / 1e9 / peak, 3),
                      "auto_us": round(msa * 1e3, 1), "auto_plan": "%s/%d" % sb.plan(xv, yv)}), flush=True)
