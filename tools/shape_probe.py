"""Every kernel family / parameter on given G x N shapes (int32 add inclusive): device time
per call (CUDA graph of back-to-back calls) and fraction of the measured copy.

    python tools/shape_probe.py 2048x65540 160x65540 ...
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

CANDS = [("auto", -1), ("lookback", 3), ("lookback", 0), ("lookback", 1), ("lookback", 2),
         ("cascade_cta", -1), ("three_stage", -1), ("three_stage", 1), ("three_stage", 4), ("fused", -1)]
if os.environ.get("SHAPE_PROBE_MID"):          # the mid-batch dispatch boundary
    CANDS = [("auto", -1), ("lookback", 3), ("lookback", 1), ("cascade_cta", -1), ("three_stage", -1)]
if os.environ.get("SHAPE_PROBE_CLUSTER"):      # the cluster family: param = 32 * variant + csize
    CANDS = [("auto", -1), ("three_stage", -1), ("lookback", 3)] + [
        ("cluster", 32 * v + c) for v in (0, 1, 2) for c in (4, 8, 16)]
shapes = [tuple(int(v) for v in a.split("x")) for a in sys.argv[1:]]
x = torch.empty(max(G * N for G, N in shapes), dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 2018)
y = torch.empty_like(x)
for G, N in shapes:
    xv, yv = x[:G * N].view(G, N), y[:G * N].view(G, N)
    row = {"G": G, "N": N, "plan": "%s/%d" % sb.plan(xv, yv)}
    for algo, param in CANDS:
        try:
            ms = device_ms(lambda: sb.scan(xv, "add", out=yv, algo=algo, param=param), reps=8)
        except Exception as e:  # noqa: BLE001
            row["%s/%d" % (algo, param)] = "n/a: %s" % str(e)[:30]
            continue
        row["%s/%d" % (algo, param)] = [round(ms * 1e3, 1), round(8.0 * G * N / (ms * 1e-3) / 1e9 / peak, 3)]
    print(json.dumps(row), flush=True)
