"""The fused cooperative three-stage kernel (SCAN_ALGO_FUSED) against the AUTO choice and the
other latency-bound families near its region: device time per call (CUDA graph of 20 calls).
One JSON line per (dtype, G, N)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402
from g1_probe import graph_ms  # noqa: E402

SHAPES = [(1, n) for n in (1 << 20, 3 << 19, 1 << 21, 5 << 19, 3 << 20, 7 << 19, 1 << 22, 9 << 19, 4849664)] + \
         [(2, 1 << 21), (4, 1 << 20), (8, 1 << 19), (16, 1 << 18), (64, 1 << 16)]
x = torch.empty(1 << 23, dtype=torch.int32, device="cuda")
y = torch.empty_like(x)
for dt, dist in (("i32", "i32"), ("f32", "f32u")):
    inputs.fill_device(x, dist, 1)
    xx = x.view(torch.float32) if dt == "f32" else x
    yy = y.view(torch.float32) if dt == "f32" else y
    for G, N in SHAPES:
        xv, yv = xx[:G * N].view(G, N), yy[:G * N].view(G, N)
        row = {"dtype": dt, "G": G, "N": N, "auto": "%s/%d" % sb.plan(xv, yv)}
        for algo, param in [("auto", -1), ("fused", -1), ("three_stage", 0), ("lookback", 3)]:
            try:
                row["%s" % algo] = round(graph_ms(lambda: sb.scan(xv, "add", out=yv, algo=algo, param=param), 20) * 1e3, 2)
            except Exception as e:  # noqa: BLE001
                row[algo] = str(e)[-24:]
        print(json.dumps(row), flush=True)
