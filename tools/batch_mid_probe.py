"""2^28 int32 as G = 2^28/N problems of N = 2^n (the paper's batch sweep), for
the n where the dispatch changes family (16-20): every candidate family / parameter, device
time per call (CUDA graph of back-to-back calls), fraction of the measured copy.  Env
switches of the library (SCANB200_LB_MODE, ...) apply.

    python tools/batch_mid_probe.py [n0 n1]      # default 15 20
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

n0, n1 = (int(sys.argv[1]), int(sys.argv[2])) if len(sys.argv) > 2 else (15, 20)
T = 1 << 28
x = torch.empty(T, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 2018)
y = torch.empty_like(x)
CANDS = [("auto", -1), ("lookback", 3), ("lookback", 0), ("cascade_cta", -1), ("three_stage", -1),
         ("three_stage", 2), ("cluster", -1)]
for n in range(n0, n1 + 1):
    N = 1 << n
    G = T // N
    xv, yv = x.view(G, N), y.view(G, N)
    row = {"n": n, "G": G, "plan": "%s/%d" % sb.plan(xv, yv)}
    for algo, param in CANDS:
        try:
            ms = device_ms(lambda: sb.scan(xv, "add", out=yv, algo=algo, param=param))
        except Exception as e:  # noqa: BLE001  (a family that rejects the shape)
            row["%s/%d" % (algo, param)] = "n/a: %s" % str(e)[:40]
            continue
        row["%s/%d" % (algo, param)] = [round(ms * 1e3, 1), round(8.0 * T / (ms * 1e-3) / 1e9 / peak, 4)]
    print(json.dumps(row), flush=True)
