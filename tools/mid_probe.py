"""Mid-size single problems (G = 1, N = 2^21..2^26: from L2-resident to HBM-bound): the
L2-staged look-back against the three-stage chain at several cascade depths K (chunk =
K x 4096 elements; <= 256 chunks run as two launches with Stage 2 folded into Stage 3).
Device time per call in us (CUDA graph of 20 calls)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402
from g1_probe import graph_ms  # noqa: E402

G = int(os.environ.get("G", "1"))
x = torch.empty(G << 26, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 2018)
y = torch.empty_like(x)
for n in range(21, 27):
    N = 1 << n
    xv, yv = x[:G * N].view(G, N), y[:G * N].view(G, N)
    row = {"G": G, "N": N, "auto": "%s/%d" % sb.plan(xv, yv)}
    for algo, param in [("auto", -1), ("lookback", 3), ("lookback", 1)] + [("three_stage", k) for k in (0, 2, 4, 8, 16, 32, 64)]:
        f = (lambda a=algo, p=param: sb.scan(xv, "add", out=yv, algo=a, param=p))
        row["%s/%d" % (algo, param)] = round(graph_ms(f, 10) * 1e3, 2)
    row["torch"] = round(graph_ms(lambda: torch.cumsum(xv, 1, dtype=xv.dtype, out=yv), 10) * 1e3, 2)
    print(json.dumps(row), flush=True)
