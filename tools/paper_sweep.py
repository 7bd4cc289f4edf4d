"""The paper's workload shape (PAPER.md:241, 249, 261 [Figs. 9-12]): 2^28 int32 elements as
G = 2^28/N problems of N = 2^n, n = 10..28, inclusive add, through the default dispatch.
Prints one JSON line per n: chosen kernel, device time, Gelem/s, % of measured copy."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402

peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                   "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6455.6
TOTAL = 1 << 28
x = torch.empty(TOTAL, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 2018)
y = torch.empty_like(x)
rows = []
for n in range(int(sys.argv[1]) if len(sys.argv) > 1 else 10, 29):
    N = 1 << n
    G = TOTAL // N
    xv, yv = x.view(G, N), y.view(G, N)
    for _ in range(3):
        sb.scan(xv, "add", out=yv)
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    s0.record()
    for _ in range(10):
        sb.scan(xv, "add", out=yv)
    s1.record()
    torch.cuda.synchronize()
    ms = s0.elapsed_time(s1) / 10
    algo, param = sb.plan(xv, yv)
    r = {"n": n, "N": N, "G": G, "kernel": "%s/%d" % (algo, param), "ms": round(ms, 4),
         "Gelem/s": round(TOTAL / ms / 1e6, 1), "frac_measured_copy": round(8 * TOTAL / ms / 1e6 / peak, 3)}
    rows.append(r)
    print(json.dumps(r), flush=True)
