"""scan_autotune (the automated form of the paper's K search) on the paper's
workload shapes: for each (G, N) the static AUTO choice and its device time next to the
tuned choice and its time.  One JSON line per shape."""
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

SHAPES = [(G, 1 << n) for G in (1, 4, 16, 64, 256, 1024) for n in (8, 10, 12, 14, 16, 18, 20, 22, 24)
          if G << n <= 1 << 26] + [(4096, 1 << 14), (1 << 16, 1 << 10), (1 << 18, 1 << 8), (3, 100003),
                                   (1000, 1000), (5000, 3000)]


def main():
    total = max(g * n for g, n in SHAPES)
    x = torch.empty(total, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32", 2018)
    y = torch.empty_like(x)
    for G, N in SHAPES:
        xv, yv = x[:G * N].view(G, N), y[:G * N].view(G, N)
        sb.autotune_clear()
        static = sb.plan(xv, yv)
        t_static = graph_ms(lambda: sb.scan(xv, "add", out=yv), 20) * 1e3
        algo, param, us = sb.autotune(xv, "add", "inclusive", out=yv)
        t_tuned = graph_ms(lambda: sb.scan(xv, "add", out=yv), 20) * 1e3
        print(json.dumps({"G": G, "N": N, "static": "%s/%d" % static, "static_us": round(t_static, 2),
                          "tuned": "%s/%d" % (algo, param), "tuned_us": round(t_tuned, 2),
                          "tuner_us": round(us, 2), "gain": round(t_static / t_tuned, 3)}), flush=True)
    sb.autotune_clear()


if __name__ == "__main__":
    main()
