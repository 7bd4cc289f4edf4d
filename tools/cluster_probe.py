"""Few medium problems: the cluster-per-problem kernel (every variant x cluster size) against
the other families that take these shapes and torch.cumsum.  Device time per call in us
(20 calls in a CUDA graph, best of 5 replays).  One JSON line per (G, N).

    python tools/cluster_probe.py [G ...]       (default G = 1; N = 2^10 .. 2^20 + ragged)
"""
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

OTHERS = [("auto", -1), ("three_stage", 0), ("three_stage", 1), ("cascade_cta", -1), ("lookback", 10),
          ("lookback", 3)]
CLUSTER = [32 * v + c for v in range(3) for c in (1, 2, 4, 8, 16)]


def main():
    gs = [int(a) for a in sys.argv[1:]] or [1]
    ns = [1 << n for n in range(10, 21)] + [1000, 5000, 12345, 100003]
    x = torch.empty(max(gs) * max(ns), dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32", 2018)
    y = torch.empty_like(x)
    for G in gs:
        for N in ns:
            xv, yv = x[:G * N].view(G, N), y[:G * N].view(G, N)
            row = {"G": G, "N": N, "auto": "%s/%d" % sb.plan(xv, yv)}
            for algo, param in OTHERS + [("cluster", p) for p in CLUSTER]:
                try:
                    f = (lambda a=algo, p=param: sb.scan(xv, "add", out=yv, algo=a, param=p))
                    row["%s/%d" % (algo, param)] = round(graph_ms(f, 20) * 1e3, 2)
                except Exception as e:  # noqa: BLE001
                    row["%s/%d" % (algo, param)] = str(e)[:40]
            f = lambda: torch.cumsum(xv, 1, dtype=xv.dtype, out=yv)  # noqa: E731
            row["torch"] = round(graph_ms(f, 20) * 1e3, 2)
            cl = {k: v for k, v in row.items() if k.startswith("cluster/") and isinstance(v, float)}
            best = min(cl, key=cl.get)
            row["best_cluster"] = [best, cl[best]]
            print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
