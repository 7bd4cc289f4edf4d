"""One problem (G = 1) of N = 2^n int32 through a look-back variant, n = n0..n1: device
time per call (events around back-to-back calls; CUDA graph for the short ones), Gelem/s and
fraction of the measured copy bandwidth at 8 B/elem.  One JSON line per point.

    python tools/lb_size_probe.py [n0 n1 [param ...]]      # default 22 33, params 3
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402

_pk = os.path.join(ROOT, "MEASURED_PEAKS.json")
peak = __import__("json").load(open(_pk))["hbm_gbs"] if os.path.exists(_pk) else 6650.0


def timed(fn, reps, graph):
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
    torch.cuda.synchronize()
    if graph:
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(reps):
                fn()
        run = g.replay
    else:
        def run():
            for _ in range(reps):
                fn()
    best = None
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record(s)
            run()
            e1.record(s)
        torch.cuda.synchronize()
        t = e0.elapsed_time(e1) / reps
        best = t if best is None else min(best, t)
    return best


def main():
    n0, n1 = (int(sys.argv[1]), int(sys.argv[2])) if len(sys.argv) > 2 else (22, 33)
    params = [int(p) for p in sys.argv[3:]] or [3]
    dist = os.environ.get("DIST", "i32")
    x = torch.empty(1 << n1, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, dist, 2018)
    if dist.startswith("f32"):
        x = x.view(torch.float32)
    y = torch.empty_like(x)
    for n in range(n0, n1 + 1):
        N = 1 << n
        xv, yv = x[:N], y[:N]
        row = {"n": n, "dist": dist, "auto": "%s/%d" % sb.plan(xv, yv)}
        for p in params:
            reps = max(3, min(50, (1 << 30) // N * 5))
            ms = timed(lambda: sb.scan(xv, "add", out=yv, algo="lookback", param=p), reps, graph=n <= 27)
            row["lb%d_us" % p] = round(ms * 1e3, 2)
            row["lb%d_frac" % p] = round(8.0 * N / (ms * 1e-3) / 1e9 / peak, 4)
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
