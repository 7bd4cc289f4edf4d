"""Small single problems (G = 1, PAPER.md:255, 259 [Fig. 11]): device time per call of every
kernel family that can take them, with torch.cumsum beside it.  Two timings per point:
`ms` = 20 calls in one CUDA graph replayed between two events (per-call throughput of
back-to-back calls); `lat_ms` = a one-call graph replayed between two events (one call's
latency, graph launch included).  One JSON line per (N, candidate)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402


def graph_ms(fn, reps):
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(reps):
            fn()
    g.replay()
    torch.cuda.synchronize()
    best = None
    for _ in range(5):
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s0.record(s)
        with torch.cuda.stream(s):
            g.replay()
        s1.record(s)
        torch.cuda.synchronize()
        t = s0.elapsed_time(s1) / reps
        best = t if best is None else min(best, t)
    return best


CANDS = [("auto", -1), ("lookback", 1), ("lookback", 2), ("lookback", 3), ("lookback", 10), ("cluster", -1), ("three_stage", 0), ("three_stage", 1), ("three_stage", 2), ("cascade_cta", -1)]


def main():
    ns = [int(a) for a in sys.argv[1:]] or [1 << n for n in range(10, 23)] + [1000, 5000, 100003]
    dt = os.environ.get("DT", "i32")
    x = torch.empty(max(ns), dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32" if dt == "i32" else "f32u", 2018)
    if dt == "f32":
        x = x.view(torch.float32)
    y = torch.empty_like(x)
    for N in ns:
        xv, yv = x[:N], y[:N]
        row = {"N": N, "dtype": dt, "auto": "%s/%d" % sb.plan(xv, yv)}
        for algo, param in CANDS:
            try:
                f = (lambda a=algo, p=param: sb.scan(xv, "add", out=yv, algo=a, param=p))
                row["%s/%d" % (algo, param)] = (round(graph_ms(f, 20) * 1e3, 2), round(graph_ms(f, 1) * 1e3, 2))
            except Exception as e:  # noqa: BLE001
                row["%s/%d" % (algo, param)] = str(e)[:40]
        f = lambda: torch.cumsum(xv, 0, dtype=xv.dtype, out=yv)  # noqa: E731
        row["torch"] = (round(graph_ms(f, 20) * 1e3, 2), round(graph_ms(f, 1) * 1e3, 2))
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
