"""Mid-size G = 1 scans (2^n int32) in two timing modes, with a size-matched copy beside them.

  warm     back-to-back calls on the SAME input / output (CUDA graph): the footprint
           (2 x 4 B x N) is near the 126 MB L2 at 2^23-2^24, so what the previous call left
           in L2 counts -- the situation of a scan whose input a producer kernel just wrote;
  rotate   the calls cycle over K distinct input / output pairs whose total footprint is
           >= 512 MiB, so every call reads its input from HBM (the cold, HBM-bound case).

The copy (torch copy_, the MEASURED_PEAKS kernel) runs in the same two modes.  frac = 8 B
per element / time / MEASURED_PEAKS hbm_gbs.  One JSON line per (n, mode).

    python tools/mid_l2_probe.py [n0 n1]        # default 22 27; env SCANB200_L2_POL etc. apply
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
peak = json.load(open(_pk))["hbm_gbs"] if os.path.exists(_pk) else 6450.0


def graph_time(fns, reps):
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for f in fns:
            f()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for r in range(reps):
            fns[r % len(fns)]()
    best = None
    for _ in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record(s)
            g.replay()
            e1.record(s)
        torch.cuda.synchronize()
        t = e0.elapsed_time(e1) / reps
        best = t if best is None else min(best, t)
    return best


def main():
    n0, n1 = (int(sys.argv[1]), int(sys.argv[2])) if len(sys.argv) > 2 else (22, 27)
    algo = os.environ.get("ALGO", "auto")
    param = int(os.environ.get("PARAM", "-1"))
    for n in range(n0, n1 + 1):
        N = 1 << n
        K = max(1, (512 << 20) // (8 * N))
        xs = []
        for k in range(K):
            x = torch.empty(N, dtype=torch.int32, device="cuda")
            inputs.fill_device(x, "i32", 2018 + k)
            xs.append(x)
        ys = [torch.empty_like(x) for x in xs]
        reps = max(8, min(64, (1 << 30) // N * 4))
        reps = max(reps, K) // K * K
        for mode in ("warm", "rotate"):
            idx = [0] if mode == "warm" else list(range(K))
            scans = [(lambda i=i: sb.scan(xs[i], "add", out=ys[i], algo=algo, param=param)) for i in idx]
            copies = [(lambda i=i: ys[i].copy_(xs[i])) for i in idx]
            ms = graph_time(scans, reps)
            cms = graph_time(copies, reps)
            row = {"n": n, "mode": mode, "K": len(idx), "plan": "%s/%d" % sb.plan(xs[0], ys[0]),
                   "l2_pol": int(os.environ.get("SCANB200_L2_POL", "0")),
                   "scan_us": round(ms * 1e3, 2), "scan_frac": round(8.0 * N / (ms * 1e-3) / 1e9 / peak, 4),
                   "copy_us": round(cms * 1e3, 2), "copy_frac": round(8.0 * N / (cms * 1e-3) / 1e9 / peak, 4),
                   "scan_over_copy": round(cms / ms, 4)}
            print(json.dumps(row), flush=True)
        del xs, ys
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
