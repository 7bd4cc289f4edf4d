"""The paper's workload shapes, through the default dispatch, with torch.cumsum beside it
as on-box library context (torch's CUDA cumsum; a 1-D int32 cumsum goes through CUB's
DeviceScan).  One JSON line per point: chosen kernel, device time, Gelem/s, % of measured
copy, and the same for torch.cumsum.

    python tools/paper_sweep.py batch [n0]   # 2^28 int32 as G = 2^28/N problems of N = 2^n,
                                             # n = n0..28 (PAPER.md:241, 249, 261 [Figs. 9-12])
    python tools/paper_sweep.py g1 [n0 [n1]] # G = 1, N = 2^n, n = n0..n1 (default 30; up to 33 on one B200)
                                             # (PAPER.md:255, 259 [Fig. 11])

Device time per call: 20 calls captured in a CUDA graph and replayed between two events
(so the small, latency-bound points are not host-launch bound)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402

_pk = os.path.join(ROOT, "MEASURED_PEAKS.json")
peak = json.load(open(_pk))["hbm_gbs"] if os.path.exists(_pk) else 6650.0


def device_ms(fn, reps=20):
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
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s0.record(s)
    with torch.cuda.stream(s):
        g.replay()
    s1.record(s)
    torch.cuda.synchronize()
    return s0.elapsed_time(s1) / reps


def main():
    mode = sys.argv[1] if len(sys.argv) > 1 else "batch"
    n0 = int(sys.argv[2]) if len(sys.argv) > 2 else 10
    n1 = 28 if mode == "batch" else (int(sys.argv[3]) if len(sys.argv) > 3 else 30)
    total_max = 1 << n1
    x = torch.empty(total_max, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32", 2018)
    y = torch.empty_like(x)
    for n in range(n0, n1 + 1):
        N = 1 << n
        G = (1 << 28) // N if mode == "batch" else 1
        total = G * N
        xv, yv = x[:total].view(G, N), y[:total].view(G, N)
        ms = device_ms(lambda: sb.scan(xv, "add", out=yv))
        # torch.cumsum into a preallocated int32 output (dtype given so it does not promote)
        tms = device_ms(lambda: torch.cumsum(xv, dim=1, dtype=torch.int32, out=yv))
        algo, param = sb.plan(xv, yv)
        r = {"mode": mode, "n": n, "N": N, "G": G, "kernel": "%s/%d" % (algo, param), "ms": round(ms, 5),
             "Gelem/s": round(total / ms / 1e6, 1), "frac_measured_copy": round(8 * total / ms / 1e6 / peak, 3),
             "torch_cumsum_ms": round(tms, 5), "torch_cumsum_Gelem/s": round(total / tms / 1e6, 1),
             "speedup_vs_torch": round(tms / ms, 2)}
        print(json.dumps(r), flush=True)


if __name__ == "__main__":
    main()
