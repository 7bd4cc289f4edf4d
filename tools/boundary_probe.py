"""cascade_cta vs look-back (variant 3) near the dispatch boundary."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
x = torch.empty(1 << 28, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 3)
y = torch.empty_like(x)
def t(xv, yv, algo, param):
    for _ in range(2):
        sb.scan(xv, "add", out=yv, algo=algo, param=param)
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); s0.record()
    for _ in range(8):
        sb.scan(xv, "add", out=yv, algo=algo, param=param)
    s1.record(); torch.cuda.synchronize()
    return s0.elapsed_time(s1) / 8
import json
PEAK = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6455.6
for G, N in [(4096, 1 << 14), (4096, 1 << 16), (2048, 1 << 17), (1024, 1 << 18), (768, 1 << 18), (592, 1 << 18),
             (512, 1 << 19), (256, 1 << 20), (128, 1 << 21), (64, 1 << 22), (16, 1 << 24), (4, 1 << 26),
             (16384, 1 << 12), (65536, 1 << 10), (1 << 18, 1 << 8), (1 << 20, 1 << 6)]:
    xv, yv = x[:G * N].view(G, N), y[:G * N].view(G, N)
    res = []
    for algo, param in [("cascade_cta", -1), ("cascade_warp", -1), ("lookback", 3), ("lookback", 2)]:
        if algo == "cascade_warp" and N > (1 << 16):
            continue
        if algo == "cascade_cta" and G < 128:
            continue
        ms = t(xv, yv, algo, param)
        res.append("%s/%d %.1f%%" % (algo, param, 100 * 8 * G * N / ms / 1e6 / PEAK))
    print("G=%d N=%d  " % (G, N) + "  ".join(res), flush=True)
