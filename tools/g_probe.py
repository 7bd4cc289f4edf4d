"""Single-problem vs few-problem look-back at 2^28 total: per-call device time by G."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
from bench import device_time
T = 1 << 28
x = torch.empty(T, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 3)
y = torch.empty_like(x)
s = torch.cuda.Stream()
for G in (1, 2, 4, 8, 1, 4):
    xv, yv = x.view(G, T // G), y.view(G, T // G)
    for param in (3, 0):
        with torch.cuda.stream(s):
            ms_graph = device_time(lambda: sb.scan(xv, "add", out=yv, algo="lookback", param=param, stream=s), s, 10)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ts = []
            for _ in range(5):
                a.record(s); sb.scan(xv, "add", out=yv, algo="lookback", param=param, stream=s); b.record(s)
                b.synchronize(); ts.append(a.elapsed_time(b))
        print("G=%d param %d graph %.1f us/call  single %s" % (G, param, ms_graph * 1e3, ["%.1f" % (t * 1e3) for t in ts]), flush=True)
