"""Does the input distribution change kernel time? (same dtype/size/kernel, different values)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
vs = [int(v) for v in sys.argv[1].split(",")]
N = 1 << 30
for dist, tdt in (("i32", torch.int32), ("small", torch.int32), ("iota", torch.int32), ("f32u", torch.float32),
                  ("f32s", torch.float32)):
    x = torch.empty(N, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, dist, 1, row_len=N)
    x = x.view(tdt)
    y = torch.empty_like(x)
    line = "%-6s" % dist
    for v in vs:
        for _ in range(2):
            sb.scan(x, "add", out=y, algo="lookback", param=v)
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize(); s0.record()
        for _ in range(5):
            sb.scan(x, "add", out=y, algo="lookback", param=v)
        s1.record(); torch.cuda.synchronize()
        ms = s0.elapsed_time(s1) / 5
        line += "  v%d %.1f%%" % (v, 100 * 8 * N / ms / 1e6 / 6455.6)
    c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    c0.record(); y.copy_(x); c1.record(); torch.cuda.synchronize()
    line += "  copy %.1f%%" % (100 * 8 * N / c0.elapsed_time(c1) / 1e6 / 6455.6)
    print(line, flush=True)
    del x, y
    torch.cuda.empty_cache()
