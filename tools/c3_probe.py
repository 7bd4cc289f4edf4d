"""configs[2]-class single large problems: device time per call for look-back variants."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
vs = [int(v) for v in sys.argv[1].split(",")] if len(sys.argv) > 1 else [0]
for dt, N in (("i32", 1 << 28), ("f32", 1 << 30)):
    x = torch.empty(N, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32" if dt == "i32" else "f32u", 1)
    if dt == "f32":
        x = x.view(torch.float32)
    y = torch.empty_like(x)
    for v in vs:
        for _ in range(3):
            sb.scan(x, "add", out=y, algo="lookback", param=v)
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize(); s0.record()
        for _ in range(10):
            sb.scan(x, "add", out=y, algo="lookback", param=v)
        s1.record(); torch.cuda.synchronize()
        ms = s0.elapsed_time(s1) / 10
        print("%s N=2^%d v%d %.3f ms %.1f GB/s (%.1f%% of 6455.6)" % (dt, N.bit_length() - 1, v, ms, 8 * N / ms / 1e6,
                                                                  100 * 8 * N / ms / 1e6 / 6455.6), flush=True)
    del x, y
    torch.cuda.empty_cache()
