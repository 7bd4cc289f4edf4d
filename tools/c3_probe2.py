"""Single large problems: device time for look-back variants over (dtype, N)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
vs = [int(v) for v in sys.argv[1].split(",")]
for dt in ("i32", "f32"):
    for n in (28, 29, 30):
        N = 1 << n
        x = torch.empty(N, dtype=torch.int32, device="cuda")
        inputs.fill_device(x, "i32" if dt == "i32" else "f32u", 1)
        if dt == "f32":
            x = x.view(torch.float32)
        y = torch.empty_like(x)
        line = "%s 2^%d" % (dt, n)
        for v in vs:
            for _ in range(3):
                sb.scan(x, "add", out=y, algo="lookback", param=v)
            s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize(); s0.record()
            for _ in range(8):
                sb.scan(x, "add", out=y, algo="lookback", param=v)
            s1.record(); torch.cuda.synchronize()
            ms = s0.elapsed_time(s1) / 8
            line += "  v%d %.1f%%" % (v, 100 * 8 * N / ms / 1e6 / 6455.6)
        print(line, flush=True)
        del x, y
        torch.cuda.empty_cache()
