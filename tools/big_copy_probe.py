"""One G = 1 int32 problem of 2^n elements, n = n0..n1, next to a torch copy_ of the same
bytes (the MEASURED_PEAKS kernel) on the same buffers: does the copy itself slow down at
the sizes where the scan does (2^32-2^33: 16-32 GiB per buffer)?  Events around single
calls, best of 3 after a warm-up.  One JSON line per n.

    python tools/big_copy_probe.py [n0 n1]       # default 28 33
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


def best(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    b = None
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        t = e0.elapsed_time(e1)
        b = t if b is None else min(b, t)
    return b


n0, n1 = (int(sys.argv[1]), int(sys.argv[2])) if len(sys.argv) > 2 else (28, 33)
x = torch.empty(1 << n1, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 2018)
y = torch.empty_like(x)
for n in range(n0, n1 + 1):
    N = 1 << n
    xv, yv = x[:N], y[:N]
    ms_scan = best(lambda: sb.scan(xv, "add", out=yv))
    ms_copy = best(lambda: yv.copy_(xv))
    gb = 8.0 * N / 1e9
    print(json.dumps({"n": n, "GiB_per_buffer": N * 4 / 2 ** 30, "plan": "%s/%d" % sb.plan(xv, yv),
                      "scan_ms": round(ms_scan, 4), "scan_frac": round(gb / (ms_scan * 1e-3) / peak, 4),
                      "copy_ms": round(ms_copy, 4), "copy_frac": round(gb / (ms_copy * 1e-3) / peak, 4),
                      "scan_over_copy": round(ms_copy / ms_scan, 4)}), flush=True)
