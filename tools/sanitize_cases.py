"""Small cases of every kernel family / variant for compute-sanitizer runs (T7).

    compute-sanitizer --tool racecheck python tools/sanitize_cases.py [--quick]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402
from paper_conf_ipps_dieguezadnm18_b200 import _lib  # noqa: E402

quick = "--quick" in sys.argv
shapes = [(20000, 3), (70001, 1), (1000, 40)] if not quick else [(70001, 1), (1000, 5)]
cases = [("cascade_cta", -1), ("cascade_warp", -1), ("three_stage", 0), ("packed_warp", -1),
         ("cluster", -1), ("cluster", 32 + 4), ("cluster", 2), ("fused", -1)] + \
        [("lookback", v) for v in _lib.LOOKBACK_VARIANTS]
for dt, dist in (("i32", "i32"), ("f32", "f32s")):
    for N, G in shapes:
        x = torch.empty(N * G, dtype=torch.int32, device="cuda")
        inputs.fill_device(x, dist, 1)
        if dt == "f32":
            x = x.view(torch.float32)
        x = x.view(G, N)
        for algo, param in cases:
            if algo == "fused" and G > 1 and N % 8192:
                continue                                  # not eligible (rejected, tested elsewhere)
            for kind in ("inclusive", "exclusive"):
                sb.scan(x, "add", kind, algo=algo, param=param)
                torch.cuda.synchronize()
        t = sb.shard_totals(x, "add")
        sb.shard_scan(x, torch.stack([t, t]), 1, 2, "add", "inclusive")
        torch.cuda.synchronize()
        print("ok", dt, N, G, flush=True)
# the persistent L2-staged look-back over several rounds (lazy round-robin look-back with the
# CTA-local previous prefix, kept tail tiles): more tiles than SMs, ragged last tile
for dt, dist in (("i32", "i32"), ("f32", "f32s")):
    N = 3 * 148 * 8192 + 1234
    x = torch.empty(N, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, dist, 2)
    if dt == "f32":
        x = x.view(torch.float32)
    for kind in ("inclusive", "exclusive"):
        sb.scan(x, "add", kind, algo="lookback", param=3)
        torch.cuda.synchronize()
    print("ok multi-round", dt, N, flush=True)
# problem starts inside the L2-staged look-back's tiles (masked reduction, literal-`small`
# head tests) and a three-stage mid batch -- the round-2 session-3 paths
for dt, dist in (("i32", "i32"), ("f32", "f32s")):
    for (G, N, algo, param) in ((60, 65540, "lookback", 3), (7, 3001, "lookback", 3), (70, 65536, "auto", -1)):
        x = torch.empty(G * N, dtype=torch.int32, device="cuda")
        inputs.fill_device(x, dist, 3)
        if dt == "f32":
            x = x.view(torch.float32)
        x = x.view(G, N)
        for kind in ("inclusive", "exclusive"):
            sb.scan(x, "add", kind, algo=algo, param=param)
            sb.scan(x, "max", kind, algo=algo, param=param)
        torch.cuda.synchronize()
        print("ok segmented", dt, G, N, algo, param, flush=True)
print("sanitize cases done")
