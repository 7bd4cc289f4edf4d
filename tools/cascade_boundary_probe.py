"""Where one CTA per problem (cascade) beats the flat look-back for a few thousand
long problems: G x N grid around G = 2048, int32 add, device time per call (CUDA graph of
back-to-back calls) and fraction of the measured copy for cascade_cta and lookback/3.

    python tools/cascade_boundary_probe.py [g2048 | small_g]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402
from tools.paper_sweep import device_ms, peak  # noqa: E402

GRIDS = {
    # round 2 session 3, first grid: G around 2048, tile-aligned and ragged N
    "g2048": [(G, N) for G in (1024, 1536, 2048, 2500, 3072, 4096)
              for N in (65536 + 4, 1 << 17, 196612, 1 << 18, 1 << 19)],
    # second grid: fewer problems (149 .. 1023) and ragged / unaligned-to-tile N
    "small_g": [(G, N) for G in (160, 300, 600, 1024)
                for N in (65540, 100000, 1 << 17, 150000, 196612, 1 << 18)]
    + [(2048, 196608), (2048, 200000), (2048, 300000), (1536, 300000), (2200, 262144), (2400, 262144)],
}
SHAPES = GRIDS[sys.argv[1] if len(sys.argv) > 1 else "g2048"]
x = torch.empty(max(G * N for G, N in SHAPES), dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 2018)
y = torch.empty_like(x)
for G, N in SHAPES:
    xv, yv = x[:G * N].view(G, N), y[:G * N].view(G, N)
    row = {"G": G, "N": N, "plan": "%s/%d" % sb.plan(xv, yv)}
    for algo, param in (("cascade_cta", -1), ("lookback", 3)):
        ms = device_ms(lambda: sb.scan(xv, "add", out=yv, algo=algo, param=param), reps=8)
        row["%s/%d" % (algo, param)] = [round(ms * 1e3, 1), round(8.0 * G * N / (ms * 1e-3) / 1e9 / peak, 4)]
    row["cascade_over_lookback"] = round(row["lookback/3"][0] / row["cascade_cta/-1"][0], 4)
    print(json.dumps(row), flush=True)
