"""Large batches of long rows (configs[3]: G = 2^16 x N = 2^16 i32 = 16 GiB in, and its
per-rank shards G = 2^16/W): CTA-per-problem cascade against the L2-staged flat look-back
and the three-stage chain.  % of measured copy at 8 B/element, 3 timed calls each."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402

peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
TOT = 1 << 32
x = torch.empty(TOT, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 4)
y = torch.empty_like(x)
for G, N in [(1 << 16, 1 << 16), (1 << 15, 1 << 16), (1 << 14, 1 << 16), (1 << 13, 1 << 16),
             (1 << 17, 1 << 15), (1 << 15, 1 << 17), (1 << 14, 1 << 18), (1 << 18, 1 << 14)]:
    xv, yv = x[:G * N].view(G, N), y[:G * N].view(G, N)
    row = {"G": G, "N": N, "auto": "%s/%d" % sb.plan(xv, yv)}
    for algo, param in [("cascade_cta", -1), ("lookback", 3), ("three_stage", 0)]:
        for _ in range(2):
            sb.scan(xv, "add", out=yv, algo=algo, param=param)
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        s0.record()
        for _ in range(3):
            sb.scan(xv, "add", out=yv, algo=algo, param=param)
        s1.record()
        torch.cuda.synchronize()
        ms = s0.elapsed_time(s1) / 3
        row["%s/%d" % (algo, param)] = round(8.0 * G * N / (ms * 1e-3) / 1e9 / peak, 4)
    print(json.dumps(row), flush=True)
