"""configs[0] and its neighbours (G = 1, N = 2^19 .. 2^21, int32 add): the two-launch
three-stage chain with K = 1 / 2 / 4 tiles per chunk and AUTO, us per call from CUDA-graph
replays of 50 back-to-back calls (bench.py's configs[0] method), best of 3.

    python tools/c1_k_probe.py
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402
from bench import device_time  # noqa: E402

x = torch.empty(1 << 21, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 1)
y = torch.empty_like(x)
s = torch.cuda.Stream()
for N in ((1 << 19), 3 << 18, (1 << 20), 3 << 19, (1 << 21)):
    row = {"N": N, "auto": "%s/%d" % sb.plan(x[:N], y[:N])}
    for algo, param in (("auto", -1), ("three_stage", 1), ("three_stage", 2), ("three_stage", 4)):
        row["%s/%d" % (algo, param)] = round(min(device_time(
            lambda: sb.scan(x[:N], "add", out=y[:N], algo=algo, param=param, stream=s), s, 50) for _ in range(3)) * 1e3, 3)
    print(json.dumps(row), flush=True)
