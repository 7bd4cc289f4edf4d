"""The fused cooperative three-stage kernel (SCAN_ALGO_FUSED) against
the AUTO choice and the other families near its region: device time per call (CUDA graph of
20 calls).  One JSON line per (dtype, G, N).   python tools/fused_probe.py [parity]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402
from g1_probe import graph_ms  # noqa: E402

if len(sys.argv) > 1 and sys.argv[1] == "parity":
    from gpu_util import assert_parity, to_device, to_host
    for dist, op, kind, G, N, prm in [("i32", "add", "inclusive", 1, 4000001, -1), ("f32s", "add", "exclusive", 1, 3000001, -1),
                                      ("u32", "max", "inclusive", 3, 8192 * 5, -1), ("i32", "add", "exclusive", 1, 8193, -1)]:
        x = inputs.generate(dist, G * N, 5).reshape(G, N)
        out = sb.scan(to_device(x), op, kind, algo="fused", param=prm)
        torch.cuda.synchronize()
        assert_parity(to_host(out, x.dtype).reshape(G, N), x, op, kind, label="fused %s %d %d" % (dist, G, N))
    print("parity ok", flush=True)
    sys.exit(0)

SHAPES = [(1, n) for n in (1 << 21, 3 << 20, 1 << 22, 4849664, 5 << 20, 6 << 20, 7 << 20, 1 << 23, 9 << 20, 9699328)]
x = torch.empty(1 << 24, dtype=torch.int32, device="cuda")
y = torch.empty_like(x)
for dt, dist in (("i32", "i32"), ("f32", "f32u")):
    inputs.fill_device(x, dist, 1)
    xx = x.view(torch.float32) if dt == "f32" else x
    yy = y.view(torch.float32) if dt == "f32" else y
    for G, N in SHAPES:
        xv, yv = xx[:G * N].view(G, N), yy[:G * N].view(G, N)
        row = {"dtype": dt, "G": G, "N": N, "auto": "%s/%d" % sb.plan(xv, yv)}
        for algo, param in [("auto", -1), ("fused", -1), ("three_stage", 0), ("lookback", 3)]:
            key = "%s/%d" % (algo, param)
            try:
                row[key] = round(graph_ms(lambda: sb.scan(xv, "add", out=yv, algo=algo, param=param), 20) * 1e3, 2)
            except Exception as e:  # noqa: BLE001
                row[key] = str(e)[-12:]
        print(json.dumps(row), flush=True)
