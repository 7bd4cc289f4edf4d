"""Scan-MPS at W = 1, n given: the bench leg's call (multi.scan_multi, peer exchange at W = 1)
timed eagerly (as bench.py scan_mps does) and as a CUDA graph, beside the public two-step
API (shard_totals + shard_scan) -- separates host overhead from device time.

    python tools/mps_w1_probe.py 13 20
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402
from paper_conf_ipps_dieguezadnm18_b200 import multi  # noqa: E402
from tools.paper_sweep import device_ms  # noqa: E402


def eager_ms(fn, reps=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


T = 1 << 28
for n in [int(v) for v in sys.argv[1:]] or [13, 20]:
    N = 1 << n
    G = T // N
    x = torch.empty(G, N, dtype=torch.int32, device="cuda")
    inputs.fill_device(x.view(-1), "i32", 7)
    y = torch.empty_like(x)
    c = multi.PeerComm.loopback(1, G)[0]
    call = lambda: multi.scan_multi(x, "add", "inclusive", mode="elements", out=y, backend="peer", comm=c)  # noqa: E731
    tot = sb.shard_totals(x, "add")
    allt = tot.view(1, G).clone()

    def steps():
        sb.shard_totals(x, "add", totals=tot)
        sb.shard_scan(x, allt, 0, 1, "add", "inclusive", out=y)
    row = {"n": n, "G": G, "peer_eager_ms": eager_ms(call), "steps_eager_ms": eager_ms(steps),
           "steps_graph_ms": device_ms(steps, reps=10)}
    try:
        row["peer_graph_ms"] = device_ms(call, reps=10)
    except Exception as e:  # noqa: BLE001
        row["peer_graph_ms"] = "n/a: %s" % str(e)[:60]
    torch.cuda.synchronize()
    c.close()
    print(json.dumps({k: (round(v, 4) if isinstance(v, float) else v) for k, v in row.items()}), flush=True)
