"""Read-only pass ceiling: Stage 1+2 of the sharded path (shard_totals) against torch's
own reductions over the same int32 array (read-only HBM bandwidth context)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
from bench import device_time
s = torch.cuda.Stream()
for n in (28, 30):
    N = 1 << n
    x = torch.empty(N, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32", 1)
    for name, fn in [("shard_totals", lambda: sb.shard_totals(x, "add", stream=s)),
                     ("torch.sum", lambda: torch.sum(x)),
                     ("torch.amax", lambda: torch.amax(x))]:
        with torch.cuda.stream(s):
            ms = device_time(fn, s, 20)
        print("N=2^%d %-14s %8.3f ms  %7.1f GB/s read" % (n, name, ms, 4 * N / ms / 1e6), flush=True)
