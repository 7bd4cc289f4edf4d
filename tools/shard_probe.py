"""Sharded path at configs[4]'s per-rank size: public Stage 1+2 / Stage 3 entry points timed
one by one, against the fused (peer) single call; outputs compared on the device."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
from paper_conf_ipps_dieguezadnm18_b200 import multi

n = int(sys.argv[1]) if len(sys.argv) > 1 else 33
N = 1 << n
x = torch.empty(N, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 5)
y1 = torch.empty_like(x)
y2 = torch.empty_like(x)
comm = multi.PeerComm.loopback(1, 1)[0]


def timeit(fn, reps=5):
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


t_fused = timeit(lambda: multi.scan_multi(x, out=y1, backend="peer", comm=comm))
tot = sb.shard_totals(x, "add")
t_tot = timeit(lambda: sb.shard_totals(x, "add", totals=tot))
t_scan = timeit(lambda: sb.shard_scan(x, tot.view(1, -1), 0, 1, "add", "inclusive", out=y2))
torch.cuda.synchronize()
same = torch.equal(y1, y2)
print("N=2^%d fused %.3f ms | stage1+2 %.3f ms (%.0f GB/s read) | stage3 %.3f ms (%.0f GB/s) | equal %s"
      % (n, t_fused, t_tot, 4 * N / t_tot / 1e6, t_scan, 8 * N / t_scan / 1e6, same))
print("plan", sb._lib.lib.scan_shard_workspace_bytes(N, 1))
comm.close()
