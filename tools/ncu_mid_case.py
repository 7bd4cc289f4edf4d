"""One G = 1, N = 2^n int32 scan through the L2-staged look-back (AUTO at 2^23-2^26), for an
ncu --set full capture of the mid-size regime (launch 3 of 4 is the profiled one).

    ncu --set full --clock-control none --launch-skip 2 --launch-count 1 -k regex:lookback_l2 \
        -o gpurun_out/mid python tools/ncu_mid_case.py 24
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 24
x = torch.empty(1 << n, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 7)
y = torch.empty_like(x)
for _ in range(4):
    sb.scan(x, "add", out=y)
torch.cuda.synchronize()
print("done", sb.plan(x, y))
