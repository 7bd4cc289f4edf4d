"""Run one scan configuration a few times (for ncu / compute-sanitizer captures).

    python tools/prof_case.py --dtype i32 --G 1 --N 268435456 --algo lookback --param 3 --reps 3
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--dtype", default="i32")
ap.add_argument("--G", type=int, default=1)
ap.add_argument("--N", type=int, default=1 << 28)
ap.add_argument("--algo", default="auto")
ap.add_argument("--param", type=int, default=-1)
ap.add_argument("--op", default="add")
ap.add_argument("--kind", default="inclusive")
ap.add_argument("--reps", type=int, default=3)
a = ap.parse_args()
dt = {"i32": torch.int32, "u32": torch.uint32, "f32": torch.float32}[a.dtype]
x = torch.empty(a.G * a.N, dtype=torch.int32, device="cuda")
inputs.fill_device(x, {"i32": "i32", "u32": "u32", "f32": "f32u"}[a.dtype], 7)
x = x.view(dt).view(a.G, a.N)
y = torch.empty_like(x)
for _ in range(a.reps):
    sb.scan(x, a.op, a.kind, out=y, algo=a.algo, param=a.param)
torch.cuda.synchronize()
print("done")
