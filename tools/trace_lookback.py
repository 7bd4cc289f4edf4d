"""Timeline of the pipelined look-back kernel (scan_debug_trace): per-tile stamps
0 data ready, 1 aggregate published, 2 inclusive published, 3 outputs written."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402
from paper_conf_ipps_dieguezadnm18_b200 import _lib  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--dtype", default="i32")
ap.add_argument("--G", type=int, default=1)
ap.add_argument("--N", type=int, default=1 << 28)
ap.add_argument("--param", type=int, default=0)
a = ap.parse_args()
dt = {"i32": torch.int32, "f32": torch.float32}[a.dtype]
x = torch.empty(a.G * a.N, dtype=torch.int32, device="cuda")
inputs.fill_device(x, {"i32": "i32", "f32": "f32u"}[a.dtype], 7)
x = x.view(dt).view(a.G, a.N)
y = torch.empty_like(x)
TILE = 16384 if a.param == 1 else 8192
tiles = (a.G * a.N + TILE - 1) // TILE
tr = torch.zeros(tiles * 4, dtype=torch.int64, device="cuda")
for _ in range(3):
    sb.scan(x, "add", out=y, algo="lookback", param=a.param)
_lib.lib.scan_debug_trace(tr.data_ptr(), tiles)
sb.scan(x, "add", out=y, algo="lookback", param=a.param)
torch.cuda.synchronize()
_lib.lib.scan_debug_trace(None, 0)
T = tr.cpu().numpy().reshape(tiles, 4).astype(np.int64)
T = T - T[:, 0].min()
ok = (T[:, 0] >= 0) & (T[:, 3] > 0)
print("tiles", tiles, "stamped", int(ok.sum()), "span us %.1f" % (T[:, 3].max() / 1e3))


def pct(v, name):
    v = np.asarray(v, dtype=np.float64) / 1e3
    print("%-28s p10 %7.2f  p50 %7.2f  p90 %7.2f  p99 %7.2f  mean %7.2f us" % (
        name, *np.percentile(v, [10, 50, 90, 99]), v.mean()))


pct(T[:, 1] - T[:, 0], "ready -> A (pass1)")
pct(T[:, 2] - T[:, 1], "A -> P (look-back)")
pct(T[:, 3] - T[:, 2], "P -> written (pass2)")
pct(T[:, 3] - T[:, 0], "ready -> written")
for grid in (296, 148) if TILE == 8192 else (148,):
    if tiles > 2 * grid:
        cyc = T[grid:, 0] - T[:-grid, 0]
        pct(cyc, "per-CTA cycle (grid %d)" % grid)
pct(np.maximum(T[1:, 1], T[:-1, 2]) - T[1:, 1], "wait on pred P after own A")
pct(T[1:, 2] - T[:-1, 2], "P(t) - P(t-1)")
# front: P publish time vs tile index
for q in (0.1, 0.25, 0.5, 0.75, 0.9, 1.0):
    k = int(q * (tiles - 1))
    print("tile %8d  ready %8.1f  A %8.1f  P %8.1f  done %8.1f us" % (k, *(T[k] / 1e3)))
