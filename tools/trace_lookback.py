"""Timeline of the look-back kernels (scan_debug_trace), 8 u64 per tile:
stamps 0 data ready, 1 aggregate published, 2 inclusive published, 3 outputs written,
4 look-back started; counters 5 descriptor read round trips, 6 windows visited."""
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
ap.add_argument("--tile", type=int, default=0, help="tile elements (default: from the variant)")
ap.add_argument("--save", default="", help="save the raw [tiles, 8] trace as .npy")
a = ap.parse_args()
dt = {"i32": torch.int32, "f32": torch.float32}[a.dtype]
x = torch.empty(a.G * a.N, dtype=torch.int32, device="cuda")
inputs.fill_device(x, {"i32": "i32", "f32": "f32u"}[a.dtype], 7)
x = x.view(dt).view(a.G, a.N)
y = torch.empty_like(x)
TILE = a.tile or {0: 16384, 4: 16384, 9: 16384, 5: 12288, 8: 18432, 6: 4096, 7: 4096, 11: 4096,
                  12: 16384}.get(a.param, 8192)
tiles = (a.G * a.N + TILE - 1) // TILE
tr = torch.zeros(tiles * 8, dtype=torch.int64, device="cuda")
for _ in range(3):
    sb.scan(x, "add", out=y, algo="lookback", param=a.param)
_lib.lib.scan_debug_trace(tr.data_ptr(), tiles)
sb.scan(x, "add", out=y, algo="lookback", param=a.param)
torch.cuda.synchronize()
_lib.lib.scan_debug_trace(None, 0)
R = tr.cpu().numpy().reshape(tiles, 8).astype(np.int64)
if a.save:
    np.save(a.save, R)
T = R[:, :5].copy()
T = T - T[:, 0].min()
print("tiles", tiles, "span us %.1f" % (T[:, 3].max() / 1e3))


def pct(v, name, scale=1e3, unit="us"):
    v = np.asarray(v, dtype=np.float64) / scale
    print("%-30s p10 %7.2f  p50 %7.2f  p90 %7.2f  p99 %7.2f  mean %7.2f %s" % (
        name, *np.percentile(v, [10, 50, 90, 99]), v.mean(), unit))


if R[:, 7].any():          # register-tile kernels also stamp the CTA entry (slot 7)
    E = R[:, 7] - R[:, 7].min()
    Z = R[:, :5] - R[:, 7].min()
    print("entry spread us %.2f; first entry -> last written us %.2f" % (E.max() / 1e3, Z[:, 3].max() / 1e3))
    pct(R[:, 0] - R[:, 7], "entry -> ready (load+scan)")
pct(T[:, 1] - T[:, 0], "ready -> A (pass1)")
pct(T[:, 4] - T[:, 1], "A -> look-back start (queue)")
pct(T[:, 2] - T[:, 4], "look-back duration")
pct(T[:, 3] - T[:, 2], "P -> written (pass2)")
pct(T[:, 3] - T[:, 0], "ready -> written")
pct(R[:, 5], "descriptor round trips", 1, "")
pct(R[:, 6], "windows", 1, "")
lb = (T[:, 2] - T[:, 4]) / np.maximum(R[:, 5], 1)
pct(lb, "look-back time / round trip")
grid = 148 if (TILE >= 12288 or a.param == 3) else 296
if tiles > 2 * grid:
    pct(T[grid:, 0] - T[:-grid, 0], "per-CTA cycle (grid %d)" % grid)
nr = tiles // grid
if nr > 2:
    rr = T[: nr * grid, 0].reshape(nr, grid)
    pct(rr.max(1) - rr.min(1), "data-ready spread per round")
    pa = T[: nr * grid, 1].reshape(nr, grid)
    pct(pa.max(1) - pa.min(1), "A spread per round")
