"""Where the end of an L2-staged look-back call goes: per-round timeline of a saved
scan_debug_trace (tools/trace_lookback.py --save X.npy) with, for every tile, the latest
aggregate (A) in its look-back window, its CTA's previous inclusive prefix (P of t - grid),
and which of the two bound its own P; plus per-CTA progress (cycle time, lateness).

    python tools/tail_analysis.py X.npy [grid]
"""
import sys

import numpy as np

R = np.load(sys.argv[1]).astype(np.int64)
grid = int(sys.argv[2]) if len(sys.argv) > 2 else 148
tiles = R.shape[0]
t0 = R[:grid, 7].min()                     # first CTA entry
T = (R[:, :5] - t0) / 1e3                  # 0 ready, 1 A, 2 P, 3 written, 4 look-back start (us)
nr = tiles // grid
print("tiles %d, grid %d, %.1f rounds; first CTA entry = 0" % (tiles, grid, tiles / grid))
E = (R[:grid, 7] - t0) / 1e3
print("CTA entry spread %.2f us; first data ready min %.2f p50 %.2f max %.2f us" % (
    E.max(), T[:grid, 0].min(), np.median(T[:grid, 0]), T[:grid, 0].max()))
print("last ready %.2f  last A %.2f  last P %.2f  last written %.2f us  (drain = last ready -> last written %.2f)" % (
    T[:, 0].max(), T[:, 1].max(), T[:, 2].max(), T[:, 3].max(), T[:, 3].max() - T[:, 0].max()))

rd = T[:nr * grid, 0].reshape(nr, grid)
late = rd - np.median(rd, axis=1, keepdims=True)
x = np.arange(2, nr)
slopes = np.array([np.polyfit(x, rd[2:, b], 1)[0] for b in range(grid)])
print("per-CTA cycle (us/tile): min %.3f p50 %.3f max %.3f; lateness in the last full round: %.2f .. %.2f us"
      % (slopes.min(), np.median(slopes), slopes.max(), late[-1].min(), late[-1].max()))
print("corr(cycle, lateness) %.2f; corr(lateness round 2, last round) %.2f" % (
    np.corrcoef(slopes, late[-1])[0, 1], np.corrcoef(late[2], late[-1])[0, 1]))

print("\nlast three rounds (us): ready / A / window-A max / look-back start / P / written")
for rnd in range(max(0, (tiles - 1) // grid - 2), (tiles - 1) // grid + 1):
    lo, hi = rnd * grid, min(tiles, rnd * grid + grid)
    rows = []
    for t in range(lo, hi):
        w0 = max(0, t - grid + 1)
        wA = T[w0:t, 1].max() if t > w0 else 0.0
        pp = T[t - grid, 2] if t >= grid else 0.0
        rows.append((T[t, 0], T[t, 1], wA, T[t, 4], T[t, 2], pp, T[t, 3]))
    a = np.array(rows)
    bound_chain = np.mean(a[:, 5] > np.maximum(a[:, 1], a[:, 2]))
    print("round %2d (%3d tiles): ready %5.2f-%5.2f  A max %5.2f  winA p50 %5.2f  P p50 %5.2f max %5.2f  "
          "written max %5.2f | P - max(A, winA) p50 %.2f, P - P(t-grid) p50 %.2f, chain-bound %.0f %%, "
          "lb start - A p50 %.2f, written - P p50 %.2f" % (
              rnd, hi - lo, a[:, 0].min(), a[:, 0].max(), a[:, 1].max(), np.median(a[:, 2]), np.median(a[:, 4]),
              a[:, 4].max(), a[:, 6].max(), np.median(a[:, 4] - np.maximum(a[:, 1], a[:, 2])),
              np.median(a[:, 4] - a[:, 5]), 100 * bound_chain, np.median(a[:, 3] - a[:, 1]),
              np.median(a[:, 6] - a[:, 4])))
