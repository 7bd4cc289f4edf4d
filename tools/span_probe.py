"""packed_warp span length for ragged short rows: span targets 4096 .. 65536 elements vs the
default choice (2048..8192, best window use), ~1 GiB of int32 per shape (G = 2^28/N),
device time per call, % of measured copy.

    python tools/span_probe.py
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402
from tools.short_probe import t, PEAK  # noqa: E402  (runs nothing at import? see below)
from tools.short_probe import x, y  # noqa: E402  (the 1 GiB buffers)

for N in [3, 100, 255, 257, 300, 600, 700, 1000, 1023]:
    G = (1 << 28) // N
    xv, yv = x[:G * N].view(G, N), y[:G * N].view(G, N)
    row = {"N": N, "G": G, "auto": "%s/%d" % sb.plan(xv)}
    for param in (-1, 4096, 8192, 12288, 16384, 32768, 65536):
        ms = t(xv, yv, "packed_warp", param)
        row["span%d" % param] = round(8.0 * G * N / ms / 1e6 / PEAK, 4)
    print(json.dumps(row), flush=True)
