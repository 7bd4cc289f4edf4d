"""Quick on-box parity of look-back variants (experiments) against the oracle: the
test_lookback_variants shapes plus multi-round shapes of the persistent L2-staged kernel.

    python tools/variant_parity.py 3 20 21 ...
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402
from gpu_util import COMBOS, DIST, NP, assert_parity, to_device, to_host  # noqa: E402

SHAPES = [(1, 3000), (3, 5000), (100, 333), (8193, 5), (65536 + 17, 3), (1 << 20, 1),
          ((1 << 23) + 123, 1), (3000017, 3), (1 << 17, 2048), (1 << 24, 1), (7777777, 2),
          (65540, 2048), (200003, 700), (8191 * 3, 1001)]

for v in [int(a) for a in sys.argv[1:]]:
    n = 0
    for op, dt in COMBOS:
        for N, G in SHAPES:
            if N * G > (1 << 22) and (op, dt) not in (("add", "i32"), ("add", "f32")):
                continue
            x = inputs.generate(DIST[dt], N * G, seed=N + G + v).reshape(G, N)
            for kind in ("inclusive", "exclusive"):
                out = sb.scan(to_device(x), op, kind, algo="lookback", param=v)
                torch.cuda.synchronize()
                assert_parity(to_host(out, NP[dt]).reshape(G, N), x, op, kind,
                              label="v%d %s %s %s N=%d G=%d" % (v, op, dt, kind, N, G))
                n += 1
    print("variant %d: %d cases exact/within tolerance" % (v, n), flush=True)
