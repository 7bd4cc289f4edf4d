"""Randomised parity: random shapes, ops, dtypes, kinds, kernel families, variants and
pointer offsets (seeded), each checked element by element against the oracle."""
import random

import numpy as np
import pytest
import torch

import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
from gpu_util import COMBOS, DIST, NP, assert_parity, to_device, to_host
from paper_conf_ipps_dieguezadnm18_b200 import _lib

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("seed", range(int(__import__("os").environ.get("SCANB200_FUZZ_SEEDS", "6"))))
def test_random_cases(seed):
    rng = random.Random(2018 + seed)
    algos = [("auto", -1), ("cascade_cta", -1), ("cascade_warp", -1), ("three_stage", 0), ("three_stage", 3),
             ("packed_warp", -1), ("packed_warp", 300), ("cluster", -1), ("cluster", 32 + 8),
             ("cluster", 64 + 2), ("cluster", 16), ("fused", -1)] + \
            [("lookback", v) for v in _lib.LOOKBACK_VARIANTS]
    for case in range(40):
        N = rng.choice([rng.randint(1, 300), rng.randint(300, 20000), rng.randint(20000, 400000)])
        G = rng.choice([1, 1, 2, rng.randint(1, 40), rng.randint(100, 5000)])
        if N * G > 3_000_000:
            G = max(1, 3_000_000 // N)
        op, dt = rng.choice(COMBOS)
        kind = rng.choice(["inclusive", "exclusive"])
        algo, param = rng.choice(algos)
        off = rng.choice([0, 0, 1, 2, 3])
        x = inputs.generate(DIST[dt], N * G + off, seed=seed * 1000 + case)
        base = to_device(x)
        xin = base[off: off + N * G].view(G, N)
        out = torch.empty(N * G + 4, dtype=base.dtype, device="cuda")[off: off + N * G].view(G, N)
        if algo == "fused" and G > 1 and N % 8192:
            with pytest.raises(sb.ScanError):            # ineligible: rejected, never mis-scanned
                sb.scan(xin, op, kind, out=out, algo=algo, param=param)
            continue
        sb.scan(xin, op, kind, out=out, algo=algo, param=param)
        torch.cuda.synchronize()
        assert_parity(to_host(out, NP[dt]).reshape(G, N), x[off:].reshape(G, N), op, kind,
                      label="fuzz seed=%d case=%d %s/%d %s %s %s N=%d G=%d off=%d" % (
                          seed, case, algo, param, op, dt, kind, N, G, off))


@pytest.mark.parametrize("seed", range(int(__import__("os").environ.get("SCANB200_FUZZ_LARGE_SEEDS", "3"))))
def test_random_multiround_lookback(seed):
    # the persistent L2-staged look-back over many rounds of its round robin (lazy look-back,
    # CTA-local previous prefix, kept tail tiles): random G x N up to 4*10^7 elements, random
    # ops / dtypes / kinds / pointer offsets (offsets take the unaligned, non-TMA path)
    rng = random.Random(7000 + seed)
    for case in range(8):
        total = rng.randint(2_000_000, 40_000_000)
        G = rng.choice([1, 1, 2, 3, rng.randint(4, 64), rng.randint(64, 2000)])
        N = max(1, total // G)
        op, dt = rng.choice(COMBOS)
        kind = rng.choice(["inclusive", "exclusive"])
        param = rng.choice([3, 3, -1])
        off = rng.choice([0, 0, 0, 1, 3])
        x = inputs.generate(DIST[dt], N * G + off, seed=seed * 100 + case)
        base = to_device(x)
        xin = base[off: off + N * G].view(G, N)
        out = torch.empty(N * G + 4, dtype=base.dtype, device="cuda")[off: off + N * G].view(G, N)
        sb.scan(xin, op, kind, out=out, algo="lookback", param=param)
        torch.cuda.synchronize()
        assert_parity(to_host(out, NP[dt]).reshape(G, N), x[off:].reshape(G, N), op, kind,
                      label="fuzz-large seed=%d case=%d lookback/%d %s %s %s N=%d G=%d off=%d" % (
                          seed, case, param, op, dt, kind, N, G, off))


@pytest.mark.parametrize("seed", range(int(__import__("os").environ.get("SCANB200_FUZZ_AUTO_SEEDS", "3"))))
def test_random_auto_mid_batches(seed):
    # AUTO on the batch regions re-measured in round 2 session 3 (DESIGN.md §5 items 11-12):
    # 65 < G < 300 in the latency-bound middle (three-stage), a few hundred to a few
    # thousand problems just above 2^16 (one CTA per problem), and their neighbours that stay
    # on the look-back -- tile-aligned and ragged N, every op / dtype / kind
    rng = random.Random(9000 + seed)
    for case in range(6):
        G = rng.choice([rng.randint(65, 299), rng.randint(300, 1100), rng.randint(1100, 3000)])
        N = rng.choice([65536, 65540, rng.randint(65537, 140000) & ~3, rng.randint(4096, 60000) & ~3,
                        rng.randint(140000, 300000) | 1])
        if N * G > 40_000_000:
            G = max(1, 40_000_000 // N)
        op, dt = rng.choice(COMBOS)
        kind = rng.choice(["inclusive", "exclusive"])
        x = inputs.generate(DIST[dt], N * G, seed=seed * 100 + case + 77)
        xd = to_device(x).view(G, N)
        plan = sb.plan(xd, op=op, kind=kind)
        out = sb.scan(xd, op, kind)
        torch.cuda.synchronize()
        assert_parity(to_host(out, NP[dt]).reshape(G, N), x.reshape(G, N), op, kind,
                      label="fuzz-auto seed=%d case=%d %s/%d %s %s %s N=%d G=%d" % (
                          seed, case, plan[0], plan[1], op, dt, kind, N, G))
        del xd, out
