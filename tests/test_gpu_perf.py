"""Perf-regression floors on the BASELINE configs, read from
tests/perf_floors.json.  The floors sit well below the measured round-1 numbers
(profiles/r01_bench_n1.json, r01_paper_sweep_*.jsonl): they catch a dispatch mistake or a
kernel regression, not box-to-box noise.  Device time from CUDA events (large configs) or
CUDA-graph replays (latency-bound ones)."""
import json
import os

import pytest
import torch

import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
FLOORS = json.load(open(os.path.join(os.path.dirname(__file__), "perf_floors.json")))


def _peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    return float(json.load(open(p))["hbm_gbs"]) if os.path.exists(p) else 6650.0


def _ms(fn, reps):
    for _ in range(2):
        fn()
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    s0.record()
    for _ in range(reps):
        fn()
    s1.record()
    torch.cuda.synchronize()
    return s0.elapsed_time(s1) / reps


def _graph_us(fn, reps=20):
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(reps):
            fn()
    g.replay()
    torch.cuda.synchronize()
    best = None
    for _ in range(3):
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s0.record(s)
        with torch.cuda.stream(s):
            g.replay()
        s1.record(s)
        torch.cuda.synchronize()
        t = s0.elapsed_time(s1) / reps * 1e3
        best = t if best is None else min(best, t)
    return best


def _frac(elems, ms):
    return 8.0 * elems / (ms * 1e-3) / 1e9 / _peak()


def test_c2_batch_rate():
    G, N = 4096, 1 << 14
    for dist, dt in (("i32", torch.int32), ("f32u", torch.float32)):
        x = torch.empty(G * N, dtype=torch.int32, device="cuda")
        inputs.fill_device(x, dist, 2)
        x = x.view(dt).view(G, N)
        y = torch.empty_like(x)
        for kind in ("inclusive", "exclusive"):
            f = _frac(G * N, _ms(lambda: sb.scan(x, "add", kind, out=y), 20))
            assert f >= FLOORS["c2_frac_min"], (dist, kind, f)


def test_c3_single_problem_rate():
    N = 1 << 30
    x = torch.empty(N, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "f32u", 3)
    x = x.view(torch.float32)
    y = torch.empty_like(x)
    f = _frac(N, _ms(lambda: sb.scan(x, "add", out=y), 5))
    assert f >= FLOORS["c3_frac_min"], f


def test_c4_rank_shard_rate():
    # configs[3] per GPU at W = 8: 2^13 problems of 2^16
    G, N = 1 << 13, 1 << 16
    x = torch.empty(G * N, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32", 4)
    x = x.view(G, N)
    y = torch.empty_like(x)
    f = _frac(G * N, _ms(lambda: sb.scan(x, "add", out=y), 10))
    assert f >= FLOORS["c4_shard_frac_min"], f


def test_paper_sweep_rates():
    # the paper's workload: 2^28 int32 as G = 2^28/N problems
    T = 1 << 28
    x = torch.empty(T, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32", 5)
    y = torch.empty_like(x)
    for n in (10, 13, 16, 17, 18, 20, 24, 28):
        N = 1 << n
        xv, yv = x.view(T // N, N), y.view(T // N, N)
        f = _frac(T, _ms(lambda: sb.scan(xv, "add", out=yv), 5))
        assert f >= FLOORS["paper_sweep_frac_min"], (n, sb.plan(xv, yv), f)


def test_latency_bound_configs():
    x = torch.empty(1 << 20, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32", 1)
    y = torch.empty_like(x)
    us = _graph_us(lambda: sb.scan(x, "add", out=y))
    assert us <= FLOORS["c1_us_max"], us                       # configs[0]
    for N in (1 << 12, 1 << 15):                                # one CTA / one cluster
        xv, yv = x[:N], y[:N]
        us = _graph_us(lambda: sb.scan(xv, "add", out=yv))
        assert us <= FLOORS["g1_small_us_max"], (N, sb.plan(xv, yv), us)


def test_mid_size_single_problem_rates():
    # G = 1, N = 2^24 / 2^25 / 2^26: the L2-staged look-back's fill and drain are a large
    # share of the call (round 2: 0.82-0.86 / 0.92-0.94 / 0.98 of copy after session 3)
    x = torch.empty(1 << 26, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32", 6)
    y = torch.empty_like(x)
    for n, key in ((24, "g1_2e24_frac_min"), (25, "g1_2e25_frac_min"), (26, "g1_2e26_frac_min")):
        N = 1 << n
        xv, yv = x[:N], y[:N]
        f = _frac(N, _graph_us(lambda: sb.scan(xv, "add", out=yv)) * 1e-3)
        assert f >= FLOORS[key], (n, sb.plan(xv, yv), f)


def test_ragged_batch_rates():
    # problems whose starts fall inside look-back tiles, and the latency-bound middle
    # (round 2 session 3: AUTO sends them to one CTA per problem / the three-stage form;
    # profiles/r02_cascade_boundary.jsonl, r02_mid_batch_shapes.jsonl)
    x = torch.empty(2048 * 65540, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32", 8)
    y = torch.empty_like(x)
    for (G, N), key in (((2048, 65540), "ragged_batch_frac_min"), ((160, 65536), "mid_batch_frac_min"),
                        ((100, 65540), "mid_batch_frac_min")):
        xv, yv = x[:G * N].view(G, N), y[:G * N].view(G, N)
        f = _frac(G * N, _graph_us(lambda: sb.scan(xv, "add", out=yv)) * 1e-3)
        assert f >= FLOORS[key], (G, N, sb.plan(xv, yv), f)


def test_short_portion_sharded_rates():
    # the sharded pipeline with short per-rank portions (warp per problem, DESIGN §8 item 4):
    # Scan-MPS at W = 8 for n <= 15 gives each rank G >= 8192 portions of <= 4096 elements.
    # Stage 1+2 reads 4 B/elem, Stage 3 moves 8 B/elem (profiles/r02_warp_shard_ab.txt:
    # 1.13 / 1.02 of copy at N_local = 1024; the CTA path read 0.33 / 0.28)
    T = 1 << 28
    x = torch.empty(T, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32", 9)
    y = torch.empty_like(x)
    for N in (1024, 4096):
        G = T // N
        xv, yv = x.view(G, N), y.view(G, N)
        tot = sb.shard_totals(xv, "add")
        allt = tot.view(1, G).clone()
        us12 = _graph_us(lambda: sb.shard_totals(xv, "add", totals=tot))
        us3 = _graph_us(lambda: sb.shard_scan(xv, allt, 0, 1, "add", "inclusive", out=yv))
        f12 = _frac(T, us12 * 1e-3) / 2          # 4 B/elem
        f3 = _frac(T, us3 * 1e-3)
        assert f12 >= FLOORS["short_portion_stage12_frac_min"], (N, f12)
        assert f3 >= FLOORS["short_portion_stage3_frac_min"], (N, f3)


def test_mid_batch_aligned_rates():
    # tile-aligned rows of 40960-65536 elements at 148 < G <= 600 (look-back since the
    # 60-shape grid, profiles/r02_mid_batch_dispatch_final.jsonl: 0.68-0.93 of copy)
    x = torch.empty(600 * 65536, dtype=torch.int32, device="cuda")
    inputs.fill_device(x, "i32", 10)
    y = torch.empty_like(x)
    for G, N in ((200, 65536), (500, 49152), (600, 65536)):
        xv, yv = x[:G * N].view(G, N), y[:G * N].view(G, N)
        f = _frac(G * N, _graph_us(lambda: sb.scan(xv, "add", out=yv)) * 1e-3)
        assert f >= FLOORS["mid_aligned_frac_min"], (G, N, sb.plan(xv, yv), f)
