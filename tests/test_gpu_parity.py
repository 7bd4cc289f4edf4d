"""Kernel parity on the B200: every kernel family, op, dtype and kind against the oracle.

Sizes span several tiles (4096 / 8192 elements) and ragged tails; G > 1 exercises the
batch boundaries.  Integer add/max and f32 max are compared bit for bit;
f32 add within 1e-5 * sum|x| of the fp64 sequential scan (north_star).
"""
import numpy as np
import pytest
import torch

import inputs
import oracle
import paper_conf_ipps_dieguezadnm18_b200 as sb
from paper_conf_ipps_dieguezadnm18_b200 import _lib
from gpu_util import COMBOS, DIST, NP, TORCH, assert_parity, device_inputs, to_device, to_host

pytestmark = pytest.mark.gpu

NS = [1, 2, 3, 4, 5, 7, 31, 32, 33, 127, 128, 129, 511, 513, 1023, 1024, 1025, 4095, 4096, 4097,
      8191, 8192, 8193, 16383, 16385, 3 * 8192 + 5, 100003]
GS = [1, 2, 3, 7]
ALGOS = ["lookback", "cascade_cta", "cascade_warp", "three_stage", "packed_warp", "cluster"]


def _run(x, op, kind, algo="auto", param=-1):
    xd = to_device(x)
    out = sb.scan(xd, op, kind, algo=algo, param=param)
    torch.cuda.synchronize()
    return to_host(out, x.dtype)


@pytest.mark.parametrize("algo", ALGOS)
@pytest.mark.parametrize("op,dt", COMBOS)
@pytest.mark.parametrize("kind", ["inclusive", "exclusive"])
def test_shapes_all_algos(algo, op, dt, kind):
    for N in NS:
        for G in GS:
            x = inputs.generate(DIST[dt], N * G, seed=1000 + N * 7 + G).reshape(G, N)
            got = _run(x, op, kind, algo)
            assert_parity(got, x, op, kind, label="%s %s %s %s N=%d G=%d" % (algo, op, dt, kind, N, G))


@pytest.mark.parametrize("variant", _lib.LOOKBACK_VARIANTS)
def test_lookback_variants(variant):
    for op, dt in COMBOS:
        for N, G in [(1, 3000), (3, 5000), (100, 333), (8193, 5), (65536 + 17, 3), (1 << 20, 1)]:
            x = inputs.generate(DIST[dt], N * G, seed=N + G).reshape(G, N)
            for kind in ("inclusive", "exclusive"):
                got = _run(x, op, kind, "lookback", variant)
                assert_parity(got, x, op, kind, label="v%d %s %s N=%d G=%d" % (variant, op, dt, N, G))


@pytest.mark.parametrize("variant", range(3))
def test_cluster_sizes(variant):
    # every cluster size (1..16 CTAs, DSMEM aggregate exchange), one round and several
    # rounds of csize tiles (register carry between rounds), ragged tails, G > 1
    for csize in (1, 2, 4, 8, 16):
        for op, dt in COMBOS:
            for N, G in [(5, 3), (4096 * csize - 3, 2), (16384 * csize + 4097, 1), (100003, 3)]:
                x = inputs.generate(DIST[dt], N * G, seed=N + 31 * G + csize).reshape(G, N)
                for kind in ("inclusive", "exclusive"):
                    got = _run(x, op, kind, "cluster", 32 * variant + csize)
                    assert_parity(got, x, op, kind, label="cluster v%d c%d %s %s %s N=%d G=%d" % (
                        variant, csize, op, dt, kind, N, G))


@pytest.mark.parametrize("K", [1, 2, 5])
def test_three_stage_cascade_depth(K):
    # Fig. 5 cascade depth: any K gives the same integer result
    x = inputs.generate("i32", 3 * 200001, 77).reshape(3, 200001)
    ref = _run(x, "add", "inclusive", "three_stage", 0)
    got = _run(x, "add", "inclusive", "three_stage", K)
    assert np.array_equal(got, ref)
    assert_parity(got, x, "add", "inclusive")


def test_three_stage_many_chunks():
    # long portions are cut into <= 16-tile chunks; more than 256 chunks per problem switch
    # Stage 2 to one CTA per problem (1024 chunk values per round, ragged last round)
    for op, dt in COMBOS:
        for G, N in [(1, (1 << 25) + 12345), (2, 300 * 65536 + 7)]:
            x = inputs.generate(DIST[dt], G * N, seed=N % 977).reshape(G, N)
            for kind in ("inclusive", "exclusive"):
                got = _run(x, op, kind, "three_stage", 0)
                assert_parity(got, x, op, kind, label="3stage-many %s %s %s G=%d" % (op, dt, kind, G))
            if op == "add" and dt == "i32":
                got1 = _run(x, op, "inclusive", "three_stage", 1)      # 1-tile chunks: Bx > 8000
                assert_parity(got1, x, op, "inclusive", label="3stage K=1")


def test_misaligned_and_inplace():
    for op, dt in COMBOS:
        N, G = 12347, 3
        x = inputs.generate(DIST[dt], N * G + 3, seed=5)
        base = to_device(x)
        for off in (1, 2, 3):                          # 4, 8, 12-byte offsets: not 16-aligned
            xin = base[off: off + N * G].view(G, N)
            for algo in ALGOS:
                out = torch.empty(N * G + 4, dtype=base.dtype, device="cuda")[1: 1 + N * G].view(G, N)
                sb.scan(xin, op, "inclusive", out=out, algo=algo)
                torch.cuda.synchronize()
                assert_parity(to_host(out, NP[dt]), x[off: off + N * G].reshape(G, N), op, "inclusive",
                              label="misaligned %s %s off=%d" % (algo, op, off))
        # in place
        for algo in ALGOS:
            xx = inputs.generate(DIST[dt], 3 * 70001, seed=6).reshape(3, 70001)
            t = to_device(xx)
            sb.scan(t, op, "exclusive", out=t, algo=algo)
            torch.cuda.synchronize()
            assert_parity(to_host(t, NP[dt]), xx, op, "exclusive", label="inplace " + algo)


def test_batch_isolation():
    # T3: a carry leaking across a problem boundary would corrupt the next problem
    G, N = 9, 5000
    for algo in ALGOS:
        x = np.zeros((G, N), np.int32)
        x[0::2, :] = 2**31 - 1
        x[1::2, :] = 1
        got = _run(x, "add", "inclusive", algo)
        assert_parity(got, x, "add", "inclusive", label="isolation " + algo)
        xm = np.full((G, N), -5, np.int32)
        xm[0, :] = 2**31 - 1
        assert_parity(_run(xm, "max", "inclusive", algo), xm, "max", "inclusive")


def test_degenerate_shapes():
    for algo in ALGOS:
        for shape in [(0,), (0, 5), (5, 0)]:
            x = torch.zeros(shape, dtype=torch.int32, device="cuda")
            out = sb.scan(x, "add", algo=algo)
            assert out.shape == x.shape
        # N = 1: inclusive = x, exclusive = identity
        x = inputs.generate("i32", 1000, 3).reshape(1000, 1)
        assert np.array_equal(_run(x, "add", "inclusive", algo), x)
        assert np.all(_run(x, "max", "exclusive", algo) == np.iinfo(np.int32).min)


def test_closed_form_c1():
    # configs[0]: inclusive add int32, N = 2^20, G = 1; north_star closed form out[i] = i(i+1)/2
    N = 1 << 20
    x = inputs.generate("iota", N, 0, row_len=N)
    got = _run(x, "add", "inclusive")
    j = np.arange(N, dtype=np.int64)
    want = (((j + 1) * (j + 2) // 2) & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
    assert np.array_equal(got, want)
    assert got[-1] == 524288
    xr = inputs.generate("i32", N, 0x5CA2018 + 1)
    assert_parity(_run(xr, "add", "inclusive"), xr, "add", "inclusive")


def test_generator_device_matches_host():
    for dist in ("i32", "u32", "f32u", "f32s", "small"):
        d = device_inputs(dist, 100003, 42, offset=12345)
        h = inputs.generate(dist, 100003, 42, offset=12345)
        assert np.array_equal(to_host(d, h.dtype), h), dist
    d = device_inputs("iota", 1000, 0, row_len=77)
    assert np.array_equal(to_host(d, np.int32), inputs.generate("iota", 1000, 0, row_len=77))


def test_determinism_ints_and_three_stage_f32():
    x = inputs.generate("i32", 1 << 22, 9)
    outs = [_run(x, "add", "inclusive") for _ in range(5)]
    assert all(np.array_equal(outs[0], o) for o in outs[1:])
    xf = inputs.generate("f32u", 1 << 22, 9)
    outs = [_run(xf, "add", "inclusive", "three_stage") for _ in range(5)]
    assert all(np.array_equal(outs[0], o) for o in outs[1:])


@pytest.mark.parametrize("param,N,G", [(-1, 300001, 2), (3, (1 << 23) + 123, 1), (3, 3000017, 3)])
def test_cuda_graph_replay_self_cleaning(param, N, G):
    # the look-back descriptors are reset-free (epoch tags): replaying a captured launch
    # must stay correct without any memset between replays -- also for the cooperative,
    # persistent L2-staged kernel over many rounds (param 3)
    x = inputs.generate("f32s", N * G, 3).reshape(G, N)
    xd = to_device(x)
    out = torch.empty_like(xd)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        sb.scan(xd, "add", out=out, algo="lookback", param=param)       # warm-up (workspace allocation)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        sb.scan(xd, "add", out=out, algo="lookback", param=param)
    for _ in range(20):
        out.zero_()
        g.replay()
    torch.cuda.synchronize()
    assert_parity(to_host(out, np.float32), x, "add", "inclusive", label="graph param=%d" % param)


@pytest.mark.parametrize("param", [0, 2, 3, 10])
def test_epoch_wrap_with_caller_workspace(param):
    # poke the epoch counter of a caller workspace to just below the 30-bit wrap and run
    # across it: the wrap launch's end-of-grid epilogue clears every descriptor (every
    # other launch advances the epoch at the start of its grid), for each look-back kernel
    N, G = 1 << 18, 3
    for op, dt in [("add", "i32"), ("add", "f32")]:
        nbytes = sb.workspace_bytes(N, G, op, TORCH[dt], "lookback", param)
        ws = torch.zeros((nbytes + 7) // 8, dtype=torch.int64, device="cuda")
        ctl = ws.view(torch.int32)
        ctl[2] = 0x3FFFFFFF - 4
        for it in range(8):
            x = inputs.generate(DIST[dt], N * G, 100 + it).reshape(G, N)
            xd = to_device(x)
            out = sb.scan(xd, op, "inclusive", algo="lookback", param=param, workspace=ws)
            torch.cuda.synchronize()
            assert_parity(to_host(out, NP[dt]), x, op, "inclusive", label="wrap it=%d" % it)
        assert int(ctl[2]) < 16


def test_c2_full_size_all_variants():
    # configs[1]: G = 4096 problems of N = 2^14, int32 and f32, inclusive and exclusive
    G, N = 4096, 1 << 14
    for dt, dist in (("i32", "i32"), ("f32", "f32u"), ("f32", "f32s")):
        xd = device_inputs(dist, G * N, 0x5CA2018 + 2).view(G, N)
        x = to_host(xd, NP[dt]).reshape(G, N)
        for kind in ("inclusive", "exclusive"):
            for algo in ALGOS:
                out = sb.scan(xd, "add", kind, algo=algo)
                torch.cuda.synchronize()
                assert_parity(to_host(out, NP[dt]).reshape(G, N), x, "add", kind, label="c2 %s %s" % (algo, kind))
        out = sb.scan(xd, "max", "inclusive")
        torch.cuda.synchronize()
        assert_parity(to_host(out, NP[dt]).reshape(G, N), x, "max", "inclusive")


@pytest.mark.parametrize("dist,kind", [("f32u", "inclusive"), ("f32s", "inclusive"), ("f32u", "exclusive")])
def test_c3_full_size_streamed(dist, kind):
    # configs[2]: one f32 add-scan of N = 2^30 (decoupled look-back); the whole output is
    # checked against the streaming oracle, 2^26 elements at a time
    N = 1 << 30
    xd = device_inputs(dist, N, 0x5CA2018 + 3)
    out = sb.scan(xd, "add", kind)
    torch.cuda.synchronize()
    so = oracle.StreamAdd(np.float32, kind)
    step = 1 << 26
    worst = 0.0
    for a in range(0, N, step):
        xc = to_host(xd[a: a + step], np.float32)
        gc = to_host(out[a: a + step], np.float32)
        ref, sabs = so.feed(xc)
        err = np.abs(gc.astype(np.float64) - ref)
        assert np.all(err <= 1e-5 * sabs), "c3 chunk %d" % (a // step)
        worst = max(worst, float(np.max(err / np.maximum(sabs, 1e-300))))
    print("c3 %s %s worst |err|/sum|x| = %.3g" % (dist, kind, worst))


def test_c4_shard_full_size_int32():
    # configs[3] per-GPU shard at W = 8: 2^13 problems of 2^16 int32 (problems mode)
    G, N = 1 << 13, 1 << 16
    xd = device_inputs("i32", G * N, 0x5CA2018 + 4).view(G, N)
    out = sb.scan(xd, "add")
    torch.cuda.synchronize()
    x = to_host(xd, np.int32).reshape(G, N)
    assert_parity(to_host(out, np.int32).reshape(G, N), x, "add", "inclusive")


def test_sharded_loopback_elements_mode():
    # T5: elements mode with W virtual ranks on one GPU; the all-gather
    # is a device concatenation.  Uneven portions, an empty one and ones shorter than a tile.
    for op, dt in COMBOS:
        for G, lens in [(1, [100000, 0, 37, 4096, 250003]), (3, [5, 8192, 0, 70001]), (2, [1 << 20] * 4)]:
            Ntot = sum(lens)
            x = inputs.generate(DIST[dt], G * Ntot, seed=len(lens) * 7 + G).reshape(G, Ntot)
            for kind in ("inclusive", "exclusive"):
                parts, totals, wss = [], [], []
                starts = np.cumsum([0] + lens)
                for r, L in enumerate(lens):
                    xl = to_device(np.ascontiguousarray(x[:, starts[r]: starts[r] + L]))
                    # each virtual rank keeps its own workspace (its chunk prefixes) between
                    # the two steps, as each real rank does on its own device
                    nb = int(sb._lib.lib.scan_shard_workspace_bytes(L, G))
                    wss.append(torch.zeros((nb + 7) // 8, dtype=torch.int64, device="cuda"))
                    totals.append(sb.shard_totals(xl, op, workspace=wss[-1]))
                    parts.append(xl)
                all_t = torch.stack(totals)                     # [W][G]
                outs = []
                for r, xl in enumerate(parts):
                    outs.append(sb.shard_scan(xl, all_t, r, len(lens), op, kind, workspace=wss[r]))
                torch.cuda.synchronize()
                got = np.concatenate([to_host(o, NP[dt]).reshape(G, -1) for o in outs], axis=1)
                assert_parity(got, x, op, kind, label="sharded %s %s %s lens=%s" % (op, dt, kind, lens))


def test_host_buffer_path():
    # scan_batch_host: H2D + scan + D2H pipelined in the library (the e2e path)
    for op, dt in COMBOS:
        for N, G in [(1000, 3), (1 << 14, 4096), ((1 << 24) + 12345, 1), (3 * (1 << 24) + 7, 2)]:
            if N * G > (1 << 26) and not (op == "add" and dt in ("i32", "f32")):
                continue
            x = inputs.generate(DIST[dt], N * G, seed=N % 1000 + G).reshape(G, N)
            pin = torch.empty(x.shape, dtype=torch.int32, pin_memory=True).numpy().view(x.dtype)
            pin[...] = x
            got = sb.scan_host(pin, op, "inclusive")
            assert_parity(got, x, op, "inclusive", label="host %s %s N=%d G=%d" % (op, dt, N, G))
            got = sb.scan_host(x, op, "exclusive")                # pageable
            assert_parity(got, x, op, "exclusive", label="host-pageable %s %s" % (op, dt))


def test_error_paths():
    x = torch.zeros(100, dtype=torch.int32, device="cuda")
    with pytest.raises(sb.ScanError):
        sb.scan(x[:60], out=x[10:70])                           # partial overlap
    from paper_conf_ipps_dieguezadnm18_b200 import _lib
    h = np.zeros(100, np.int32)
    rc = _lib.lib.scan_batch(h.ctypes.data, h.ctypes.data, 100, 1, 0, 0, 0, None)
    assert rc == 1                                              # host pointer -> INVALID_ARG


@pytest.mark.parametrize("param", [-1, 100, 4096])
def test_packed_short_rows(param):
    # several whole short problems per warp (segmented spans, PAPER.md:98 L_x < 32): every
    # residue of N mod 4 (span alignment), spans shorter / longer than one window, ragged G
    for op, dt in COMBOS:
        for N in [1, 2, 3, 5, 17, 64, 100, 255, 256, 257, 511, 1000, 1023, 1030]:
            G = 150001 // N + 3
            x = inputs.generate(DIST[dt], N * G, seed=N * 31 + G).reshape(G, N)
            for kind in ("inclusive", "exclusive"):
                got = _run(x, op, kind, "packed_warp", param)
                assert_parity(got, x, op, kind, label="packed p=%d %s %s %s N=%d" % (param, op, dt, kind, N))


def test_auto_short_rows_use_packed():
    x = torch.zeros((4096, 300), dtype=torch.int32, device="cuda")
    assert sb.plan(x)[0] == "packed_warp"
    assert sb.plan(torch.zeros((1 << 21, 1), dtype=torch.int32, device="cuda"))[0] == "packed_warp"
    y = torch.zeros((4096, 1000), dtype=torch.int32, device="cuda")
    assert sb.plan(y)[0] == "cascade_warp"


def test_auto_dispatch_regions():
    # the measured regions of choose_algo (profiles/r01_cluster_probe.jsonl,
    # r01_autotune_probe.jsonl); each shape must also scan exactly through AUTO
    want = {(1, 4096): "cascade_cta", (100, 8192): "cascade_cta", (1, 20000): "cluster", (4, 32768): "cluster", (4, 65536): "three_stage",
            (64, 65536): "three_stage", (1, 1 << 20): "three_stage", (1000, 1000): "cascade_warp",
            (256, 4096): "cascade_cta", (1024, 65536): "cascade_cta", (1, 1 << 21): "three_stage", (1, 1 << 22): "fused", (1, 1 << 23): "lookback",
            (4096, 16384): "cascade_cta", (300, 65540): "cascade_cta", (160, 65540): "three_stage", (120, 100003): "lookback",
            (100, 20484): "three_stage", (160, 40960): "lookback", (100, 12292): "cascade_cta"}
    sb.autotune_clear()
    for (G, N), algo in want.items():
        x = inputs.generate("i32", G * N, seed=G + N).reshape(G, N)
        xd = to_device(x)
        assert sb.plan(xd)[0] == algo, (G, N, sb.plan(xd))
        out = sb.scan(xd, "add", "exclusive")
        torch.cuda.synchronize()
        assert_parity(to_host(out, x.dtype), x, "add", "exclusive", label="auto G=%d N=%d" % (G, N))
    # round 2: the cascade region above 2^16 (profiles/r02_cascade_boundary.jsonl); large
    # shapes, so the choice only (both families' parity is covered above and in the fuzz)
    for (G, N), algo in {(1024, 131072): "cascade_cta", (2048, 196612): "cascade_cta",
                         (2500, 1 << 18): "cascade_cta", (2048, 1 << 18): "lookback",
                         (1536, 196612): "lookback", (2200, 1 << 19): "lookback",
                         (100, 65536): "lookback", (100, 65540): "three_stage", (250, 131072): "lookback",
                         # profiles/r02_mid_batch_dispatch.jsonl
                         (200, 65536): "lookback", (500, 49152): "lookback", (800, 65536): "cascade_cta",
                         (200, 65532): "three_stage", (100, 32772): "three_stage", (70, 20484): "three_stage",
                         (100, 32768): "three_stage", (140, 10244): "cascade_cta", (148, 28676): "cascade_cta",
                         (132, 28676): "three_stage"}.items():
        xd = torch.empty((G, N), dtype=torch.int32, device="cuda")
        assert sb.plan(xd)[0] == algo, (G, N, sb.plan(xd))
        del xd


def test_autotune_table():
    # scan_autotune (the automated K search of PAPER.md:183): the measured winner becomes
    # the AUTO choice for that exact shape, results stay exact, clear() restores the rules
    sb.autotune_clear()
    for G, N in [(1, 20000), (3, 100003), (512, 1000)]:
        x = inputs.generate("i32", G * N, seed=G + N).reshape(G, N)
        xd = to_device(x)
        before = sb.plan(xd)
        before_max = sb.plan(xd, op="max", kind="exclusive")
        algo, param, us = sb.autotune(xd, "add", "inclusive")
        assert algo in sb.ALGOS and algo != "auto" and us > 0.0
        assert sb.plan(xd) == (algo, param)
        # the tuned choice applies to (op, dtype, kind) it was measured on only
        assert sb.plan(xd, op="max", kind="exclusive") == before_max
        assert sb.plan(xd.view(torch.float32)) == before
        for op, dt in COMBOS:
            xx = inputs.generate(DIST[dt], G * N, seed=3 * G + N).reshape(G, N)
            for kind in ("inclusive", "exclusive"):
                assert_parity(_run(xx, op, kind), xx, op, kind, label="tuned %s/%d %s %s" % (algo, param, op, dt))
        sb.autotune_clear()
        assert sb.plan(xd) == before
    with pytest.raises(sb.ScanError):
        sb.autotune(xd, "add", "inclusive", out=xd)          # in-place tuning is rejected


def test_autotune_with_caller_workspace():
    # a caller workspace is sized for the static AUTO choice (scan_workspace_bytes(AUTO)):
    # with one, AUTO must ignore the tuned table and still scan exactly
    sb.autotune_clear()
    G, N = 64, 65536                        # static rule: three-stage; with a workspace: look-back
    x = inputs.generate("i32", G * N, seed=77).reshape(G, N)
    xd = to_device(x)
    sb.autotune(xd, "add", "inclusive")
    nbytes = sb.workspace_bytes(N, G, "add", torch.int32, "auto")
    ws = torch.zeros(nbytes, dtype=torch.uint8, device="cuda")
    for kind in ("inclusive", "exclusive"):
        out = sb.scan(xd, "add", kind, workspace=ws)
        torch.cuda.synchronize()
        assert_parity(to_host(out, np.int32), x, "add", kind, label="tuned + caller workspace")
    sb.autotune_clear()


@pytest.mark.parametrize("algo,G,N", [("cascade_cta", 512, 8192), ("cascade_warp", 2000, 1000),
                                      ("packed_warp", 20000, 100), ("cluster", 3, 30000),
                                      ("three_stage", 1, 1 << 20), ("auto", 4096, 4096),
                                      ("lookback/3", 1, 1 << 22), ("lookback/3", 3, 1000003),
                                      ("fused", 1, 1 << 22), ("fused", 4, 1 << 16)])
def test_back_to_back_ordering(algo, G, N):
    # the single-kernel families and Stage 1 are launched as programmatic dependents of the
    # stream's previous kernel and wait before their first access: chains of dependent
    # calls and torch kernels on one stream, with no synchronisation, must stay ordered
    # (the L2-staged look-back, "lookback/3", is a programmatic dependent too)
    algo, param = (algo.split("/")[0], int(algo.split("/")[1])) if "/" in algo else (algo, -1)
    x = inputs.generate("small", G * N, seed=G + N).reshape(G, N)
    ref = x
    xd = to_device(x)
    for r in range(3):
        xd.add_(1)                                              # torch kernel writes the input
        y = sb.scan(xd, "add", "inclusive", algo=algo, param=param)     # reads it right behind
        sb.scan(y, "max", "inclusive", out=y, algo=algo, param=param)   # in place, right behind
        xd = sb.scan(y, "add", "exclusive", algo=algo, param=param)     # next round's input
        ref = (ref.astype(np.int64) + 1).astype(np.int32)        # wraps like torch int32 add_
        ref = oracle.scan(oracle.scan(ref, "add", "inclusive"), "max", "inclusive")
        ref = oracle.scan(ref, "add", "exclusive")
    torch.cuda.synchronize()
    got = to_host(xd, np.int32)
    assert np.array_equal(got, ref), algo


@pytest.mark.parametrize("op,dt", COMBOS)
def test_fused_family(op, dt):
    # SCAN_ALGO_FUSED: the three stages in one cooperative launch, one 8192-element tile per
    # CTA held in registers across one grid barrier.  One problem of any N (ragged last
    # tile), or G problems with N a multiple of the tile; unaligned pointers take the
    # scalar path; shapes beyond the co-resident capacity or with ragged multi-problem
    # layouts are rejected (SCAN_ERR_UNSUPPORTED), never mis-scanned.
    shapes = [(1, 1), (1, 8191), (1, 8193), (1, 1000003), (1, 4 * 1024 * 1024 + 5), (3, 8192), (5, 8192 * 9),
              (64, 65536)]
    for G, N in shapes:
        x = inputs.generate(DIST[dt], G * N, seed=G * 31 + N % 977).reshape(G, N)
        for kind in ("inclusive", "exclusive"):
            got = _run(x, op, kind, "fused")
            assert_parity(got, x, op, kind, label="fused %s %s %s G=%d N=%d" % (op, dt, kind, G, N))
    # unaligned base pointers
    x = inputs.generate(DIST[dt], 300001 + 1, seed=5)
    base = to_device(x)
    xin = base[1:]
    out = torch.empty(300001 + 4, dtype=base.dtype, device="cuda")[3:300004]
    sb.scan(xin, op, "inclusive", out=out, algo="fused")
    torch.cuda.synchronize()
    assert_parity(to_host(out, NP[dt]), x[1:], op, "inclusive", label="fused unaligned")
    # ineligible: ragged N with G > 1, and more tiles than CTAs fit at once
    with pytest.raises(sb.ScanError):
        sb.scan(torch.zeros((3, 10000), dtype=TORCH[dt], device="cuda"), op, algo="fused")
    with pytest.raises(sb.ScanError):
        sb.scan(torch.zeros(1 << 26, dtype=TORCH[dt], device="cuda"), op, algo="fused")
