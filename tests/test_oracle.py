"""Pins for the CPU oracle (oracle/) against what the paper and mathematics fix.

Nothing here runs the CUDA path.  Each test pins the oracle to something other than
itself: the Fig. 1 worked example, the north_star closed form, exact
rational arithmetic, an independent pure-Python literal reading of the definition
(PAPER.md:29), numpy library routines (special cases), and algebraic invariants.
"""
import itertools
import math
import os
from fractions import Fraction

import numpy as np
import pytest

import inputs
import oracle
from oracle import ref

GOLD = os.path.join(os.path.dirname(__file__), "golden")
MASK = 0xFFFFFFFF


def _read_golden(name):
    rows = {}
    with open(os.path.join(GOLD, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            key, *vals = line.split()
            rows[key] = vals
    return rows


# ------------------------------------------------------------------ Fig. 1
def test_fig1_worked_example():
    g = _read_golden("fig1_lf_n8.txt")
    x = np.array([int(v) for v in g["input"]], np.int32)
    for kind in ("inclusive", "exclusive"):
        want = np.array([int(v) for v in g[kind]], np.int32)
        assert np.array_equal(oracle.scan(x, "add", kind), want)
        assert np.array_equal(oracle.scan(x.astype(np.uint32), "add", kind), want.astype(np.uint32))
        got = oracle.scan(x.astype(np.float32), "add", kind)
        assert np.array_equal(got, want.astype(np.float64))


# ------------------------------------------------------------------ closed form (north_star)
def test_closed_form_iota_i32_c1_size():
    N = 1 << 20
    x = inputs.generate("iota", N, 0, row_len=N)
    out = oracle.scan(x, "add")
    j = np.arange(N, dtype=np.int64)
    want = (((j + 1) * (j + 2) // 2) & MASK).astype(np.uint32).view(np.int32)
    assert np.array_equal(out, want)
    for line in open(os.path.join(GOLD, "closed_form_iota.txt")):
        if line.startswith("#") or not line.strip():
            continue
        jj, v = map(int, line.split())
        assert int(out[jj]) == v, (jj, int(out[jj]), v)


def test_closed_form_iota_u32_batch():
    N, G = 100003, 3
    x = inputs.generate("iota", N * G, 0, row_len=N).view(np.uint32).reshape(G, N)
    out = oracle.scan(x, "add")
    j = np.arange(N, dtype=np.int64)
    want = (((j + 1) * (j + 2) // 2) & MASK).astype(np.uint32)
    for g in range(G):
        assert np.array_equal(out[g], want)


def test_closed_form_iota_f32_exact_in_fp64():
    # fp64 prefix of 1..N is exact while (j+1)(j+2)/2 <= 2^53 (SURVEY §8(c) pins table).
    N = 1 << 20
    x = inputs.generate("iotaf", N, 0, row_len=N)
    out = oracle.scan(x, "add")
    j = np.arange(N, dtype=np.float64)
    assert np.array_equal(out, (j + 1) * (j + 2) / 2)
    ex = oracle.scan(x, "add", "exclusive")
    assert np.array_equal(ex, j * (j + 1) / 2)


def test_constant_input():
    N = 70000
    for c in (1, 7, -3, 2**31 - 1):
        x = np.full(N, c, np.int64).astype(np.uint32)
        out = oracle.scan(x, "add")
        i = np.arange(1, N + 1, dtype=np.int64)
        assert np.array_equal(out, ((i * (c & MASK)) & MASK).astype(np.uint32))


# ------------------------------------------------------------------ brute force, literal definition
@pytest.mark.parametrize("op", ["add", "max"])
@pytest.mark.parametrize("dt", ["i32", "u32", "f32"])
@pytest.mark.parametrize("kind", ["inclusive", "exclusive"])
def test_literal_definition_tiny(op, dt, kind):
    dist = {"i32": "i32", "u32": "u32", "f32": "f32s"}[dt]
    for N, G in [(0, 3), (1, 1), (2, 5), (3, 2), (8, 1), (31, 2), (33, 3), (70, 2)]:
        x = inputs.generate(dist, N * G, seed=N * 31 + G).reshape(G, N)
        got = oracle.scan(x, op, kind)
        for g in range(G):
            want = ref.scan_literal([v.item() for v in x[g]], op, dt, kind)
            for i in range(N):
                if dt == "f32" and op == "add":
                    exact = want[i]
                    n_terms = i + 1 if kind == "inclusive" else i
                    sabs = sum(abs(Fraction(float(v))) for v in x[g][:n_terms])
                    err = abs(Fraction(float(got[g, i])) - exact)
                    assert err <= Fraction(max(n_terms, 1)) * Fraction(2) ** -53 * sabs
                else:
                    assert got[g, i] == want[i], (N, G, g, i)


def test_itertools_accumulate_ints():
    for dt, dist in (("i32", "i32"), ("u32", "u32")):
        x = inputs.generate(dist, 257, 11)
        want = [v & MASK for v in itertools.accumulate(int(v) & MASK for v in x)]
        got = oracle.scan(x, "add").view(np.uint32)
        assert [int(v) for v in got] == want
        wmax = list(itertools.accumulate((int(v) for v in x), max))
        assert [int(v) for v in oracle.scan(x, "max")] == wmax


# ------------------------------------------------------------------ library special cases
@pytest.mark.parametrize("dist", ["i32", "u32", "small"])
def test_numpy_cumsum_mod32(dist):
    G, N = 7, 12345
    x = inputs.generate(dist, G * N, 5).reshape(G, N)
    want = (np.cumsum(x.astype(np.int64), axis=1) & MASK).astype(np.uint32).view(x.dtype)
    assert np.array_equal(oracle.scan(x, "add"), want)


@pytest.mark.parametrize("dist", ["i32", "u32", "f32u", "f32s"])
def test_numpy_maximum_accumulate(dist):
    G, N = 5, 9999
    x = inputs.generate(dist, G * N, 9).reshape(G, N)
    assert np.array_equal(oracle.scan(x, "max"), np.maximum.accumulate(x, axis=1))


def test_f32_add_against_math_fsum():
    # math.fsum is the correctly rounded (exact then rounded) sum: a library special case.
    x = inputs.generate("f32u", 4000, 3)
    out = oracle.scan(x, "add")
    xs = [float(v) for v in x]
    for i in (0, 1, 10, 999, 3999):
        exact = math.fsum(xs[: i + 1])
        assert abs(out[i] - exact) <= (i + 1) * 2.0**-53 * exact


# ------------------------------------------------------------------ invariants
@pytest.mark.parametrize("op", ["add", "max"])
@pytest.mark.parametrize("dist", ["i32", "u32", "f32u", "f32s"])
def test_exclusive_is_shifted_inclusive(op, dist):
    G, N = 4, 3001
    x = inputs.generate(dist, G * N, 21).reshape(G, N)
    inc = oracle.scan(x, op, "inclusive")
    exc = oracle.scan(x, op, "exclusive")
    ident = oracle.identity(op, x.dtype)
    assert np.all(exc[:, 0] == ident)
    assert np.array_equal(exc[:, 1:], inc[:, :-1])


def test_int_add_paper_identity_incl_minus_excl():
    # PAPER.md:124 [§3.1]: exclusive = inclusive - own value (valid for integer add, mod 2^32).
    x = inputs.generate("i32", 5000, 4)
    inc = oracle.scan(x, "add").view(np.uint32)
    exc = oracle.scan(x, "add", "exclusive").view(np.uint32)
    assert np.array_equal(inc - exc, x.view(np.uint32))


def test_add_linearity():
    a = inputs.generate("i32", 20000, 1).reshape(4, 5000)
    b = inputs.generate("i32", 20000, 2).reshape(4, 5000)
    s = (a.view(np.uint32) + b.view(np.uint32)).view(np.int32)
    lhs = oracle.scan(s, "add").view(np.uint32)
    rhs = oracle.scan(a, "add").view(np.uint32) + oracle.scan(b, "add").view(np.uint32)
    assert np.array_equal(lhs, rhs)


@pytest.mark.parametrize("dist", ["i32", "u32", "f32s"])
def test_max_invariants(dist):
    x = inputs.generate(dist, 3 * 4000, 8).reshape(3, 4000)
    inc = oracle.scan(x, "max")
    assert np.all(inc[:, 1:] >= inc[:, :-1])                  # monotone
    assert np.all(inc >= x)                                     # dominates input
    assert np.array_equal(oracle.scan(inc, "max"), inc)         # idempotent
    for g in range(3):                                          # each value is some x_k, k<=i
        for i in range(0, 4000, 97):
            assert inc[g, i] in x[g, : i + 1]


def test_batch_isolation():
    # G independent problems: batched == each row alone; nothing leaks across rows.
    G, N = 6, 777
    x = inputs.generate("i32", G * N, 13).reshape(G, N)
    x[1, :] = 2**31 - 1            # would overflow into row 2 if a carry leaked
    batched = oracle.scan(x, "add")
    for g in range(G):
        assert np.array_equal(batched[g], oracle.scan(x[g].copy(), "add"))


def test_totals_equal_last_inclusive():
    for dist in ("i32", "f32u"):
        x = inputs.generate(dist, 5 * 1000, 17).reshape(5, 1000)
        t = oracle.totals(x)
        inc = oracle.scan(x, "add")
        if dist == "i32":
            assert np.array_equal(t, inc[:, -1].view(np.uint32))
            assert [int(v) for v in t] == [int(r.astype(np.int64).sum()) & MASK for r in x]
        else:
            assert np.array_equal(t, inc[:, -1])


def test_f32_abs_prefix_and_sharded_concat():
    # sabs is the prefix of |x|; the sharded oracle is the scan of the rank-ordered
    # concatenation (PAPER.md:197 [§4.1]): scanning chunks with carried totals gives the same.
    x = inputs.generate("f32s", 9000, 23)
    out, sabs = oracle.scan(x, "add", with_abs=True)
    assert np.allclose(sabs, np.cumsum(np.abs(x.astype(np.float64))), rtol=1e-12, atol=0)
    cuts = [0, 1000, 1000, 4096, 9000]          # includes an empty shard
    carry = 0.0
    for a, b in zip(cuts[:-1], cuts[1:]):
        part = oracle.scan(x[a:b].copy(), "add") + carry if b > a else np.zeros(0)
        assert np.allclose(part, out[a:b], rtol=0, atol=1e-9)
        carry += float(oracle.totals(x[a:b].copy(), N=max(b - a, 1))[0]) if b > a else 0.0


def test_degenerate_shapes():
    assert oracle.scan(np.zeros((0, 5), np.int32), "add").shape == (0, 5)
    assert oracle.scan(np.zeros((3, 0), np.int32), "add").shape == (3, 0)
    x = inputs.generate("i32", 10, 1).reshape(10, 1)         # N = 1: inclusive = x, exclusive = identity
    assert np.array_equal(oracle.scan(x, "add"), x)
    assert np.all(oracle.scan(x, "max", "exclusive") == -(2**31))


@pytest.mark.parametrize("dist,kind", [("i32", "inclusive"), ("u32", "exclusive"), ("f32u", "inclusive"),
                                       ("f32s", "exclusive")])
def test_streaming_oracle_equals_one_shot(dist, kind):
    x = inputs.generate(dist, 50000, 31)
    s = oracle.StreamAdd(x.dtype, kind)
    parts = [s.feed(x[a:b]) for a, b in [(0, 1), (1, 4097), (4097, 4097), (4097, 50000)]]
    if x.dtype == np.float32:
        ref, sabs = oracle.scan(x, "add", kind, with_abs=True)
        assert np.array_equal(np.concatenate([p[0] for p in parts]), ref)
        assert np.array_equal(np.concatenate([p[1] for p in parts]), sabs)
    else:
        assert np.array_equal(np.concatenate(parts), oracle.scan(x, "add", kind))


# ------------------------------------------------------------------ the |x| prefix (tolerance basis)
# north_star: |err_i| <= 1e-5 * sum_{k<=i} |x_k| (inclusive); reading R3 takes
# k < i for exclusive, so exclusive element 0 has bound 0 and must be exact.  The bound
# itself comes from the oracle's `sabs`, so it is pinned here against an independent
# numpy cumsum of |x| in fp64 -- per problem (G >= 3, reset at every problem start), for
# both kinds, one-shot and streamed.  A sum over k <= i in the exclusive form, or a
# missing reset between problems, fails these.
def _abs_prefix_np(x2d):
    return np.cumsum(np.abs(x2d.astype(np.float64)), axis=1)


@pytest.mark.parametrize("dist", ["f32u", "f32s"])
def test_sabs_inclusive_per_problem(dist):
    G, N = 5, 1237
    x = inputs.generate(dist, G * N, 41).reshape(G, N)
    x[:, 0] = np.float32(0.75)                 # nonzero first element in every problem
    _, sabs = oracle.scan(x, "add", "inclusive", with_abs=True)
    ref_abs = _abs_prefix_np(x)
    assert np.allclose(sabs, ref_abs, rtol=1e-12, atol=0)
    # reset per problem: row g starts at |x[g,0]|, not at the previous row's total
    assert np.all(sabs[:, 0] == np.float64(0.75))
    assert np.all(np.diff(sabs, axis=1) >= 0)


@pytest.mark.parametrize("dist", ["f32u", "f32s"])
def test_sabs_exclusive_is_shifted_and_starts_at_zero(dist):
    G, N = 4, 999
    x = inputs.generate(dist, G * N, 43).reshape(G, N)
    x[:, 0] = np.float32(-2.5)
    _, sabs_e = oracle.scan(x, "add", "exclusive", with_abs=True)
    _, sabs_i = oracle.scan(x, "add", "inclusive", with_abs=True)
    assert np.all(sabs_e[:, 0] == 0.0)                       # empty range 0..-1 (reading R2/R3)
    assert np.array_equal(sabs_e[:, 1:], sabs_i[:, :-1])     # sum over k < i
    ref_abs = _abs_prefix_np(x)
    assert np.allclose(sabs_e[:, 1:], ref_abs[:, :-1], rtol=1e-12, atol=0)
    # the exclusive bound is strictly below the inclusive one by |x_i| (never k <= i)
    assert np.allclose(sabs_i - sabs_e, np.abs(x.astype(np.float64)), rtol=1e-9, atol=1e-12)


@pytest.mark.parametrize("kind", ["inclusive", "exclusive"])
def test_stream_sabs_against_numpy(kind):
    x = inputs.generate("f32s", 30011, 47)
    x[0] = np.float32(1.5)
    s = oracle.StreamAdd(np.float32, kind)
    ys, sa = zip(*[s.feed(x[a:b]) for a, b in [(0, 3), (3, 8195), (8195, 8195), (8195, 30011)]])
    sa = np.concatenate(sa)
    ys = np.concatenate(ys)
    ref_abs = np.cumsum(np.abs(x.astype(np.float64)))
    ref_val = np.cumsum(x.astype(np.float64))
    if kind == "exclusive":
        assert sa[0] == 0.0 and ys[0] == 0.0
        assert np.allclose(sa[1:], ref_abs[:-1], rtol=1e-12, atol=0)
        assert np.allclose(ys[1:], ref_val[:-1], rtol=0, atol=1e-9)
    else:
        assert sa[0] == 1.5
        assert np.allclose(sa, ref_abs, rtol=1e-12, atol=0)
        assert np.allclose(ys, ref_val, rtol=0, atol=1e-9)
