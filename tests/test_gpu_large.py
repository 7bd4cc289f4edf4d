"""Full-size single-GPU configurations beyond round 1's coverage, checked in full.

* One int32 / uint32 problem of N = 2^31 + 4099 elements (8 GiB in + 8 GiB out) through the
  AUTO path (the L2-staged look-back): tile and element indices beyond 2^31, a ragged last
  tile, 8-byte descriptors; every output element against the streaming oracle.
* configs[2]'s shape in int32 (G = 1, N = 2^30), inclusive and exclusive.
The north_star asks for N "from 2^10 to beyond one GPU's HBM" (the sharded path covers the
latter); PAPER.md:96 defines the problem for any N.
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ipps_dieguezadnm18_b200 as sb
from gpu_util import device_inputs, to_host

pytestmark = pytest.mark.gpu


def _check_streamed(xd, out, kind, dtype, label):
    so = oracle.StreamAdd(dtype, kind)
    n = xd.numel()
    step = 1 << 26
    for a in range(0, n, step):
        ref = so.feed(to_host(xd[a: a + step], dtype))
        got = to_host(out[a: a + step], dtype)
        if not np.array_equal(got, ref):
            i = int(np.argmax(got != ref))
            raise AssertionError("%s: chunk %d, first bad element %d: got %r ref %r" % (
                label, a // step, a + i, got[i], ref[i]))


@pytest.mark.parametrize("dist,kind", [("i32", "inclusive"), ("u32", "exclusive")])
def test_single_problem_beyond_2e31_elements(dist, kind):
    N = (1 << 31) + 4099
    dtype = np.int32 if dist == "i32" else np.uint32
    xd = device_inputs(dist, N, 0x5CA2018 + 9)
    assert sb.plan(xd) == ("lookback", 3)
    out = sb.scan(xd, "add", kind)
    torch.cuda.synchronize()
    _check_streamed(xd, out, kind, dtype, "N=2^31+4099 %s %s" % (dist, kind))
    del xd, out
    torch.cuda.empty_cache()


@pytest.mark.parametrize("kind", ["inclusive", "exclusive"])
def test_c3_shape_int32_full(kind):
    N = 1 << 30
    xd = device_inputs("i32", N, 0x5CA2018 + 3)
    out = sb.scan(xd, "add", kind)
    torch.cuda.synchronize()
    _check_streamed(xd, out, kind, np.int32, "int32 N=2^30 %s" % kind)
    del xd, out
    torch.cuda.empty_cache()


@pytest.mark.parametrize("G,N,op,dist,kind", [
    (5, 3000017, "add", "i32", "inclusive"), (5, 3000017, "add", "i32", "exclusive"),
    (5, 3000017, "add", "f32s", "inclusive"), (5, 3000017, "max", "i32", "exclusive"),
    (3, 7 * 8192 * 148 + 5, "add", "u32", "inclusive"), (2048, 1 << 17, "add", "i32", "inclusive"),
    (2048, 65540, "add", "i32", "exclusive"), (700, 200003, "add", "f32s", "inclusive"),
    (150, 200003, "max", "f32s", "exclusive"), (300, 100004, "max", "u32", "inclusive")])
def test_lookback_multiround_segmented(G, N, op, dist, kind):
    # the persistent L2-staged look-back over MANY rounds of the CTA round robin with problem
    # starts inside tiles (segmented tiles publish P at once; the lazy look-back's window and
    # the CTA-local previous prefix must both stop at problem boundaries); (2048, 2^17) is the
    # paper-sweep point n = 17, checked in full
    import inputs
    from gpu_util import assert_parity
    xd = device_inputs(dist, G * N, 0x5CA2018 + 11 + G).view(G, N)
    # forced: AUTO sends (2048, 2^17) to one CTA per problem since round 2 session 3
    out = sb.scan(xd, op, kind, algo="lookback", param=3)
    torch.cuda.synchronize()
    dt = inputs.DIST_DTYPE[dist]
    x = to_host(xd, dt).reshape(G, N)
    assert_parity(to_host(out, dt).reshape(G, N), x, op, kind, label="multiround G=%d N=%d" % (G, N))
    del xd, out
    torch.cuda.empty_cache()
