"""Ordering and forward-progress safety of the launch machinery on the B200.

* Cross-call programmatic dependent launch (PDL): every kernel of the library triggers its
  dependents early; a kernel may touch memory before its own griddepcontrol.wait only if
  its primary waited before triggering (scan_chunked.cu, chunk_reduce_kernel).  The fused
  two-launch three-stage path (Stage 3 loads its first tile before waiting) is issued right
  behind kernels that trigger at entry and write its input LATE.
* Persistent look-back grids use a static round-robin tile schedule, so CTA b waits on
  tiles of CTAs with higher index: the grid is launched cooperatively (co-resident or a
  loud launch error).  A spinning kernel holding half the SMs on another stream, and
  several persistent grids issued from several host threads / streams at once, must not
  deadlock and must stay exact.
"""
import os
import subprocess
import sys
import time

import numpy as np
import pytest
import torch

import inputs
import oracle
import paper_conf_ipps_dieguezadnm18_b200 as sb
from gpu_util import device_inputs, spin_lib, to_host

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


def _stream_ref_tail(x_host, tail, kind="inclusive"):
    """Oracle inclusive add-scan of x (int32) over all of it; returns its last `tail` values."""
    so = oracle.StreamAdd(np.int32, kind)
    n = x_host.shape[0]
    step = 1 << 26
    out = None
    for a in range(0, n, step):
        r = so.feed(x_host[a: a + step])
        if a + step >= n - tail:
            out = r if out is None else np.concatenate([out, r])
    return out[-tail:]


@pytest.mark.parametrize("writer", ["lookback/3", "cascade_cta"])
def test_fused_three_stage_behind_late_writer(writer):
    # a writer that triggers its dependents at entry (the L2 look-back,
    # the CTA cascade) writes y; its LAST tiles are written at the very end.  Right behind
    # it, with no synchronisation, the fused two-launch three-stage path (AUTO for G = 1,
    # N = 2^20) scans the tail of y in place.  Stage 3 must not read the tail before the
    # writer is complete.
    algo, param = (writer.split("/")[0], int(writer.split("/")[1])) if "/" in writer else (writer, -1)
    tail = 1 << 20
    if algo == "lookback":
        G, N = 1, 1 << 28
    else:
        G, N = 1 << 14, 1 << 14                       # 2^28 elements, one CTA per problem
    xd = device_inputs("small", G * N, 777).view(G, N)
    xh = to_host(xd, np.int32).reshape(G, N)
    if algo == "lookback":
        ref_tail = _stream_ref_tail(xh.reshape(-1), tail)
    else:
        ref_tail = oracle.scan(xh[-(tail // N):], "add", "inclusive").reshape(-1)
    ref_tail = oracle.scan(ref_tail, "add", "inclusive")
    y = torch.empty_like(xd)
    t = y.view(-1)[G * N - tail:]
    assert sb.plan(t) == ("three_stage", -1)
    for it in range(4):
        y.fill_(-7)                                    # stale contents a racing read would see
        sb.scan(xd, "add", "inclusive", out=y, algo=algo, param=param)
        sb.scan(t, "add", "inclusive", out=t)          # fused three-stage, right behind
        torch.cuda.synchronize()
        got = to_host(t, np.int32)
        assert np.array_equal(got, ref_tail), "iteration %d: %d wrong" % (it, int((got != ref_tail).sum()))


def test_lookback_with_half_the_sms_taken():
    # A foreign kernel holds ~half the SMs (one 200 KiB-smem CTA per SM) on another stream
    # until the host releases it.  The cooperative persistent look-back launched meanwhile
    # must complete (after the release) and be exact; also the f32 fp64-carry path.
    spin = spin_lib()
    flag = torch.zeros(1, dtype=torch.int32, pin_memory=True)
    side = torch.cuda.Stream()
    for dist, N in (("i32", 1 << 26), ("f32u", 1 << 27)):
        xd = device_inputs(dist, N, 4242)
        x = to_host(xd, np.float32 if dist.startswith("f32") else np.int32)
        assert sb.plan(xd)[0] == "lookback"
        flag[0] = 0
        torch.cuda.synchronize()
        rc = spin.spin_launch(flag.data_ptr(), 74, 200 * 1024, 20 * 10**9, side.cuda_stream)
        assert rc == 0
        time.sleep(0.05)
        y = sb.scan(xd, "add", "inclusive")
        done = torch.cuda.Event()
        done.record()
        time.sleep(0.3)
        flag[0] = 1                                    # release the foreign SMs
        done.synchronize()
        torch.cuda.synchronize()
        if dist == "i32":
            assert np.array_equal(to_host(y, np.int32), oracle.scan(x, "add", "inclusive"))
        else:
            ref, sabs = oracle.scan(x, "add", "inclusive", with_abs=True)
            assert np.all(np.abs(to_host(y, np.float32) - ref) <= 1e-5 * sabs)


def test_concurrent_first_use_and_streams():
    # fresh process: first use of every kernel from 8 host threads at once (per-device
    # opt-in / occupancy caches under contention), and persistent cooperative grids on 8
    # streams at once; a deadlock would hang, so the worker runs under a time limit
    env = dict(os.environ, PYTHONPATH=os.pathsep.join([os.path.dirname(HERE), HERE]))
    r = subprocess.run([sys.executable, os.path.join(HERE, "safety_worker.py"), "9", "6"], env=env,
                       capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-3000:]
    assert r.stdout.strip().splitlines()[-1] == "ok", r.stdout[-2000:]
