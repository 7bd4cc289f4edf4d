"""Fused peer-memory exchange of the sharded path (scan_comm_create_peer): the Stage 2
kernel pushes the G portion totals into the later ranks' mailboxes with one-sided stores
and the Stage 3 kernel waits for them on the device (PAPER.md:195-205 [§4.1], the
paper's P2P writes of PAPER.md:53, 199 folded into the kernels).

The box has one GPU, so the ranks share it:
* loopback: W virtual ranks in this process (mailboxes are plain device memory), issued
  rank by rank on one stream -- the protocol's flags, acks, mailbox halves and epochs over
  many consecutive calls, uneven and empty portions, every op/dtype;
* two processes: two real ranks on cuda:0 in separate CUDA contexts, the mailboxes mapped
  with cudaIpcOpenMemHandle, the handle exchange over a gloo group; the kernels of the
  two ranks really wait on each other across contexts (the GPU time-slices them).
"""
import os
import random
import subprocess
import sys

import numpy as np
import pytest
import torch

import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
from gpu_util import COMBOS, DIST, NP, assert_parity, to_device, to_host
from paper_conf_ipps_dieguezadnm18_b200 import _lib, multi

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


def _run_loopback(comms, parts, op, kind):
    """One sharded call on every virtual rank, rank order, one stream."""
    outs = []
    for r, xl in enumerate(parts):
        outs.append(multi.scan_multi(xl, op, kind, mode="elements", backend="peer", comm=comms[r]))
    return outs


@pytest.mark.parametrize("W", [2, 3, 5, 8])
def test_peer_loopback_parity(W):
    rng = random.Random(W)
    max_G = 4
    comms = multi.PeerComm.loopback(W, max_G)
    try:
        calls = 0
        for op, dt in COMBOS:
            for G in (1, 3):
                lens = [rng.choice([0, 1, 37, 4096, 10007, 70001, 300000]) for _ in range(W)]
                if sum(lens) == 0:
                    lens[-1] = 5
                Ntot = sum(lens)
                x = inputs.generate(DIST[dt], G * Ntot, seed=W * 100 + G + calls).reshape(G, Ntot)
                starts = np.cumsum([0] + lens)
                parts = [to_device(np.ascontiguousarray(x[:, starts[r]:starts[r] + L])) for r, L in enumerate(lens)]
                for kind in ("inclusive", "exclusive"):
                    outs = _run_loopback(comms, parts, op, kind)
                    calls += 1
                    torch.cuda.synchronize()
                    got = np.concatenate([to_host(o, NP[dt]).reshape(G, -1) for o in outs], axis=1)
                    assert_parity(got, x, op, kind, label="peer W=%d %s %s %s lens=%s" % (W, op, dt, kind, lens))
        assert calls >= 20          # both mailbox halves reused many times (acks exercised)
    finally:
        torch.cuda.synchronize()
        for c in comms:
            c.close()


@pytest.mark.parametrize("W", [2, 4])
def test_short_portions_warp_path(W):
    # many problems with short per-rank portions (N_local <= 4096, G >= 1184) take the
    # warp-per-problem Stage 1 / Stage 3 (scan_api.cu run_three_stage); ranks with longer
    # or empty portions take the CTA path / the bare acknowledgement in the same call, so
    # the mixed paths must interoperate through the mailboxes.  Both exchanges: the fused
    # peer stores and the public two-step API with the totals stacked on the host side.
    rng = random.Random(17 + W)
    for op, dt in COMBOS:
        G = rng.choice([1184, 1500, 3000])
        lens = [rng.choice([0, 1, 37, 1000, 2048, 4096, 4097, 6000]) for _ in range(W)]
        if sum(lens) == 0:
            lens[0] = 100
        Ntot = sum(lens)
        x = inputs.generate(DIST[dt], G * Ntot, seed=W * 1000 + len(op) + Ntot).reshape(G, Ntot)
        starts = np.cumsum([0] + lens)
        parts = [to_device(np.ascontiguousarray(x[:, starts[r]:starts[r] + L])) for r, L in enumerate(lens)]
        comms = multi.PeerComm.loopback(W, G)
        try:
            for kind in ("inclusive", "exclusive"):
                outs = _run_loopback(comms, parts, op, kind)
                torch.cuda.synchronize()
                got = np.concatenate([to_host(o, NP[dt]).reshape(G, -1) for o in outs], axis=1)
                assert_parity(got, x, op, kind, label="warp-path peer W=%d %s %s %s G=%d lens=%s" % (
                    W, op, dt, kind, G, lens))
        finally:
            torch.cuda.synchronize()
            for c in comms:
                c.close()
        # the public steps: Stage 1+2 on every rank, the [W, G] totals stacked, Stage 3
        for kind in ("inclusive", "exclusive"):
            tots = [sb.shard_totals(xl, op) for xl in parts]
            allt = torch.stack(tots)
            outs = [sb.shard_scan(xl, allt, r, W, op, kind) for r, xl in enumerate(parts)]
            torch.cuda.synchronize()
            got = np.concatenate([to_host(o, NP[dt]).reshape(G, -1) for o in outs], axis=1)
            assert_parity(got, x, op, kind, label="warp-path steps W=%d %s %s %s G=%d lens=%s" % (
                W, op, dt, kind, G, lens))


def test_peer_loopback_many_epochs_graph_free():
    # 64 back-to-back calls with no host sync in between: the ack protocol alone keeps
    # a mailbox half from being overwritten before the later ranks read it
    W, G, L = 4, 2, 50000
    comms = multi.PeerComm.loopback(W, G)
    try:
        xs = [inputs.generate("i32", G * L * W, seed=s).reshape(G, L * W) for s in range(4)]
        parts = [[to_device(np.ascontiguousarray(x[:, r * L:(r + 1) * L])) for r in range(W)] for x in xs]
        results = []
        for it in range(64):
            outs = _run_loopback(comms, parts[it % 4], "add", "inclusive")
            results.append(outs)
        torch.cuda.synchronize()
        for it in (0, 1, 2, 3, 61, 62, 63):
            got = np.concatenate([to_host(o, np.int32).reshape(G, -1) for o in results[it]], axis=1)
            assert_parity(got, xs[it % 4], "add", "inclusive", label="epoch %d" % it)
    finally:
        torch.cuda.synchronize()
        for c in comms:
            c.close()


def test_peer_argument_checks():
    c = multi.PeerComm.loopback(1, 2)[0]
    try:
        x = torch.zeros(3, 10, dtype=torch.int32, device="cuda")
        with pytest.raises(sb.ScanError):          # G = 3 > max_G = 2
            multi.scan_multi(x, backend="peer", comm=c)
        y = multi.scan_multi(torch.ones(2, 10, dtype=torch.int32, device="cuda"), backend="peer", comm=c)
        torch.cuda.synchronize()
        assert y[1].tolist() == list(range(1, 11))
    finally:
        c.close()
    import ctypes
    h = ctypes.c_void_p(0)
    assert _lib.lib.scan_comm_create_peer(0, 9, 4, ctypes.byref(h)) == 2     # > 8 ranks: UNSUPPORTED
    assert _lib.lib.scan_comm_create_peer(2, 2, 4, ctypes.byref(h)) == 1     # rank out of range
    a = multi.PeerComm.loopback(2, 4)
    b = multi.PeerComm(8, rank=0, world=2, _open=False)
    try:
        # handles of communicators with different max_G must be rejected
        with pytest.raises(sb.ScanError):
            b.open([b.peer_handle(), a[1].peer_handle()])
    finally:
        for c in a + [b]:
            c.close()


def test_peer_two_processes_ipc(tmp_path):
    """Two real ranks (two processes, two CUDA contexts on cuda:0, IPC-mapped mailboxes)."""
    port = random.randint(20000, 40000)
    env = dict(os.environ, PYTHONPATH=os.pathsep.join([os.path.dirname(HERE), HERE]))
    procs = [subprocess.Popen([sys.executable, os.path.join(HERE, "peer_worker.py"), str(r), "2", str(port),
                               str(tmp_path)], env=env, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)
             for r in range(2)]
    logs = []
    try:
        for p in procs:
            out, _ = p.communicate(timeout=240)
            logs.append(out.decode(errors="replace"))
    finally:
        for p in procs:
            if p.poll() is None:
                p.kill()
    for r, p in enumerate(procs):
        assert p.returncode == 0, "rank %d failed:\n%s" % (r, logs[r][-3000:])
        assert open(os.path.join(tmp_path, "rank%d" % r)).read().startswith("ok"), logs[r][-2000:]


def test_peer_setup_failure_is_collective(tmp_path):
    """A rank that cannot map its peers makes EVERY rank raise PeerUnavailable (bench.py then
    runs the legs on the NCCL exchange) instead of leaving the others waiting on mailboxes."""
    port = random.randint(20000, 40000)
    env = dict(os.environ, PYTHONPATH=os.pathsep.join([os.path.dirname(HERE), HERE]))
    procs = [subprocess.Popen([sys.executable, os.path.join(HERE, "peer_worker.py"), str(r), "2", str(port),
                               str(tmp_path), "failopen"], env=env, stdout=subprocess.PIPE,
                              stderr=subprocess.STDOUT) for r in range(2)]
    logs = []
    try:
        for p in procs:
            out, _ = p.communicate(timeout=180)
            logs.append(out.decode(errors="replace"))
    finally:
        for p in procs:
            if p.poll() is None:
                p.kill()
    for r, p in enumerate(procs):
        assert p.returncode == 0, "rank %d failed:\n%s" % (r, logs[r][-3000:])
        assert open(os.path.join(tmp_path, "rank%d" % r)).read() == "ok-unavailable", logs[r][-2000:]


def test_c5_rank_portion_full_size():
    """configs[4] (N = 2^36 over 8 GPUs) gives every rank a 2^33-element int32 portion
    (32 GiB in + 32 GiB out).  Here the portion runs at full size as the LAST rank of a
    W = 2 loopback whose rank 0 holds a 3*2^20 prefix (non-trivial carry through the fused
    exchange), in the launch configuration bench.py times; every output element is checked
    against the streaming oracle of the concatenated problem."""
    from gpu_util import device_inputs
    import oracle
    L0, L1 = 3 << 20, 1 << 33
    seed = 0x5CA2018 + 5
    comms = multi.PeerComm.loopback(2, 1)
    try:
        x0 = device_inputs("i32", L0, seed)
        x1 = device_inputs("i32", L1, seed, offset=L0)        # the same counter stream, continued
        y0 = multi.scan_multi(x0, "add", "inclusive", mode="elements", backend="peer", comm=comms[0])
        y1 = multi.scan_multi(x1, "add", "inclusive", mode="elements", backend="peer", comm=comms[1])
        torch.cuda.synchronize()
        so = oracle.StreamAdd(np.int32, "inclusive")
        assert np.array_equal(to_host(y0, np.int32), so.feed(to_host(x0, np.int32)))
        del x0, y0
        step = 1 << 26
        for a in range(0, L1, step):
            ref = so.feed(to_host(x1[a:a + step], np.int32))
            got = to_host(y1[a:a + step], np.int32)
            assert np.array_equal(got, ref), "c5 rank portion chunk %d" % (a // step)
    finally:
        torch.cuda.synchronize()
        for c in comms:
            c.close()
