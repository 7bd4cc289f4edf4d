#!/usr/bin/env python
"""Benchmark of the batched scan hot path on B200 (one JSON line on rank 0).

Metric (BASELINE.json): Gelem/s (and % of the HBM roofline) of int32/f32 scans at 1/2/4/8
GPUs.  Workload at N=1 = configs[1]: G = 4096 problems of N = 2^14 elements; one STEP is
the four scans that config names -- add-scan of int32 and of f32, inclusive and exclusive
-- each over the whole 2^26-element batch (256 MiB in + 256 MiB out per scan, larger
than the 126 MB L2, so no flush is needed between steps).  Under torchrun (--gpus N > 1)
every rank scans its own G = 4096 problems (problems mode, Case 1 of PAPER.md:191-193, no
collective on the data path): weak scaling, value = elements of all ranks / max-over-ranks
time.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--no-extras] [--sweep]

`--impl reference` times the CPU oracle (the only reference this paper-only run has) on
host cores, on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

G_C2, N_C2 = 4096, 1 << 14
SEED = 0x5CA2018
METRIC = "Gelem/s and % of HBM roofline, int32/f32 scan at 1/2/4/8 B200"
VARIANTS = [("i32", "add", "inclusive"), ("i32", "add", "exclusive"),
            ("f32", "add", "inclusive"), ("f32", "add", "exclusive")]
DIST = {"i32": "i32", "f32": "f32u"}
TDT = {"i32": torch.int32, "f32": torch.float32}
NPDT = {"i32": np.int32, "f32": np.float32}


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured", d
    return 6650.0, "fallback (B200_PROFILING.md)", {}


# ---------------------------------------------------------------- multi-rank plumbing
# SCANB200_BENCH_BACKEND=gloo + SCANB200_BENCH_ONE_GPU=1 run every rank on cuda:0 with a gloo
# process group: a dry run of the multi-rank control flow (barriers, max over ranks, the
# peer-memory exchange between processes) on a one-GPU box; NCCL refuses two ranks on one GPU.
DIST_BACKEND = os.environ.get("SCANB200_BENCH_BACKEND", "nccl")
ONE_GPU = os.environ.get("SCANB200_BENCH_ONE_GPU") == "1"


def max_over_ranks(v: float, world: int) -> float:
    if world == 1:
        return v
    dev = "cuda" if DIST_BACKEND == "nccl" else "cpu"
    t = torch.tensor([v], dtype=torch.float64, device=dev)
    torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
    return float(t.item())


def all_gather_totals(t: torch.Tensor, world: int) -> torch.Tensor:
    """[W, G] totals of all ranks (the torch-backend exchange of the phase breakdown)."""
    from paper_conf_ipps_dieguezadnm18_b200 import multi
    if world == 1:
        return t.view(1, -1)
    if DIST_BACKEND == "nccl":
        return multi.exchange_totals(t)
    parts = [torch.empty_like(t, device="cpu") for _ in range(world)]
    torch.distributed.all_gather(parts, t.cpu())
    return torch.stack(parts).to(t.device)


# ---------------------------------------------------------------- clocks during the timed region
class ClockSampler:
    def __init__(self, dev_index: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        self._t = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        nv = self.nv
        names = {
            getattr(nv, "nvmlClocksEventReasonHwSlowdown", 0x8): "hw_slowdown",
            getattr(nv, "nvmlClocksEventReasonHwThermalSlowdown", 0x40): "hw_thermal_slowdown",
            getattr(nv, "nvmlClocksEventReasonSwThermalSlowdown", 0x20): "sw_thermal_slowdown",
            getattr(nv, "nvmlClocksEventReasonSwPowerCap", 0x4): "sw_power_cap",
        }
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in names.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.002)

    def __enter__(self):
        if self.nv is not None:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                "samples": len(self.samples)}


# ---------------------------------------------------------------- the device workload
def make_inputs(rank: int, device):
    import inputs
    xs = {}
    for dt in ("i32", "f32"):
        t = torch.empty(G_C2 * N_C2, dtype=torch.int32, device=device)
        inputs.fill_device(t, DIST[dt], SEED + 2, offset=rank * G_C2 * N_C2)
        xs[dt] = t.view(TDT[dt]).view(G_C2, N_C2)
    return xs


def step(sb, xs, outs, events=None):
    for i, (dt, op, kind) in enumerate(VARIANTS):
        if events is not None:
            events[i][0].record()
        sb.scan(xs[dt], op, kind, out=outs[i])
        if events is not None:
            events[i][1].record()


def timed_steps(sb, xs, outs, K, per_launch=False):
    """K steps between two events on the launching stream; optionally per-launch events."""
    ev = None
    if per_launch:
        ev = [[(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
               for _ in VARIANTS] for _ in range(K)]
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    s0.record()
    for k in range(K):
        step(sb, xs, outs, ev[k] if ev else None)
    s1.record()
    torch.cuda.synchronize()
    total_ms = s0.elapsed_time(s1)
    launch_ms = None
    if ev:
        launch_ms = [statistics.mean(ev[k][i][0].elapsed_time(ev[k][i][1]) for k in range(K))
                     for i in range(len(VARIANTS))]
    return total_ms, launch_ms


def kernel_times(sb, xs, outs, reps):
    res = []
    for i, (dt, op, kind) in enumerate(VARIANTS):
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        s0.record()
        for _ in range(reps):
            sb.scan(xs[dt], op, kind, out=outs[i])
        s1.record()
        torch.cuda.synchronize()
        res.append(s0.elapsed_time(s1) / reps)
    return res


def e2e(sb, world=1, K=3):
    """The same step through the public host-buffer API: pinned host in -> scan -> host out.
    Under torchrun every rank runs it at once on its own GPU (its own PCIe link); the time
    is the max over ranks and the value counts the elements of all ranks."""
    import inputs
    hin, hout = {}, []
    for dt in ("i32", "f32"):
        a = torch.empty(G_C2 * N_C2, dtype=torch.int32, pin_memory=True).numpy().view(NPDT[dt])
        a[:] = inputs.generate(DIST[dt], G_C2 * N_C2, SEED + 2)
        hin[dt] = a.reshape(G_C2, N_C2)
    for _ in VARIANTS:
        hout.append(torch.empty(G_C2 * N_C2, dtype=torch.int32, pin_memory=True).numpy()
                    .view(np.int32).reshape(G_C2, N_C2))

    def one():
        for i, (dt, op, kind) in enumerate(VARIANTS):
            sb.scan_host(hin[dt], op, kind, out=hout[i].view(NPDT[dt]))
    one()
    if world > 1:
        torch.distributed.barrier()
    t0 = time.perf_counter()
    for _ in range(K):
        one()
    dt_s = (time.perf_counter() - t0) / K
    dt_s = max_over_ranks(dt_s, world)
    elems = len(VARIANTS) * G_C2 * N_C2
    res = {"value": world * elems / dt_s / 1e9, "unit": "Gelem/s", "ms_per_step": dt_s * 1e3, "steps": K,
           "h2d_bytes_per_step": elems * 4, "d2h_bytes_per_step": elems * 4,
           "api": "scan_batch_host (pinned host buffers, library-pipelined H2D/scan/D2H)",
           "timing": "host wall clock around the synchronous calls, max over ranks"}
    res["pcie_ceiling"] = pcie_ceiling(elems * 4)
    res["frac_of_pcie_ceiling"] = (elems / dt_s / 1e9) / res["pcie_ceiling"]["Gelem/s_ceiling"]
    return res


def pcie_ceiling(nbytes: int, reps: int = 3):
    """Context for e2e: plain torch pinned-memory copies of the step's bytes, H2D and D2H
    at the same time on two streams (what any host-buffer scan must move)."""
    h_in = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    h_out = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d_in = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    d_out = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

    def both():
        with torch.cuda.stream(s1):
            d_in.copy_(h_in, non_blocking=True)
        with torch.cuda.stream(s2):
            h_out.copy_(d_out, non_blocking=True)
        torch.cuda.synchronize()
    both()
    t0 = time.perf_counter()
    for _ in range(reps):
        both()
    dt_s = (time.perf_counter() - t0) / reps
    gbs = nbytes / dt_s / 1e9
    del d_in, d_out
    torch.cuda.empty_cache()
    return {"GB/s_each_way": gbs, "Gelem/s_ceiling": gbs / 4,
            "how": "torch pinned H2D + D2H copies of %d bytes each, concurrently on two streams" % nbytes}


def c4_problems(sb, dev, world, rank, reps=5):
    """configs[3]: G = 2^16 problems of N = 2^16 int32 sharded by problem (Case 1,
    PAPER.md:191-193): rank r scans problems [floor(rG/W), floor((r+1)G/W)), no
    collective.  Strong scaling (the total is fixed); at W = 1 the whole 16 GiB batch."""
    import inputs
    from paper_conf_ipps_dieguezadnm18_b200 import multi
    G, N = 1 << 16, 1 << 16
    g0, g1 = multi.partition(G, world, rank)
    x = torch.empty((g1 - g0) * N, dtype=torch.int32, device=dev)
    inputs.fill_device(x, "i32", SEED + 4, offset=g0 * N)
    x = x.view(g1 - g0, N)
    y = torch.empty_like(x)
    for _ in range(2):
        multi.scan_multi(x, "add", "inclusive", mode="problems", out=y)
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s0.record()
    for _ in range(reps):
        multi.scan_multi(x, "add", "inclusive", mode="problems", out=y)
    s1.record()
    torch.cuda.synchronize()
    ms = max_over_ranks(s0.elapsed_time(s1) / reps, world)
    hbm, _, _ = _peaks()
    per_gpu_gbs = 8.0 * G * N / world / (ms * 1e-3) / 1e9
    kern = "%s %s" % sb.plan(x, y)
    del x, y
    torch.cuda.empty_cache()
    return {"G": G, "N": N, "problems_per_gpu": G // world, "ms": ms, "Gelem/s": G * N / ms / 1e6,
            "per_gpu_GB/s": per_gpu_gbs, "per_gpu_frac_measured_hbm": per_gpu_gbs / hbm,
            "scaling": "strong (fixed 2^32-element batch)", "kernel": kern}


# ---------------------------------------------------------------- CPU oracle (reference arm / baseline)
def cpu_oracle_rate(budget_s: float = 12.0):
    """The oracle as it stands (one thread, sequential C loop) on the same workload: it
    scans whole 2^26-element variants of the c2 batch until the time budget is used."""
    import inputs
    import oracle
    xs = {dt: inputs.generate(DIST[dt], G_C2 * N_C2, SEED + 2).reshape(G_C2, N_C2) for dt in ("i32", "f32")}
    oracle.scan(xs["i32"][:4], "add")            # load / build
    done, t_scan, steps = 0, 0.0, 0
    while t_scan < budget_s or steps < 1:
        for dt, op, kind in VARIANTS:
            t0 = time.perf_counter()
            oracle.scan(xs[dt], op, kind)
            t_scan += time.perf_counter() - t0
            done += G_C2 * N_C2
        steps += 1
    return {"value": done / t_scan / 1e9, "unit": "Gelem/s", "cores": 1, "kind": "oracle",
            "sample": "%d full steps of the c2 workload (4 x 4096 x 2^14 elements each), "
                      "single-threaded C oracle, %.1f s of scan time" % (steps, t_scan),
            "host_cpu": _cpu_name(), "host_cores_available": len(os.sched_getaffinity(0)),
            "ms_per_step": t_scan / steps * 1e3}


def cpu_oracle_steps(steps: int, warmup: int, g_sample: int = 256):
    """Reference arm: the oracle as it stands, `warmup` untimed + `steps` timed steps; each
    step scans a bounded sample of the c2 batch (g_sample of its 4096 problems, all four
    variants), so 200 steps stay within a few minutes on the host."""
    import inputs
    import oracle
    xs = {dt: inputs.generate(DIST[dt], g_sample * N_C2, SEED + 2).reshape(g_sample, N_C2)
          for dt in ("i32", "f32")}

    def one():
        for dt, op, kind in VARIANTS:
            oracle.scan(xs[dt], op, kind)
    for _ in range(warmup):
        one()
    t0 = time.perf_counter()
    for _ in range(steps):
        one()
    t = time.perf_counter() - t0
    elems = steps * len(VARIANTS) * g_sample * N_C2
    return {"value": elems / t / 1e9, "unit": "Gelem/s", "cores": 1, "kind": "oracle",
            "sample": "%d problems of the c2 batch (of 4096) x 4 variants per step, %d timed steps, "
                      "single-threaded C oracle" % (g_sample, steps),
            "host_cpu": _cpu_name(), "host_cores_available": len(os.sched_getaffinity(0)),
            "ms_per_step": t / steps * 1e3}


def _cpu_name():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


# ---------------------------------------------------------------- extra configs (context)
def extras(sb, dev):
    import inputs
    out = {}
    # c1: N = 2^20, G = 1, inclusive int32 add: latency-bound, L2 resident
    x = torch.empty(1 << 20, dtype=torch.int32, device=dev)
    inputs.fill_device(x, "i32", SEED + 1)
    y = torch.empty_like(x)
    for _ in range(10):
        sb.scan(x, "add", out=y)
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    s0.record()
    for _ in range(200):
        sb.scan(x, "add", out=y)
    s1.record()
    torch.cuda.synchronize()
    us = s0.elapsed_time(s1) / 200 * 1e3
    gs = torch.cuda.Stream(dev)
    dev_us = device_time(lambda: sb.scan(x, "add", out=y, stream=gs), gs, 50) * 1e3
    out["c1_i32_incl_N2^20"] = {"us_per_scan_device": dev_us, "Gelem/s_device": (1 << 20) / dev_us / 1e3,
                                "us_per_scan_host_launch": us,
                                "note": "L2-resident (8 MiB); device = 50 launches replayed from a CUDA graph; "
                                        "host_launch = back-to-back Python calls (host-bound)",
                                "kernel": "%s %s" % sb.plan(x, y)}
    del x, y
    # c3: N = 2^30 f32 inclusive add, single problem (look-back)
    N = 1 << 30
    x = torch.empty(N, dtype=torch.int32, device=dev)
    inputs.fill_device(x, "f32u", SEED + 3)
    x = x.view(torch.float32)
    y = torch.empty_like(x)
    for _ in range(3):
        sb.scan(x, "add", out=y)
    torch.cuda.synchronize()
    s0.record()
    for _ in range(10):
        sb.scan(x, "add", out=y)
    s1.record()
    torch.cuda.synchronize()
    ms = s0.elapsed_time(s1) / 10
    hbm, _, _ = _peaks()
    gbs = 8.0 * N / (ms * 1e-3) / 1e9
    out["c3_f32_incl_N2^30"] = {"ms": ms, "Gelem/s": N / ms / 1e6, "GB/s": gbs,
                                "frac_measured_hbm": gbs / hbm, "frac_8TBs": gbs / 8000.0}
    del x, y
    torch.cuda.empty_cache()
    return out


def elements_mode(sb, dev, world, rank, n_local=1 << int(os.environ.get("SCANB200_BENCH_ELEMS_LOG2", "33")),
                  reps=10):
    """configs[4]: one int32 add-scan sharded by elements (Multi-GPU Problem Scattering,
    PAPER.md:195-205): each rank owns a contiguous 2^33-element portion (32 GiB in + 32 GiB
    out) of ONE problem -- at W = 8 the problem is configs[4]'s N = 2^36.  Stage 1+2 ->
    exchange -> Stage 3.  Weak-scaled (N = W x 2^33).  At W = 1 the same two-pass pipeline
    runs with no peer (its 1-GPU reference rate)."""
    import inputs
    from paper_conf_ipps_dieguezadnm18_b200 import multi
    x = torch.empty(n_local, dtype=torch.int32, device=dev)
    inputs.fill_device(x, "i32", SEED + 5, offset=rank * n_local)
    y = torch.empty_like(x)
    # the fused exchange (Stage 2 pushes the totals into later ranks' HBM, Stage 3 waits on
    # the device; no collective call) is the product path; NCCL all-gather beside it
    comms = {"peer": multi.PeerComm(1) if world > 1 else multi.PeerComm.loopback(1, 1)[0]}
    if world > 1 and DIST_BACKEND == "nccl":
        comms["nccl"] = multi.NativeComm()

    def run(name):
        multi.scan_multi(x, "add", "inclusive", mode="elements", out=y,
                         backend="peer" if name == "peer" else "native", comm=comms[name])
    times = {}
    for name in comms:
        for _ in range(3):
            run(name)
        torch.cuda.synchronize()
        if world > 1:
            torch.distributed.barrier()
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s0.record()
        for _ in range(reps):
            run(name)
        s1.record()
        torch.cuda.synchronize()
        times[name] = max_over_ranks(s0.elapsed_time(s1) / reps, world)
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    for c in comms.values():
        c.close()
    ms = times["peer"]
    # per-phase breakdown (the paper's Fig. 14): Stage 1+2 / exchange /
    # Stage 3, events between the three steps of the torch-backend path
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    ph = [0.0, 0.0, 0.0]
    t = sb.shard_totals(x, "add")                 # warm-up (workspace growth), totals reused
    torch.cuda.synchronize()
    for _ in range(reps):
        ev[0].record()
        sb.shard_totals(x, "add", totals=t)
        ev[1].record()
        allt = all_gather_totals(t, world)
        ev[2].record()
        sb.shard_scan(x, allt, rank, world, "add", "inclusive", out=y)
        ev[3].record()
        torch.cuda.synchronize()
        for k in range(3):
            ph[k] += ev[k].elapsed_time(ev[k + 1]) / reps
    hbm, _, _ = _peaks()
    per_gpu_gbs = 12.0 * n_local / (ms * 1e-3) / 1e9          # reduce pass (4 B) + scan pass (8 B)
    return {"N_total": world * n_local, "N_per_gpu": n_local, "ms": ms,
            "Gelem/s": world * n_local / ms / 1e6, "per_gpu_GB/s_at_12B_per_elem": per_gpu_gbs,
            "per_gpu_frac_measured_hbm": per_gpu_gbs / hbm,
            "exchange": ("fused peer stores in the Stage 2/3 kernels (scan_comm_create_peer)" if world > 1
                         else "none (W=1; the fused-exchange kernels run with no peers)"),
            "ms_by_exchange": times,
            "phases_ms_rank%d" % rank: {"stage1+2_reduce": ph[0], "exchange": ph[1], "stage3_scan": ph[2]}}


def sweep(sb, dev):
    """On-box parameter search (the automated form of the paper's K search)."""
    import inputs
    rows = []
    shapes = [("i32", 1, 1 << 20), ("i32", 1, 1 << 24), ("i32", 1, 1 << 28), ("f32", 1, 1 << 30),
              ("i32", 4096, 1 << 14), ("f32", 4096, 1 << 14), ("i32", 1 << 16, 1 << 10),
              ("i32", 1 << 14, 1 << 12), ("i32", 256, 1 << 20), ("i32", 16, 1 << 24), ("i32", 1 << 18, 1 << 8),
              ("i32", 1 << 20, 1 << 6), ("i32", 1 << 13, 1 << 16)]
    cands = [("lookback", v) for v in sb._lib.LOOKBACK_VARIANTS] + [
        ("cascade_cta", -1), ("cascade_warp", -1), ("three_stage", 0)]
    s = torch.cuda.Stream(dev)
    for dt, G, N in shapes:
        x = torch.empty(G * N, dtype=torch.int32, device=dev)
        inputs.fill_device(x, DIST[dt], 1)
        x = x.view(TDT[dt]).view(G, N)
        y = torch.empty_like(x)
        for algo, param in cands:
            if algo == "cascade_cta" and G < 148:
                continue
            if algo == "cascade_warp" and (G < 1024 or N > (1 << 16)):
                continue
            reps = 20 if G * N < (1 << 26) else 5
            ms = device_time(lambda: sb.scan(x, "add", out=y, algo=algo, param=param, stream=s), s, reps)
            rows.append({"dtype": dt, "G": G, "N": N, "algo": algo, "param": param, "ms": ms,
                         "GB/s": 8.0 * G * N / ms / 1e6})
            print(json.dumps(rows[-1]), file=sys.stderr, flush=True)
        del x, y
        torch.cuda.empty_cache()
    return rows


def device_time(fn, s, reps):
    """Device time per call: warm up on stream s, capture `reps` calls into a CUDA graph,
    replay it between two events (removes the Python/launch overhead from small cases)."""
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(reps):
            fn()
    with torch.cuda.stream(s):
        g.replay()
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s0.record(s)
        g.replay()
        s1.record(s)
    torch.cuda.synchronize()
    return s0.elapsed_time(s1) / reps


# ---------------------------------------------------------------- main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-extras", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--sweep", action="store_true")
    ap.add_argument("--no-cpu", action="store_true", help="skip the CPU oracle baseline (profiling runs)")
    args = ap.parse_args()

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    hbm, hbm_src, _ = _peaks()
    config = {"workload": "configs[1]: batch scan G=4096 x N=2^14 per GPU, int32 and f32 add, "
                          "inclusive and exclusive (4 scans per step)",
              "G_per_gpu": G_C2, "N": N_C2, "layout": "row-major, stride N",
              "l2": "inputs larger than L2 (256 MiB in + 256 MiB out per scan), no flush",
              "parallelism": "problems sharded by rank (Case 1)" if world > 1 else "single GPU"}

    if args.impl == "reference":
        if rank != 0:
            return
        r = cpu_oracle_steps(args.steps, args.warmup)
        print(json.dumps({"impl": "reference", "metric": METRIC, "value": r["value"], "unit": "Gelem/s",
                          "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
                          "ms_per_step": r["ms_per_step"], "higher_is_better": True, "scaling": "weak",
                          "vs_baseline": None, "dtype": "i32+f32", "data": "synthetic (splitmix64)",
                          "config": config, "cpu_baseline": r,
                          "e2e": {"value": r["value"], "unit": "Gelem/s", "h2d_bytes_per_step": 0,
                                  "d2h_bytes_per_step": 0}}), flush=True)
        return

    import paper_conf_ipps_dieguezadnm18_b200 as sb
    if ONE_GPU:
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        import torch.distributed as dist
        if DIST_BACKEND == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(DIST_BACKEND)
    if args.sweep:
        rows = sweep(sb, dev)
        if rank == 0:
            print(json.dumps({"sweep": rows}))
        return

    xs = make_inputs(rank, dev)
    outs = [torch.empty((G_C2, N_C2), dtype=TDT[dt], device=dev) for dt, _, _ in VARIANTS]
    for _ in range(max(args.warmup, 3)):
        step(sb, xs, outs)
    torch.cuda.synchronize()

    # timed region: barrier + synchronize on both sides, device events, max over ranks
    if world > 1:
        torch.distributed.barrier()
    with ClockSampler(local) as clk:
        total_ms, _ = timed_steps(sb, xs, outs, args.steps)
    if world > 1:
        torch.distributed.barrier()
        total_ms = max_over_ranks(total_ms, world)
    # average launch duration of the dominant kernel, live over the timed region: every
    # launch in it is the same kernel family on the same bytes (the plan is checked below),
    # so it is the timed region's device time / its launches.  Events between launches are
    # avoided on purpose: an event pair around each ~85 us launch adds ~2 us of gap (measured).
    # Per-variant averages (reps back-to-back launches of one call between two events on the
    # launching stream) are reported beside it.
    launch_ms = kernel_times(sb, xs, outs, max(20, args.steps // 4))
    plans = {sb.plan(xs[dt], outs[i]) for i, (dt, _, _) in enumerate(VARIANTS)}
    live_launch_ms = total_ms / (args.steps * len(VARIANTS))

    ms_step = total_ms / args.steps
    elems_step = len(VARIANTS) * G_C2 * N_C2 * world
    value = elems_step / (ms_step * 1e-3) / 1e9
    bytes_launch = 2 * 4 * G_C2 * N_C2
    dom = max(range(len(VARIANTS)), key=lambda i: launch_ms[i])
    if len(plans) == 1:
        achieved, dom_ms, timing = (bytes_launch / (live_launch_ms * 1e-3) / 1e9, live_launch_ms,
                                    "timed region device time / launches (all launches are this kernel)")
    else:
        achieved, dom_ms, timing = (bytes_launch / (launch_ms[dom] * 1e-3) / 1e9, launch_ms[dom],
                                    "back-to-back launches of the slowest variant between two events")
    algo, param = sb.plan(xs[VARIANTS[dom][0]], outs[dom])
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tpath):
        try:
            traffic = json.load(open(tpath)).get("bytes_per_launch")
        except Exception:
            traffic = None
    res = {
        "metric": METRIC, "value": value, "unit": "Gelem/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "i32+f32", "data": "synthetic (splitmix64 counter-based, device-generated)",
        "config": config,
        "hbm_frac_of_step": {"algorithmic_GB/s": elems_step / world * 8 / (ms_step * 1e-3) / 1e9,
                             "frac": elems_step / world * 8 / (ms_step * 1e-3) / 1e9 / hbm, "peak_src": hbm_src},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                     "frac": achieved / hbm, "traffic": traffic,
                     "kernel": "%s [algo=%s param=%d] on %s %s %s" % (
                         sb.KERNEL_NAMES[algo], algo, param, *VARIANTS[dom]),
                     "bytes_per_launch": bytes_launch, "ms_per_launch": dom_ms, "timing": timing,
                     "bytes_basis": "2 x 4 B x G x N (read input once, write output once)",
                     "peak_src": hbm_src + " copy bandwidth (MEASURED_PEAKS.json hbm_gbs)"},
        "per_launch_ms": {"%s_%s_%s" % v: m for v, m in zip(VARIANTS, launch_ms)},

        "gpu_launches": len(VARIANTS) * args.steps,
        "clocks": clk.summary(),
    }
    if not args.no_extras:
        el = elements_mode(sb, dev, world, rank)
        res["elements_mode_sharded_problem"] = el
        torch.cuda.empty_cache()
        res["c4_problems_mode"] = c4_problems(sb, dev, world, rank)
    if not args.no_e2e:
        res["e2e"] = e2e(sb, world)
    if rank == 0 and world == 1 and not args.no_cpu:
        res["cpu_baseline"] = cpu_oracle_rate()
    if rank == 0 and world == 1 and not args.no_extras:
        del xs, outs
        torch.cuda.empty_cache()
        res["extras"] = extras(sb, dev)
    if rank == 0:
        print(json.dumps(res), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
