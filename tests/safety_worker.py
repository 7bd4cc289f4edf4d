"""Worker of tests/test_gpu_safety.py::test_concurrent_first_use_and_streams (run as a
script in a fresh process, so every kernel's first-use setup -- the per-device shared
memory opt-in and occupancy cache of scan_launch.cu -- happens under contention).

T host threads, each with its own CUDA stream, issue look-back (persistent cooperative
grids that each want every SM), fused (a cooperative grid with a grid barrier), cluster,
three-stage and cascade scans at the same time.
Two persistent grids on two streams must never deadlock by splitting the SMs between
them; every result must be exact.  Prints "ok" or the first failure.
"""
import sys
import threading

import numpy as np
import torch

import inputs
import oracle
import paper_conf_ipps_dieguezadnm18_b200 as sb
from gpu_util import to_host

CASES = [("lookback", 3, 1, 1 << 24), ("lookback", 0, 1, 1 << 23), ("lookback", 1, 3, 1000003),
         ("lookback", 2, 5000, 100), ("cluster", -1, 3, 30000), ("three_stage", 0, 2, 1 << 20),
         ("cascade_cta", -1, 512, 8192), ("lookback", 3, 2, 1 << 23), ("fused", -1, 1, 3 << 20)]


def worker(k, errors, iters):
    try:
        s = torch.cuda.Stream()
        algo, param, G, N = CASES[k % len(CASES)]
        x = inputs.generate("i32", G * N, seed=100 + k).reshape(G, N)
        ref = oracle.scan(x, "add", "inclusive")
        with torch.cuda.stream(s):
            xd = torch.from_numpy(x).cuda(non_blocking=False)
            outs = [torch.empty_like(xd) for _ in range(iters)]
            for i in range(iters):
                sb.scan(xd, "add", "inclusive", out=outs[i], algo=algo, param=param, stream=s)
        s.synchronize()
        for i in range(iters):
            if not np.array_equal(to_host(outs[i], np.int32), ref):
                errors.append("thread %d %s/%d iter %d mismatch" % (k, algo, param, i))
                return
    except Exception as e:                       # noqa: BLE001 -- reported to the parent
        errors.append("thread %d: %r" % (k, e))


def main():
    threads = int(sys.argv[1]) if len(sys.argv) > 1 else 8
    iters = int(sys.argv[2]) if len(sys.argv) > 2 else 6
    torch.cuda.set_device(0)
    errors = []
    ts = [threading.Thread(target=worker, args=(k, errors, iters)) for k in range(threads)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    torch.cuda.synchronize()
    print("ok" if not errors else errors[0], flush=True)


if __name__ == "__main__":
    main()
