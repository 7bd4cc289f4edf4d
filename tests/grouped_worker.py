"""One rank of tests/test_gpu_grouped.py (run as a script): MP-PC grouping on the CUDA path.

PAPER.md:213-217 [§4.1.1, Fig. 8]: the W ranks form Y = W/V groups of V consecutive ranks;
group y solves problems [yG/Y, (y+1)G/Y) and, inside the group, rank v owns the contiguous
portion v of each of those problems (multi.grouped_plan).  Every rank runs elements mode
on its group's sub-communicator (multi.make_groups) through the product path --
backend "peer" (fused exchange in the kernels over CUDA-IPC-mapped mailboxes) and
backend "torch" (Stage 1+2 kernel -> all-gather of the G totals on the group -> Stage 3
kernel) -- and compares its slice with the oracle of the FULL batch, element by element.
All ranks share cuda:0 (one GPU on the box); the group plumbing is gloo.
"""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

import inputs
import oracle
from gpu_util import to_device, to_host
from paper_conf_ipps_dieguezadnm18_b200 import multi

CASES = [("add", "i32", "inclusive", 7, 300001), ("add", "f32s", "exclusive", 5, 123457),
         ("max", "u32", "inclusive", 4, 4099), ("add", "u32", "exclusive", 9, 1000003),
         ("max", "f32s", "exclusive", 6, 77), ("add", "i32", "inclusive", 3, 2)]


def main():
    rank, world, V, port, outdir = (int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]),
                                    sys.argv[5])
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    mine = multi.make_groups(V)
    msgs = []
    max_G = max(c[3] for c in CASES)
    comm = multi.PeerComm(max_G, group=mine)
    try:
        for it, (op, dname, kind, G, N) in enumerate(CASES):
            plan = multi.grouped_plan(G, N, world, V, rank)
            (g0, g1), (e0, e1) = plan["problems"], plan["elements"]
            x = inputs.generate(dname, G * N, seed=900 + it).reshape(G, N)
            xl = to_device(np.ascontiguousarray(x[g0:g1, e0:e1]))
            if dname.startswith("f32") and op == "add":
                ref, sabs = oracle.scan(x, op, kind, with_abs=True)
                ref, sabs = ref[g0:g1, e0:e1], sabs[g0:g1, e0:e1]
            else:
                ref = oracle.scan(x, op, kind)[g0:g1, e0:e1]
            for backend in ("peer", "torch"):
                if g1 == g0:
                    continue
                out = multi.scan_multi(xl, op, kind, mode="elements", group=mine, backend=backend,
                                       comm=comm if backend == "peer" else None)
                torch.cuda.synchronize()
                got = to_host(out, x.dtype).reshape(g1 - g0, e1 - e0)
                if dname.startswith("f32") and op == "add":
                    ok = bool(np.all(np.abs(got.astype(np.float64) - ref) <= 1e-5 * sabs))
                else:
                    ok = np.array_equal(got, ref)
                if not ok:
                    msgs.append("BAD it=%d %s %s %s %s group=%d member=%d" % (it, backend, op, dname, kind,
                                                                             plan["group"], plan["member"]))
    finally:
        torch.cuda.synchronize()
        dist.barrier()
        comm.close()
        with open(os.path.join(outdir, "rank%d" % rank), "w") as f:
            f.write(msgs[0] if msgs else "ok")
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
