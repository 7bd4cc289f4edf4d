"""One rank of tests/test_gpu_peer.py::test_peer_two_processes_ipc (run as a script).

Both ranks use cuda:0 (the box has one GPU); the mailboxes are exchanged as CUDA IPC
handles over a gloo process group and every sharded call then runs with no collective:
rank 1's Stage 3 waits on the device for the totals rank 0's Stage 2 stores into it.
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


def main():
    rank, world, port, outdir = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    G = 3
    if len(sys.argv) > 5 and sys.argv[5] == "failopen":
        # rank 1 cannot map its peers: EVERY rank must get PeerUnavailable (and no rank may
        # go on to wait on a mailbox nobody writes)
        if rank == 1:
            def broken_open(self, blobs):
                raise RuntimeError("simulated: no peer access")
            multi.PeerComm.open = broken_open
        try:
            multi.PeerComm(G, group=None)
            msg = "BAD: no error"
        except multi.PeerUnavailable as e:
            msg = "ok-unavailable" if "simulated" in str(e) and "[1]" in str(e) else "BAD: %s" % e
        dist.barrier()
        with open(os.path.join(outdir, "rank%d" % rank), "w") as f:
            f.write(msg)
        dist.destroy_process_group()
        return
    comm = multi.PeerComm(G, group=None)
    msg = "ok"
    try:
        for it, (op, dist_name, kind, N) in enumerate([("add", "i32", "inclusive", 300001),
                                                       ("add", "f32s", "exclusive", 123457),
                                                       ("max", "u32", "inclusive", 4096),
                                                       ("add", "i32", "exclusive", 2 * 1000003),
                                                       ("add", "u32", "inclusive", 7)] * 2):
            x = inputs.generate(dist_name, G * N, seed=31 + it).reshape(G, N)
            a, b = multi.partition(N, world, rank)
            xl = to_device(np.ascontiguousarray(x[:, a:b]))
            out = multi.scan_multi(xl, op, kind, mode="elements", backend="peer", comm=comm)
            torch.cuda.synchronize()
            ref_full = x
            got_local = to_host(out, x.dtype).reshape(G, b - a)
            # parity of this rank's slice against the oracle of the whole problem
            if x.dtype == np.float32 and op == "add":
                ref, sabs = oracle.scan(ref_full, op, kind, with_abs=True)
                bad = np.abs(got_local - ref[:, a:b]) > 1e-5 * sabs[:, a:b]
                if bad.any():
                    msg = "BAD f32 it=%d" % it
            else:
                if not np.array_equal(got_local, oracle.scan(ref_full, op, kind)[:, a:b]):
                    msg = "BAD it=%d %s %s %s" % (it, op, dist_name, kind)
    finally:
        torch.cuda.synchronize()
        dist.barrier()
        comm.close()
        with open(os.path.join(outdir, "rank%d" % rank), "w") as f:
            f.write(msg)
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
