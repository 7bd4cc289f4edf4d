"""Soak test of the fused peer-memory exchange (scan_comm_create_peer) with W real ranks
(W processes sharing cuda:0, CUDA-IPC-mapped mailboxes, gloo plumbing): many consecutive
elements-mode calls with random G (up to 2048: the short-portion
warp path too) and random (uneven, sometimes empty) portions -- the
mailbox halves, flags and acknowledgements cycle through hundreds of epochs.  Every 7th
call is checked against the oracle of the whole batch.

    python tools/peer_soak.py W ITERS        # spawns W ranks, prints one line per rank
"""
import os
import random
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)


def rank_main(rank, world, iters, port):
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import numpy as np
    import torch
    import torch.distributed as dist
    import inputs
    import oracle
    from gpu_util import to_device, to_host
    from paper_conf_ipps_dieguezadnm18_b200 import multi
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    comm = multi.PeerComm(2048)
    rng = random.Random(1234)                   # identical sequence on every rank
    bad = 0
    for it in range(iters):
        G = rng.choice([1, 1, 2, 3, 17, 64, 1300, 2048])
        if G > 64:      # many short portions: the warp-per-problem Stage 1 / Stage 3 (N_local <= 4096)
            lens = [rng.choice([0, 1, 37, 1000, 2048, 4096, 5000]) for _ in range(world)]
        else:
            lens = [rng.choice([0, 1, 5, 4096, 9000, 70001]) for _ in range(world)]
        if sum(lens) == 0:
            lens[-1] = 3
        Ntot = sum(lens)
        op, dname, kind = rng.choice([("add", "i32", "inclusive"), ("add", "u32", "exclusive"),
                                      ("max", "i32", "inclusive"), ("add", "f32s", "exclusive")])
        x = inputs.generate(dname, G * Ntot, seed=it).reshape(G, Ntot)
        a = sum(lens[:rank])
        xl = to_device(np.ascontiguousarray(x[:, a:a + lens[rank]]))
        out = multi.scan_multi(xl, op, kind, mode="elements", backend="peer", comm=comm)
        if it % 7 == 0:
            torch.cuda.synchronize()
            got = to_host(out, x.dtype).reshape(G, lens[rank])
            if x.dtype == np.float32:
                ref, sabs = oracle.scan(x, op, kind, with_abs=True)
                ok = bool(np.all(np.abs(got - ref[:, a:a + lens[rank]]) <= 1e-5 * sabs[:, a:a + lens[rank]]))
            else:
                ok = np.array_equal(got, oracle.scan(x, op, kind)[:, a:a + lens[rank]])
            bad += 0 if ok else 1
    torch.cuda.synchronize()
    dist.barrier()
    comm.close()
    print("rank %d: %d calls, %d checked, %d bad" % (rank, iters, (iters + 6) // 7, bad), flush=True)
    dist.destroy_process_group()
    return bad


if __name__ == "__main__":
    if len(sys.argv) > 4 and sys.argv[1] == "--rank":
        sys.exit(1 if rank_main(int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), int(sys.argv[5])) else 0)
    W, iters = int(sys.argv[1]), int(sys.argv[2])
    port = random.randint(20000, 40000)
    procs = [subprocess.Popen([sys.executable, os.path.abspath(__file__), "--rank", str(r), str(W), str(iters), str(port)])
             for r in range(W)]
    rc = [p.wait(timeout=3000) for p in procs]
    print("soak W=%d iters=%d: exit codes %s" % (W, iters, rc))
    sys.exit(max(rc))
