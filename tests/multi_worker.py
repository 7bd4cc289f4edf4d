"""Worker bodies for the multi-process tests (spawned by torch.multiprocessing)."""
import os

import numpy as np
import torch
import torch.distributed as dist

import inputs
import oracle


def _init(rank, world, port, backend):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group(backend, rank=rank, world_size=world)


def gloo_elements_worker(rank, world, port, G, N, dist_name, kind, result_dir):
    """Elements mode host logic on CPU: partition + exchange_totals (gloo) + rank-ordered
    carries; the local Stage 1+2/3 arithmetic is the ORACLE here (test side), the product
    supplies the plan and the exchange."""
    _init(rank, world, port, "gloo")
    from paper_conf_ipps_dieguezadnm18_b200.multi import exchange_totals, partition
    a, b = partition(N, world, rank)
    full = inputs.generate(dist_name, G * N, 2018).reshape(G, N)
    xl = np.ascontiguousarray(full[:, a:b])
    if xl.dtype == np.float32:
        tot = oracle.totals(xl, N=b - a) if b > a else np.zeros(G)
        slots = torch.from_numpy(tot.view(np.int64).copy())
    else:
        tot = oracle.totals(xl, N=b - a) if b > a else np.zeros(G, np.uint32)
        slots = torch.from_numpy(tot.astype(np.int64))
    allt = exchange_totals(slots)                     # [W, G], rank-major
    assert tuple(allt.shape) == (world, G)
    mine = allt[rank].numpy()
    assert np.array_equal(mine, slots.numpy())
    # carry of rank r = fold of totals of ranks < r (Stage 2 of PAPER.md:197-205)
    if xl.dtype == np.float32:
        carry = allt[:rank].numpy().view(np.float64).sum(axis=0) if rank else np.zeros(G)
        local = oracle.scan(xl, "add", kind) if b > a else np.zeros((G, 0))
        got = local + carry[:, None]
        ref, sabs = oracle.scan(full, "add", kind, with_abs=True)
        ok = np.all(np.abs(got - ref[:, a:b]) <= 1e-12 * np.maximum(sabs[:, a:b], 1))
    else:
        carry = (allt[:rank].numpy().astype(np.uint64).sum(axis=0) & 0xFFFFFFFF).astype(np.uint32) if rank \
            else np.zeros(G, np.uint32)
        local = oracle.scan(xl, "add", kind).view(np.uint32) if b > a else np.zeros((G, 0), np.uint32)
        got = (local + carry[:, None]).view(xl.dtype)
        ok = np.array_equal(got, oracle.scan(full, "add", kind)[:, a:b])
    with open(os.path.join(result_dir, "rank%d" % rank), "w") as f:
        f.write("ok" if ok else "BAD")
    dist.barrier()
    dist.destroy_process_group()


def gloo_problems_worker(rank, world, port, G, result_dir):
    _init(rank, world, port, "gloo")
    from paper_conf_ipps_dieguezadnm18_b200.multi import partition
    a, b = partition(G, world, rank)
    t = torch.tensor([a, b], dtype=torch.int64)
    gathered = [torch.zeros(2, dtype=torch.int64) for _ in range(world)]
    dist.all_gather(gathered, t)
    spans = [tuple(x.tolist()) for x in gathered]
    ok = spans[0][0] == 0 and spans[-1][1] == G and all(spans[i][1] == spans[i + 1][0] for i in range(world - 1))
    with open(os.path.join(result_dir, "rank%d" % rank), "w") as f:
        f.write("ok" if ok else "BAD %s" % spans)
    dist.destroy_process_group()


def gloo_grouped_worker(rank, world, port, V, G, N, result_dir):
    """MP-PC grouping: Y = W/V groups, each scatters its problems over its V ranks."""
    _init(rank, world, port, "gloo")
    from paper_conf_ipps_dieguezadnm18_b200.multi import exchange_totals, grouped_plan, make_groups
    sub = make_groups(V)
    plan = grouped_plan(G, N, world, V, rank)
    g0, g1 = plan["problems"]
    e0, e1 = plan["elements"]
    full = inputs.generate("i32", G * N, 77).reshape(G, N)
    xl = np.ascontiguousarray(full[g0:g1, e0:e1])
    ng = g1 - g0
    tot = oracle.totals(xl, N=e1 - e0) if (e1 > e0 and ng) else np.zeros(ng, np.uint32)
    allt = exchange_totals(torch.from_numpy(tot.astype(np.int64)), group=sub)     # [V, ng]
    v = plan["member"]
    carry = (allt[:v].numpy().astype(np.uint64).sum(axis=0) & 0xFFFFFFFF).astype(np.uint32) if v \
        else np.zeros(ng, np.uint32)
    local = oracle.scan(xl, "add").view(np.uint32) if (e1 > e0 and ng) else np.zeros((ng, e1 - e0), np.uint32)
    got = (local + carry[:, None]).view(np.int32)
    ok = np.array_equal(got, oracle.scan(full, "add")[g0:g1, e0:e1])
    with open(os.path.join(result_dir, "rank%d" % rank), "w") as f:
        f.write("ok" if ok else "BAD")
    dist.barrier()
    dist.destroy_process_group()
