"""Multi-GPU layer on the one GPU the box gives: a world-size-1 NCCL process group drives
the real collective path (torch all_gather_into_tensor and the native scan_batch_multi on
the group's ncclComm_t); multi-rank carries are covered by the loopback test in
test_gpu_parity.py and by the gloo tests."""
import os
import random

import numpy as np
import pytest
import torch
import torch.distributed as dist

import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
from gpu_util import COMBOS, DIST, NP, assert_parity, to_device, to_host
from paper_conf_ipps_dieguezadnm18_b200 import multi

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def nccl_world1():
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(random.randint(20000, 40000))
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    yield
    dist.destroy_process_group()


@pytest.mark.parametrize("backend", ["torch", "native"])
def test_elements_mode_world1(nccl_world1, backend):
    comm = multi.NativeComm() if backend == "native" else None
    try:
        for op, dt in COMBOS:
            for G, N in [(1, 300001), (3, 4096 * 5 + 3), (2, 0)]:
                x = inputs.generate(DIST[dt], G * N, seed=G + N).reshape(G, N)
                xd = to_device(x)
                out = multi.scan_multi(xd, op, "inclusive", mode="elements", backend=backend, comm=comm)
                torch.cuda.synchronize()
                assert_parity(to_host(out, NP[dt]).reshape(G, N), x, op, "inclusive",
                              label="multi %s %s %s" % (backend, op, dt))
    finally:
        if comm is not None:
            comm.close()


def test_problems_mode_world1(nccl_world1):
    G, N = 1000, 5000
    x = inputs.generate("i32", G * N, 3).reshape(G, N)
    a, b = multi.partition(G, 1, 0)
    out = multi.scan_multi(to_device(x[a:b]), "add", "exclusive", mode="problems")
    torch.cuda.synchronize()
    assert_parity(to_host(out, np.int32).reshape(b - a, N), x[a:b], "add", "exclusive")
