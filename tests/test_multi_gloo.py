"""Multi-process host logic of the multi-GPU layer on CPU (gloo, world_size 2 and 3)."""
import os
import random

import pytest
import torch.multiprocessing as mp

import multi_worker
from paper_conf_ipps_dieguezadnm18_b200.multi import partition


def _port():
    return random.randint(20000, 40000)


def test_partition_covers_everything():
    for n in (0, 1, 2, 7, 4096, 65536 + 3):
        for w in (1, 2, 3, 8):
            spans = [partition(n, w, r) for r in range(w)]
            assert spans[0][0] == 0 and spans[-1][1] == n
            assert all(spans[i][1] == spans[i + 1][0] for i in range(w - 1))
            assert max(b - a for a, b in spans) - min(b - a for a, b in spans) <= 1
    with pytest.raises(ValueError):
        partition(5, 0, 0)


@pytest.mark.parametrize("world,G,N,dist_name,kind", [
    (2, 3, 10001, "i32", "inclusive"),
    (2, 1, 4097, "f32s", "exclusive"),
    (3, 2, 2, "u32", "inclusive"),          # a rank with an empty portion
])
def test_gloo_elements_mode(tmp_path, world, G, N, dist_name, kind):
    mp.spawn(multi_worker.gloo_elements_worker, args=(world, _port(), G, N, dist_name, kind, str(tmp_path)),
             nprocs=world, join=True)
    for r in range(world):
        assert open(os.path.join(tmp_path, "rank%d" % r)).read() == "ok"


def test_gloo_problems_mode(tmp_path):
    mp.spawn(multi_worker.gloo_problems_worker, args=(2, _port(), 4097, str(tmp_path)), nprocs=2, join=True)
    for r in range(2):
        assert open(os.path.join(tmp_path, "rank%d" % r)).read() == "ok"


def test_grouped_plan_covers_everything():
    from paper_conf_ipps_dieguezadnm18_b200.multi import grouped_plan
    G, N, W, V = 7, 1001, 8, 4
    cells = set()
    for r in range(W):
        p = grouped_plan(G, N, W, V, r)
        assert p["groups"] == 2 and p["group"] == r // V and p["member"] == r % V
        for g in range(*p["problems"]):
            cells.add((g, p["elements"]))
    for g in range(G):
        spans = sorted(e for gg, e in cells if gg == g)
        assert spans[0][0] == 0 and spans[-1][1] == N and len(spans) == V


def test_gloo_grouped_mode(tmp_path):
    mp.spawn(multi_worker.gloo_grouped_worker, args=(4, _port(), 2, 5, 3001, str(tmp_path)), nprocs=4, join=True)
    for r in range(4):
        assert open(os.path.join(tmp_path, "rank%d" % r)).read() == "ok"
