"""MP-PC grouping on the GPU path (PAPER.md:213-217 [§4.1.1, Fig. 8]).

W = 4 real ranks (four processes, four CUDA contexts sharing cuda:0), Y = W/V groups of V
ranks from multi.make_groups; each group scans its share of the problems in elements mode
on its own sub-communicator, through the product kernels with both exchanges (fused peer
stores over CUDA-IPC-mapped mailboxes, and the torch all-gather of the totals).  Every
rank compares its slice with the oracle of the whole batch (tests/grouped_worker.py); no
oracle arithmetic is used on the product side.
"""
import os
import random
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.mark.parametrize("W,V", [(4, 2), (4, 4), (4, 1)])
def test_grouped_elements_mode_processes(tmp_path, W, V):
    port = random.randint(20000, 40000)
    env = dict(os.environ, PYTHONPATH=os.pathsep.join([os.path.dirname(HERE), HERE]))
    procs = [subprocess.Popen([sys.executable, os.path.join(HERE, "grouped_worker.py"), str(r), str(W), str(V),
                               str(port), str(tmp_path)], env=env, stdout=subprocess.PIPE,
                              stderr=subprocess.STDOUT) for r in range(W)]
    logs = []
    try:
        for p in procs:
            out, _ = p.communicate(timeout=400)
            logs.append(out.decode(errors="replace"))
    finally:
        for p in procs:
            if p.poll() is None:
                p.kill()
    for r, p in enumerate(procs):
        assert p.returncode == 0, "rank %d failed:\n%s" % (r, logs[r][-3000:])
        assert open(os.path.join(tmp_path, "rank%d" % r)).read().startswith("ok"), \
            open(os.path.join(tmp_path, "rank%d" % r)).read()
