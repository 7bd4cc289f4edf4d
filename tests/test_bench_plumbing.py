"""CPU checks of bench.py's multi-rank plumbing (no GPU): `--gpus N` outside torchrun
re-launches N ranks by itself (torch.distributed.run, 127.0.0.1), ranks meet in a gloo
group, the max/min over ranks reach rank 0, and only rank 0 prints one JSON line; a
WORLD_SIZE that disagrees with --gpus fails loudly."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env=None, timeout=240):
    e = dict(os.environ)
    for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT"):
        e.pop(k, None)
    e.update(env or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True,
                          text=True, timeout=timeout, env=e)


def test_bench_spawns_ranks_for_gpus_n():
    r = _run(["--gpus", "3", "--dry-run", "--steps", "5", "--warmup", "3"])
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 3 and d["dry_run"] is True
    assert d["ranks_seen"] == {"max": 3.0, "min": 1.0}
    assert d["config"]["parallelism"].endswith("dp3")


def test_bench_world_size_mismatch_fails_loudly():
    r = _run(["--gpus", "2", "--dry-run"], env={"WORLD_SIZE": "1", "RANK": "0", "LOCAL_RANK": "0"})
    assert r.returncode == 2
    assert "WORLD_SIZE" in r.stderr


def test_reference_arm_runs_on_cpu():
    # the reference arm of this paper-only run is the CPU oracle (no GPU needed): one JSON
    # line with impl=reference, the base contract's keys, cpu_baseline and a zero-copy e2e
    r = _run(["--impl", "reference", "--steps", "2", "--warmup", "1"])
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["unit"] == "Gelem/s" and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert d["higher_is_better"] is True and d["steps"] == 2 and d["warmup"] == 1
