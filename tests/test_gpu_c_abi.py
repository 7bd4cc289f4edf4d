"""The C-ABI from a plain C program (tests/c/abi_demo.c): compiled with gcc against
include/scan_b200.h and libscanb200.so, run on the GPU; no Python in the data path."""
import os
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_ipps_dieguezadnm18_b200")


def _build(tmp_path):
    exe = str(tmp_path / "abi_demo")
    cuda = "/usr/local/cuda"
    subprocess.check_call(["gcc", "-O2", "-std=c11", os.path.join(ROOT, "tests", "c", "abi_demo.c"),
                           "-I", os.path.join(ROOT, "include"), "-I", cuda + "/include",
                           "-L", PKG, "-lscanb200", "-L", cuda + "/lib64", "-lcudart",
                           "-Wl,-rpath," + PKG, "-o", exe])
    return exe


def test_c_program_builds(tmp_path):
    assert os.path.exists(_build(tmp_path))


@pytest.mark.gpu
def test_c_program_runs(tmp_path):
    exe = _build(tmp_path)
    r = subprocess.run([exe], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr
    assert "abi_demo ok" in r.stdout
