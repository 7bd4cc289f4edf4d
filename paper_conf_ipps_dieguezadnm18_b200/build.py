"""Build the native libraries in-tree with nvcc for sm_100a (no JIT, no torch extension).

    libscanb200.so   <- paper_conf_ipps_dieguezadnm18_b200/csrc/*.cu   (the product)
    inputs/libinputs.so <- inputs/gen.cu                                 (shared input generator)

Flags: -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo, IEEE float (no fast-math).
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(ROOT, "build")
LIB = os.path.join(PKG, "libscanb200.so")
GEN_SRC = os.path.join(ROOT, "inputs", "gen.cu")
GEN_LIB = os.path.join(ROOT, "inputs", "libinputs.so")

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xptxas", "-v",
         "-I", os.path.join(ROOT, "include"), "-I", CSRC]


def _newer(target: str, deps: list[str]) -> bool:
    if not os.path.exists(target):
        return False
    t = os.path.getmtime(target)
    return all(os.path.getmtime(d) <= t for d in deps)


def _run(cmd: list[str], log: str | None = None) -> None:
    r = subprocess.run(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)
    if log:
        with open(log, "w") as f:
            f.write(r.stdout)
    if r.returncode != 0:
        sys.stderr.write(r.stdout)
        raise RuntimeError("build failed: " + " ".join(cmd))


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    headers = sorted(glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh"))
                     + glob.glob(os.path.join(ROOT, "include", "*.h")))
    objs = []
    jobs = []
    for s in srcs:
        o = os.path.join(BUILD, os.path.basename(s) + ".o")
        objs.append(o)
        if force or not _newer(o, [s] + headers):
            jobs.append(([NVCC, *ARCH, *FLAGS, "-c", s, "-o", o], o + ".log"))
    with cf.ThreadPoolExecutor(max_workers=min(8, max(1, len(jobs)))) as ex:
        list(ex.map(lambda j: _run(*j), jobs))
    if force or jobs or not _newer(LIB, objs):
        tmp = LIB + ".tmp%d" % os.getpid()
        _run([NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart", "-ldl"])
        os.replace(tmp, LIB)
    if force or not _newer(GEN_LIB, [GEN_SRC]):
        tmp = GEN_LIB + ".tmp%d" % os.getpid()
        _run([NVCC, *ARCH, "-O3", "-Xcompiler", "-fPIC", "-shared", "-o", tmp, GEN_SRC])
        os.replace(tmp, GEN_LIB)
    if verbose:
        for j in glob.glob(os.path.join(BUILD, "*.log")):
            print(open(j).read())
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
