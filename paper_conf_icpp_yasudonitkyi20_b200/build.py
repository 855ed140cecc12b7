"""Build libabs.so (the C-ABI library of include/abs.h) in-tree with nvcc for
sm_100a.  No JIT cache: the .so sits next to this file so it travels with the
repository snapshot to the GPU box."""
from __future__ import annotations

import os
import shutil
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libabs.so")
TIMING_LIB = os.path.join(HERE, "libabs_timing.so")  # diagnostics variant (-DABS_TIMING)
SOURCES = ["abs_round.cu", "abs_round_warp.cu", "abs_setup.cu", "abs_init_mma.cu", "abs_host.cpp"]
HEADERS = ["abs_internal.h", "abs_round_common.cuh", "philox.hpp", "ptx.cuh"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "abs.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, timing: bool = False) -> str:
    lib = TIMING_LIB if timing else LIB
    if not force and not timing and not _stale():
        return LIB
    tmp = lib + ".tmp%d" % os.getpid()
    cmd = [nvcc(), *ARCH, *(["-DABS_TIMING"] if timing else []), "-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC",
           "-Xcompiler", "-fvisibility=hidden", "-Xcompiler", "-fopenmp", "-I", os.path.join(ROOT, "include"), "-I", CSRC,
           "-o", tmp] + [os.path.join(CSRC, f) for f in SOURCES] + ["-lpthread", "-lgomp"]
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(tmp, lib)
    return lib


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True, timing="--timing" in sys.argv))
