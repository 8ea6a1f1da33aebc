"""Build the sm_100a shared library libspgemm_b200.so in-tree with nvcc (no torch JIT cache).

The library exports the C ABI declared in include/spgemm.h.  Cross-compiles without a GPU.
"""
from __future__ import annotations

import glob
import os
import shutil
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
SOURCES = [os.path.join(CSRC, f) for f in ("api.cu", "panels.cu", "kernels.cu")]
HEADERS = sorted(glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) +
                 glob.glob(os.path.join(ROOT, "include", "*.h")))
LIB = os.path.join(HERE, "libspgemm_b200.so")

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC,-O3,-Wall",
    "-Xptxas", "-O3",
]
OBJDIR = os.path.join(HERE, "build")


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def _obj(src: str) -> str:
    return os.path.join(OBJDIR, os.path.basename(src)[:-3] + ".o")


def _newest_dep() -> float:
    return max(os.path.getmtime(f) for f in HEADERS + [__file__])


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in SOURCES + HEADERS + [__file__])


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile every translation unit for sm_100a in parallel (one nvcc per .cu; a unit is rebuilt
    when it or any header is newer than its object), then link the shared library."""
    if not force and not stale():
        return LIB
    os.makedirs(OBJDIR, exist_ok=True)
    dep = _newest_dep()
    procs = []
    for src in SOURCES:
        o = _obj(src)
        if force or not os.path.exists(o) or os.path.getmtime(o) < max(os.path.getmtime(src), dep):
            tmp = o + f".tmp{os.getpid()}"
            cmd = [nvcc(), *NVCC_FLAGS, "-c", "-o", tmp, src]
            if verbose:
                print(" ".join(cmd), file=sys.stderr)
            procs.append((subprocess.Popen(cmd), tmp, o))
    bad = False
    for p, tmp, o in procs:
        if p.wait() != 0:
            bad = True
        else:
            os.replace(tmp, o)
    if bad:
        raise subprocess.CalledProcessError(1, "nvcc")
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [nvcc(), "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", tmp, *[_obj(s) for s in SOURCES]]
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
