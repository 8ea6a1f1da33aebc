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
# the checked build: device-side bounds checks (SPG_CHECK in kernels.cu) that print and trap; loaded
# by capi when SPGEMM_CHECKED=1 (tests/test_gpu_checked.py) -- compute-sanitizer is closed on the GPU pool
LIB_CHECKED = os.path.join(HERE, "libspgemm_b200_checked.so")

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


def _obj(src: str, checked: bool = False) -> str:
    base = os.path.basename(src)[:-3]
    return os.path.join(OBJDIR, base + ("_checked.o" if checked else ".o"))


# translation units compiled differently in the checked build (the others' objects are shared)
CHECKED_SOURCES = [os.path.join(CSRC, "kernels.cu")]


def _newest_dep() -> float:
    return max(os.path.getmtime(f) for f in HEADERS + [__file__])


def stale() -> bool:
    for lib in (LIB, LIB_CHECKED):
        if not os.path.exists(lib):
            return True
        t = os.path.getmtime(lib)
        if any(os.path.getmtime(s) > t for s in SOURCES + HEADERS + [__file__]):
            return True
    return False


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile every translation unit for sm_100a in parallel (one nvcc per .cu; a unit is rebuilt
    when it or any header is newer than its object), then link the shared library and its checked
    variant (kernels.cu with -DSPGEMM_CHECKS)."""
    if not force and not stale():
        return LIB
    os.makedirs(OBJDIR, exist_ok=True)
    dep = _newest_dep()
    procs = []
    units = [(s, False) for s in SOURCES] + [(s, True) for s in CHECKED_SOURCES]
    for src, chk in units:
        o = _obj(src, chk)
        if force or not os.path.exists(o) or os.path.getmtime(o) < max(os.path.getmtime(src), dep):
            tmp = o + f".tmp{os.getpid()}"
            cmd = [nvcc(), *NVCC_FLAGS, *(["-DSPGEMM_CHECKS"] if chk else []), "-c", "-o", tmp, src]
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
    for lib, chk in ((LIB, False), (LIB_CHECKED, True)):
        objs = [_obj(s, chk and s in CHECKED_SOURCES) for s in SOURCES]
        tmp = lib + f".tmp{os.getpid()}"
        cmd = [nvcc(), "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", tmp, *objs]
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        subprocess.check_call(cmd)
        os.replace(tmp, lib)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
