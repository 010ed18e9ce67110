"""In-tree build of libdgr.so (nvcc, sm_100a) — the B200 DGR solver behind include/dgr.h."""
from __future__ import annotations

import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libdgr.so")
SOURCES = [os.path.join(CSRC, f) for f in ("dgr_api.cu", "dgr_kernels.cu", "dgr_forest.cu")]
HEADERS = [os.path.join(CSRC, "dgr_internal.h"), os.path.join(ROOT, "include", "dgr.h")]

NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17",
              "-Xcompiler", "-fPIC,-fopenmp", "-shared", "-lgomp"]


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if c and (os.path.sep not in c or os.path.exists(c)):
            return c
    return "nvcc"


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in SOURCES + HEADERS)


def build(verbose: bool = False, force: bool = False) -> str:
    if not force and not stale():
        return LIB
    extra = os.environ.get("DGR_NVCC_EXTRA", "").split()
    cmd = [nvcc(), *NVCC_FLAGS, *extra, "-I" + os.path.join(ROOT, "include"), "-o", LIB, *SOURCES, "-lnccl"]
    if verbose:
        print(" ".join(cmd))
    subprocess.check_call(cmd)
    return LIB


if __name__ == "__main__":
    build(verbose=True, force=True)
