"""Builds libdedup_b200.so (sm_100a) in-tree with nvcc.

The library is plain C ABI (include/dedup.h); it statically links the CUDA
runtime, so it does not depend on the PyTorch build.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libdedup_b200.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

def _nccl():
    """The NCCL that torch loads (the wheel's)."""
    try:
        import nvidia.nccl
        base = list(nvidia.nccl.__path__)[0]
        return os.path.join(base, "include"), os.path.join(base, "lib")
    except Exception:
        return None, None


NCCL_INC, NCCL_LIB = _nccl()

FLAGS = [
    "-O3", "-std=c++17", "-lineinfo",
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-Xcompiler", "-fPIC", "-shared",
    "-I", os.path.join(ROOT, "include"),
]
if NCCL_INC:
    FLAGS += ["-I", NCCL_INC, "-L", NCCL_LIB, "-l:libnccl.so.2",
              "-Xlinker", f"-rpath={NCCL_LIB}"]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def deps():
    return sources() + glob.glob(os.path.join(CSRC, "*.h")) + [
        *glob.glob(os.path.join(ROOT, "include", "*.h")), __file__]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(p) > t for p in deps())


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not stale():
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [NVCC, *FLAGS, "-o", tmp, *sources()]
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
