"""Build the sm_100a shared library (in-tree): liblocassm.so next to this file.

nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -shared -Xcompiler -fPIC
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SO = os.path.join(HERE, "liblocassm.so")
SRC = [os.path.join(HERE, "csrc", "locassm.cu"), os.path.join(HERE, "csrc", "la_cpu.cpp")]
DEPS = SRC + sorted(glob.glob(os.path.join(HERE, "csrc", "*.cu*")) + glob.glob(os.path.join(HERE, "csrc", "*.h")) +
                   glob.glob(os.path.join(HERE, "csrc", "*.cpp"))) + [os.path.join(ROOT, "include", "locassm.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-shared", "-Xcompiler", "-fPIC", "-I" + os.path.join(ROOT, "include")]


def build(force: bool = False, verbose: bool = False) -> str:
    stale = not os.path.exists(SO) or os.path.getmtime(SO) < max(os.path.getmtime(p) for p in DEPS)
    if force or stale:
        cmd = [NVCC, *FLAGS, *os.environ.get("LA_NVCC_EXTRA", "").split(), "-o", SO, *SRC]
        if verbose:
            cmd.insert(1, "-Xptxas=-v")
            print(" ".join(cmd), file=sys.stderr)
        subprocess.check_call(cmd)
    return SO


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
