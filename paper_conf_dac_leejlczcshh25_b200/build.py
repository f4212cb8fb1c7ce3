"""Build libigk.so (sm_100a) in-tree with nvcc."""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SO = os.path.join(HERE, "libigk.so")
SRCS = ["csrc/igk.cu"]
DEPS = ["csrc/igk.cu", "csrc/common.cuh", "csrc/apply.cuh", "csrc/refine.cuh", "csrc/step.cuh", "csrc/recount.cuh", "csrc/recount3.cuh", "csrc/fgp.cuh", "../include/igk.h"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC", "-shared", "-Xptxas", "-v"]


def stale() -> bool:
    if not os.path.exists(SO):
        return True
    t = os.path.getmtime(SO)
    return any(os.path.getmtime(os.path.join(HERE, p)) > t for p in DEPS)


def build(force: bool = False, verbose: bool = False) -> str:
    if force or stale():
        cmd = [NVCC, *FLAGS, *[os.path.join(HERE, s) for s in SRCS], "-o", SO]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("nvcc failed:\n" + r.stdout + r.stderr)
        if verbose:
            print(r.stderr)
    return SO


if __name__ == "__main__":
    build(force=True, verbose=True)
