"""Build libgsnp.so in-tree for sm_100a (nvcc cross-compiles without a GPU)."""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SRC = os.path.join(HERE, "csrc", "gsnp.cu")
SRC_DEEP = os.path.join(HERE, "csrc", "gsnp_deep.cu")   # deep-window kernel, 384-thread CTAs
DEPS = [SRC, SRC_DEEP, os.path.join(HERE, "csrc", "gsnp_kernels.cuh"),
        os.path.join(HERE, "csrc", "gsnp_compress.cuh"), os.path.join(HERE, "csrc", "gsnp_dense.cuh"),
        os.path.join(HERE, "csrc", "gsnp_parse.cuh"),
        os.path.join(HERE, "csrc", "gsnp_pack.cuh"),
        os.path.join(ROOT, "include", "gsnp.h")]
LIB = os.path.join(HERE, "libgsnp.so")

NVCC_FLAGS = ["-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo",
              "--fmad=false", "-Xcompiler", "-fPIC,-ffp-contract=off", "-shared",
              "-I" + os.path.join(ROOT, "include")]


def build(force: bool = False, verbose: bool = False) -> str:
    stale = not os.path.exists(LIB) or any(os.path.getmtime(LIB) < os.path.getmtime(d) for d in DEPS)
    if force or stale:
        nvcc = os.environ.get("NVCC", "nvcc")
        cmd = [nvcc] + NVCC_FLAGS + (["-Xptxas", "-v"] if verbose else []) + ["-o", LIB, SRC, SRC_DEEP]
        subprocess.check_call(cmd)
    return LIB


if __name__ == "__main__":
    import sys
    print(build(force="-f" in sys.argv, verbose="-v" in sys.argv))
