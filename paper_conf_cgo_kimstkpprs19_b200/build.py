"""Build libtc.so in-tree (nvcc, sm_100a).  Used by __graft_entry__.build() and the tests."""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
SO = os.path.join(HERE, "libtc.so")
SOURCES = ["api.cu", "contraction.cpp", "planner.cpp", "tiles.cpp", "kernels_00.cu", "kernels_01.cu",
           "kernels_10.cu", "kernels_11.cu", "kernels_bf16.cu"]
HEADERS = ["contraction.hpp", "planner.hpp", "kparams.hpp", "kernel_f64.cuh", "tiles.hpp",
           "kernel_table.cuh", "kernel_bf16.cuh"]
NVCC_FLAGS = ["-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo",
              "-Xcompiler", "-fPIC", "-shared"]


def _stale() -> bool:
    if not os.path.exists(SO):
        return True
    t = os.path.getmtime(SO)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS]
    deps.append(os.path.join(os.path.dirname(HERE), "include", "libtc.h"))
    return any(os.path.getmtime(d) > t for d in deps if os.path.exists(d))


def build(force: bool = False, verbose: bool = False) -> str:
    if force or _stale():
        nvcc = os.path.join(os.environ.get("CUDA_HOME", "/usr/local/cuda"), "bin", "nvcc")
        cmd = [nvcc] + NVCC_FLAGS + (["-Xptxas", "-v"] if verbose else []) + SOURCES + ["-o", SO]
        subprocess.check_call(cmd, cwd=CSRC)
    return SO


if __name__ == "__main__":
    build(force=True, verbose=True)
