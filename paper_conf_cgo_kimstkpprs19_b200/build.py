"""Build libtc.so in-tree (nvcc, sm_100a).  Used by __graft_entry__.build() and the tests."""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
SO = os.path.join(HERE, "libtc.so")
SOURCES = ["api.cu", "group_api.cu", "contraction.cpp", "planner.cpp", "tiles.cpp", "group.cpp",
           "kernels_00.cu", "kernels_01.cu", "kernels_10.cu", "kernels_11.cu", "kernels_umma.cu", "kernels_umma_tma.cu", "kernels_umma_pair.cu", "kernels_umma_f32out.cu",
           "kernels_group.cu", "stream.cpp", "kernels_stream.cu", "kernels_stream_beta.cu"]
HEADERS = ["contraction.hpp", "planner.hpp", "kparams.hpp", "kernel_f64.cuh", "tiles.hpp", "variants.def",
           "kernel_table.cuh", "kernel_umma.cuh", "group.hpp", "kernel_group.cuh", "plan_internal.hpp", "stream.hpp", "kernel_stream.cuh"]
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
    """Compile every translation unit in parallel (the kernel tables are split across TUs),
    then link libtc.so."""
    if force or _stale():
        from concurrent.futures import ThreadPoolExecutor
        nvcc = os.path.join(os.environ.get("CUDA_HOME", "/usr/local/cuda"), "bin", "nvcc")
        # (a side build, e.g. tools/trace_umma.py's -DTC_TRACE library, keeps its own objects)
        objdir = os.path.join(HERE, "build") if SO == os.path.join(HERE, "libtc.so") else os.path.dirname(SO)
        os.makedirs(objdir, exist_ok=True)
        cflags = [f for f in NVCC_FLAGS if f != "-shared"]

        def one(src):
            obj = os.path.join(objdir, os.path.splitext(src)[0] + ".o")
            cmd = [nvcc] + cflags + (["-Xptxas", "-v"] if verbose else []) + ["-c", src, "-o", obj]
            r = subprocess.run(cmd, cwd=CSRC, capture_output=True, text=True)
            if r.returncode != 0:
                raise RuntimeError(f"nvcc failed on {src}:\n{r.stderr}")
            if verbose:
                print(r.stderr)
            return obj

        with ThreadPoolExecutor(max_workers=max(1, min(len(SOURCES), os.cpu_count() or 1))) as ex:
            objs = list(ex.map(one, SOURCES))
        subprocess.check_call([nvcc, "-shared", "-gencode", "arch=compute_100a,code=sm_100a"] + objs +
                              ["-o", SO + ".tmp"])
        os.replace(SO + ".tmp", SO)
    return SO


if __name__ == "__main__":
    build(force=True, verbose=True)
