"""Build the in-tree C-ABI library libcuart.so (sm_100a) with nvcc + g++.

    python -m paper_conf_icpp_koppehelggp21_b200.build [--force]

Host code (builder, CPU layout walker) is compiled with g++ -O3 -fopenmp; the
kernels and the C ABI with nvcc for ``-gencode arch=compute_100a,code=sm_100a``
(-lineinfo for ncu source mapping).  The CUDA runtime is linked statically so the
library loads on a machine without a GPU (the CPU tests check its exports).
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
OUT = os.path.join(PKG, "libcuart.so")
BUILD = os.path.join(ROOT, "build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_root():
    """NCCL 2.28 shipped with the PyTorch wheels (headers + libnccl.so.2); the multi-GPU
    layer (csrc/dist.cu) links it for its NCCL transport and bootstrap."""
    import nvidia.nccl
    return list(nvidia.nccl.__path__)[0]


NCCL_ROOT = _nccl_root()
NCCL_LIB = os.path.join(NCCL_ROOT, "lib")


def _sources():
    return [os.path.join(CSRC, f) for f in sorted(os.listdir(CSRC))
            if f.endswith((".cu", ".cpp", ".h", ".cuh"))] + [os.path.join(ROOT, "include", "cuart.h")]


def _run(cmd):
    print("+", " ".join(cmd), flush=True)
    subprocess.check_call(cmd)


def build(force: bool = False, verbose_ptxas: bool = False) -> str:
    srcs = _sources()
    if not force and os.path.exists(OUT) and os.path.getmtime(OUT) >= max(os.path.getmtime(s) for s in srcs):
        return OUT
    os.makedirs(BUILD, exist_ok=True)
    inc = ["-I", os.path.join(ROOT, "include"), "-I", CSRC, "-I", os.path.join(NCCL_ROOT, "include")]
    inc += os.environ.get("CUART_DEFS", "").split()          # e.g. "-DCUART_N16_BYTES=256" (layout experiments)
    objs = []
    for f in sorted(os.listdir(CSRC)):
        src = os.path.join(CSRC, f)
        obj = os.path.join(BUILD, f + ".o")
        if f.endswith(".cpp"):
            _run(["g++", "-O3", "-std=c++17", "-fPIC", "-fopenmp", "-march=x86-64-v2", *inc, "-c", src, "-o", obj])
        elif f.endswith(".cu"):
            cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-fopenmp",
                   *inc, "-c", src, "-o", obj]
            if verbose_ptxas:
                cmd.insert(1, "-Xptxas=-v")
            _run(cmd)
        else:
            continue
        objs.append(obj)
    tmp = OUT + f".tmp{os.getpid()}"
    _run([NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs, "-Xcompiler", "-fopenmp", "-lgomp",
          "-L", NCCL_LIB, "-l:libnccl.so.2", "-Xlinker", "-rpath=" + NCCL_LIB])
    os.replace(tmp, OUT)
    return OUT


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose_ptxas="-v" in sys.argv)
