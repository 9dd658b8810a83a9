"""Build the sm_100a shared library in-tree (libproclus.so next to this file).

nvcc cross-compiles for B200 without a GPU: ``-gencode
arch=compute_100a,code=sm_100a``, ``-lineinfo`` for ncu source mapping,
``-fmad=false`` (no contraction anywhere; the fp64 path also uses explicit
``__d*_rn`` intrinsics), static cudart, NCCL for the multi-GPU allreduce.
"""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libproclus.so")
SOURCES = ["proclus_kernels.cu", "proclus_api.cu"]
HEADERS = ["proclus_device.cuh", "proclus_kernels.h"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17", "-fmad=false",
    "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
    "-shared", "-cudart", "static",
]


def _inputs():
    files = [os.path.join(CSRC, f) for f in SOURCES + HEADERS]
    files.append(os.path.join(HERE, "..", "include", "proclus.h"))
    return files


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(f) > t for f in _inputs())


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not needs_build():
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    extra = os.environ.get("PROCLUS_NVCC_EXTRA", "").split()
    cmd = [NVCC, *FLAGS, *extra, "-o", tmp, *[os.path.join(CSRC, s) for s in SOURCES], "-lnccl"]
    if verbose:
        print(" ".join(cmd))
    subprocess.check_call(cmd, cwd=CSRC)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True))
