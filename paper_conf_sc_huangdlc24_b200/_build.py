"""Build libcszp2.so in-tree with nvcc for sm_100a (no JIT cache, no torch ext)."""
from __future__ import annotations

import glob
import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libcszp2.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC", "-shared",
    "-I", os.path.join(ROOT, "include"),
]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cuh"))
                  + glob.glob(os.path.join(CSRC, "*.cpp"))
                  + [os.path.join(ROOT, "include", "cszp2.h")])


def build(force: bool = False, verbose: bool = False) -> str:
    srcs = sources()
    if not force and os.path.exists(LIB) and os.path.getmtime(LIB) >= max(map(os.path.getmtime, srcs)):
        return LIB
    cmd = [NVCC, *NVCC_FLAGS, "-o", LIB + ".tmp", os.path.join(CSRC, "cszp2_api.cu")]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    subprocess.check_call(cmd)
    os.replace(LIB + ".tmp", LIB)
    build_cli()
    return LIB


CLI = os.path.join(PKG, "cszp2")


def build_cli() -> str:
    """The `cszp2` command-line tool (csrc/cszp2_cli.cpp): host C++ over the C ABI,
    linked against the in-tree libcszp2.so (rpath $ORIGIN) and cudart."""
    cuda = os.path.dirname(os.path.dirname(os.path.realpath(NVCC)))
    cmd = ["g++", "-O2", "-std=c++17", "-I", os.path.join(ROOT, "include"), "-I", os.path.join(cuda, "include"),
           "-o", CLI + ".tmp", os.path.join(CSRC, "cszp2_cli.cpp"), "-L", PKG, "-lcszp2",
           "-L", os.path.join(cuda, "lib64"), "-lcudart", "-Wl,-rpath,$ORIGIN"]
    subprocess.check_call(cmd)
    os.replace(CLI + ".tmp", CLI)
    return CLI


if __name__ == "__main__":
    print(build(force=True, verbose=True))
