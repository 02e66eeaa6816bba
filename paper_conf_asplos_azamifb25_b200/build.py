"""Build liblcf.so (the C-ABI library) for sm_100a with nvcc, in-tree."""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
LIB = os.path.join(PKG, "liblcf.so")
CPU_LIB = os.path.join(PKG, "liblcf_cpu.so")  # the multi-threaded CPU codec (NEXT-2), a separate library
CPU_SRC = os.path.join(PKG, "cpu", "lcf_cpu.cpp")
CXX_FLAGS = ["-O3", "-std=c++17", "-fPIC", "-shared", "-pthread", "-Wall", "-Wextra"]
NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
              "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall", "-shared"]


def sources():
    return sorted(glob.glob(os.path.join(PKG, "csrc", "*.cu")))


def headers():
    return sorted(glob.glob(os.path.join(PKG, "csrc", "*.cuh")) + [os.path.join(ROOT, "include", "lcf.h")])


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(p) > t for p in sources() + headers())


def build_cpu(force: bool = False) -> str:
    """liblcf_cpu.so: plain g++ (baseline x86-64 ISA: the .so travels to other hosts)."""
    hdr = os.path.join(ROOT, "include", "lcf_cpu.h")
    if not force and os.path.exists(CPU_LIB) and os.path.getmtime(CPU_LIB) > max(
            os.path.getmtime(CPU_SRC), os.path.getmtime(hdr)):
        return CPU_LIB
    tmp = CPU_LIB + f".tmp{os.getpid()}"
    subprocess.check_call([os.environ.get("CXX", "g++"), *CXX_FLAGS, "-I", os.path.join(ROOT, "include"), "-o", tmp,
                           CPU_SRC])
    os.replace(tmp, CPU_LIB)
    return CPU_LIB


def build(force: bool = False, verbose: bool = False) -> str:
    build_cpu(force)
    if not force and not stale():
        return LIB
    nvcc = os.environ.get("NVCC", "nvcc")
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [nvcc, *NVCC_FLAGS, "-I", os.path.join(ROOT, "include"), "-o", tmp, *sources()]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
