"""Builds libhirace.so in-tree for sm_100a (nvcc cross-compiles without a GPU).

    python -m paper_conf_sc_jacobsonbg24_b200.build [--verbose]
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIBDIR = os.path.join(PKG, "lib")
SO = os.path.join(LIBDIR, "libhirace.so")
EXDIR = os.path.join(PKG, "examples")
EXSO = os.path.join(LIBDIR, "libhirace_examples.so")
EXSO_AGG = os.path.join(LIBDIR, "libhirace_examples_agg.so")  # inline hooks with warp aggregation
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def headers():
    return sorted(glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) +
                  glob.glob(os.path.join(INCLUDE, "*")))


def ex_sources():
    return sorted(glob.glob(os.path.join(EXDIR, "*.cu")))


def stale(so, srcs) -> bool:
    if not os.path.exists(so):
        return True
    t = os.path.getmtime(so)
    return any(os.path.getmtime(p) > t for p in srcs + headers())


def _nvcc(so, srcs, verbose, defines=()):
    cmd = [NVCC, *ARCH, "-lineinfo", "-O3", "-std=c++17", "-Xcompiler", "-fPIC,-O2", "-shared",
           *[f"-D{d}" for d in defines], "-I", INCLUDE, "-I", CSRC, "-o", so + ".tmp", *srcs]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    subprocess.check_call(cmd)
    os.replace(so + ".tmp", so)


def build(force: bool = False, verbose: bool = False) -> str:
    """libhirace.so (the checker) and libhirace_examples.so (native programs checked inline)."""
    os.makedirs(LIBDIR, exist_ok=True)
    if force or stale(SO, sources()):
        _nvcc(SO, sources(), verbose)
    if force or stale(EXSO, ex_sources()):
        _nvcc(EXSO, ex_sources(), verbose)
    if force or stale(EXSO_AGG, ex_sources()):
        _nvcc(EXSO_AGG, ex_sources(), verbose, defines=("HIRACE_INLINE_AGGREGATE=1",))
    return SO


if __name__ == "__main__":
    print(build(force=True, verbose="--verbose" in sys.argv))
