"""Build the native libraries in-tree (nvcc cross-compiles sm_100a without a GPU).

  libvbatched.so  — the product: CUDA kernels + C ABI (include/vbatched.h)
  vbgen/libvbgen.so — device twin of the seeded input generator (test/bench infrastructure)

Usage: python -m paper_conf_ipps_abdelfattahhtd16_b200.build [--force] [--verbose]
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libvbatched.so")
GEN_SRC = os.path.join(ROOT, "vbgen", "gen.cu")
GEN_LIB = os.path.join(ROOT, "vbgen", "libvbgen.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-shared", "-cudart", "shared",
          "-Xlinker", "-rpath,/usr/local/cuda/lib64"]


def _stale(target: str, sources: list[str]) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(s) > t for s in sources)


def build_lib(force: bool = False, verbose: bool = False) -> str:
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    deps = srcs + glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h")) + \
        [os.path.join(ROOT, "include", "vbatched.h")]
    if force or _stale(LIB, deps):
        cmd = [NVCC, *ARCH, *COMMON, "-I", os.path.join(ROOT, "include"), "-o", LIB, *srcs]
        if verbose:
            cmd.insert(1, "-Xptxas=-v")
        subprocess.check_call(cmd)
    return LIB


def build_gen(force: bool = False) -> str:
    if force or _stale(GEN_LIB, [GEN_SRC]):
        subprocess.check_call([NVCC, *ARCH, *COMMON, "-o", GEN_LIB, GEN_SRC])
    return GEN_LIB


def build_all(force: bool = False, verbose: bool = False) -> None:
    build_lib(force, verbose)
    build_gen(force)


if __name__ == "__main__":
    build_all(force="--force" in sys.argv, verbose="--verbose" in sys.argv)
