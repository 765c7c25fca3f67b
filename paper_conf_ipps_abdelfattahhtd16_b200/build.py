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
from concurrent.futures import ThreadPoolExecutor

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
        # one object per translation unit, compiled in parallel (whole-program device code stays
        # per file: no relocatable device code, the units share only inline headers), then linked
        objdir = os.path.join(PKG, "build")
        os.makedirs(objdir, exist_ok=True)
        cflags = [f for f in COMMON if f not in ("-shared",)]
        inc = ["-I", os.path.join(ROOT, "include")]
        hdrs = [d for d in deps if not d.endswith(".cu")]

        def compile_one(src: str) -> str:
            obj = os.path.join(objdir, os.path.basename(src)[:-3] + ".o")
            if force or _stale(obj, [src, *hdrs]):
                cmd = [NVCC, *ARCH, *cflags, *inc, "-c", src, "-o", obj]
                if verbose:
                    cmd.insert(1, "-Xptxas=-v")
                subprocess.check_call(cmd)
            return obj

        with ThreadPoolExecutor(max_workers=min(len(srcs), os.cpu_count() or 1)) as ex:
            objs = list(ex.map(compile_one, srcs))
        subprocess.check_call([NVCC, *ARCH, *COMMON, "-o", LIB, *objs])
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
