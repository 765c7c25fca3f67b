"""CPU library baseline (bench.py only): LAPACK dpotrf one core per matrix — the paper's best
CPU competitor ("MKL, one core per matrix"), run on the bench
host's cores. MKL is the copy inside libtorch_cpu.so (LP64 `dpotrf_`); see lapack_batch.c.
Neither the product package nor the oracle uses this module."""
from __future__ import annotations

import ctypes
import os
import subprocess
import time

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liblapack_batch.so")
SRC_PATH = os.path.join(_HERE, "lapack_batch.c")


def build(force: bool = False) -> str:
    if force or not os.path.exists(LIB_PATH) or os.path.getmtime(LIB_PATH) < os.path.getmtime(SRC_PATH):
        subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-pthread", "-o", LIB_PATH,
                               SRC_PATH, "-ldl"])
    return LIB_PATH


def mkl_path() -> str:
    import torch
    return os.path.join(os.path.dirname(torch.__file__), "lib", "libtorch_cpu.so")


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.lapack_batch_dpotrf.restype = ctypes.c_int
        _lib.lapack_batch_is_mkl.restype = ctypes.c_int
    return _lib


def dpotrf_batch(arena: np.ndarray, offsets, n, ld, nthreads: int, lib_path: str | None = None):
    """Factor the matrices of a flat float64 arena in place with sequential LAPACK dpotrf,
    `nthreads` threads pulling matrices in LPT order (n descending). Returns (seconds, info)."""
    lib_path = lib_path or mkl_path()
    n = np.ascontiguousarray(n, dtype=np.int32)
    ld = np.ascontiguousarray(ld, dtype=np.int32)
    B = len(n)
    base = arena.ctypes.data
    ptrs = (ctypes.c_void_p * max(B, 1))(*[base + 8 * int(o) for o in offsets])
    order = np.ascontiguousarray(np.argsort(-n, kind="stable"), dtype=np.int32)
    info = np.zeros(B, dtype=np.int32)
    ip = ctypes.POINTER(ctypes.c_int)
    t0 = time.perf_counter()
    rc = lib().lapack_batch_dpotrf(lib_path.encode(), ptrs, n.ctypes.data_as(ip),
                                   ld.ctypes.data_as(ip), info.ctypes.data_as(ip),
                                   order.ctypes.data_as(ip), B, int(nthreads))
    dt = time.perf_counter() - t0
    if rc != 0:
        raise RuntimeError(f"lapack_batch_dpotrf failed ({rc}) with {lib_path}")
    return dt, info


def openblas_path() -> str | None:
    """scipy's bundled OpenBLAS (LP64 `scipy_dpotrf_`), the secondary CPU baseline."""
    import glob
    import scipy
    libs = glob.glob(os.path.join(os.path.dirname(os.path.dirname(scipy.__file__)), "scipy.libs",
                                  "libscipy_openblas-*.so"))
    return libs[0] if libs else None


def is_mkl(lib_path: str | None = None) -> bool:
    return bool(lib().lapack_batch_is_mkl((lib_path or mkl_path()).encode()))
