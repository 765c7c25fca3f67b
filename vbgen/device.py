"""ctypes wrapper for vbgen/libvbgen.so (the device twin of vbgen.f1_matrix)."""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libvbgen.so")
_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} not built (python -m paper_conf_ipps_abdelfattahhtd16_b200.build)")
        L = ctypes.CDLL(LIB_PATH)
        v = ctypes.c_void_p
        L.vbgen_fill_f1.argtypes = [ctypes.c_uint64, ctypes.c_int, v, v, v, v, ctypes.c_int,
                                    ctypes.c_int, v]
        L.vbgen_fill_f1.restype = ctypes.c_int
        _lib = L
    return _lib


def fill_f1(seed: int, batch: int, d_n: int, d_ldda: int, d_ptrs: int, d_gidx: int | None,
            nonspd_mod: int, poison: int, stream: int) -> None:
    """poison: bit 0 = NaN sentinels outside the referenced triangle, bit 1 = upper storage."""
    rc = lib().vbgen_fill_f1(int(seed), int(batch), d_n, d_ldda, d_ptrs, d_gidx, int(nonspd_mod),
                             int(poison), stream)
    if rc != 0:
        raise RuntimeError(f"vbgen_fill_f1 failed: cudaError {rc}")
