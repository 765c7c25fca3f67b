"""paper_conf_ipps_abdelfattahhtd16_b200 — B200-native variable-size batched Cholesky.

Thin Python binding over the C ABI of ``libvbatched.so`` (``include/vbatched.h``): argument
marshalling only. Every arithmetic step runs in the library's CUDA kernels (sm_100a);
there is no CPU fallback — if the shared library is missing or cannot load, importing the
functions raises.

Arguments that the C ABI takes as device pointers accept either an int (raw address) or a
torch CUDA tensor of the right dtype (int32 for sizes/info, int64 for pointer arrays,
float64 for matrices, float32 for vbatched_spotrf). ``stream`` accepts None (torch's current stream), a
``torch.cuda.Stream`` or a raw handle.
"""
from __future__ import annotations

import ctypes
import os

__all__ = [
    "vbatched_dpotrf", "vbatched_dpotrf_nomax", "vbatched_dpotrf_host",
    "vbatched_dpotrf_workspace_size", "vbatched_dpotrf_scan", "vbatched_dpotrf_factor", "vbatched_dgemm",
    "vbatched_dsyrk", "vbatched_dtrsm", "vbatched_partition_lpt", "vbatched_version",
    "vbatched_host_alloc", "vbatched_host_free", "vbatched_dpotrf_kernel_launches", "vbatched_dpotrf_kernel_names",
    "vbatched_release_host_staging", "factor_kernel_names", "vbatched_dgetrf", "vbatched_dgeqrf", "vbatched_zpotrf", "vbatched_cpotrf", "lib", "LIB_PATH", "VBatchedError",
]

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("VBATCHED_LIB", os.path.join(_HERE, "libvbatched.so"))

_vp = ctypes.c_void_p
_i = ctypes.c_int
_c = ctypes.c_char
_d = ctypes.c_double

_lib = None


class VBatchedError(RuntimeError):
    pass


def lib() -> ctypes.CDLL:
    """Load libvbatched.so (raises if it was not built: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise VBatchedError(f"{LIB_PATH} not built; run __graft_entry__.build() or "
                                "python -m paper_conf_ipps_abdelfattahhtd16_b200.build")
        L = ctypes.CDLL(LIB_PATH)
        L.vbatched_dpotrf.argtypes = [_c, _vp, _vp, _vp, _vp, _i, _i, _vp]
        L.vbatched_dpotrf_nomax.argtypes = [_c, _vp, _vp, _vp, _vp, _i, _vp]
        L.vbatched_spotrf.argtypes = [_c, _vp, _vp, _vp, _vp, _i, _i, _vp]
        L.vbatched_spotrf_nomax.argtypes = [_c, _vp, _vp, _vp, _vp, _i, _vp]
        L.vbatched_dpotrf_workspace_size.argtypes = [_i]
        L.vbatched_dpotrf_workspace_size.restype = ctypes.c_size_t
        L.vbatched_dpotrf_scan.argtypes = [_c, _vp, _vp, _vp, _i, _i, _vp, _vp]
        L.vbatched_dpotrf_factor.argtypes = [_c, _vp, _vp, _vp, _vp, _i, _i, _vp, _vp]
        L.vbatched_dpotrf_host.argtypes = [_c, _vp, _vp, _vp, _vp, _i, _i, ctypes.c_size_t, _vp]
        L.vbatched_dgemm.argtypes = [_c, _c, _vp, _vp, _vp, _d, _vp, _vp, _vp, _vp, _d, _vp, _vp,
                                     _i, _i, _i, _i, _vp]
        L.vbatched_dsyrk.argtypes = [_c, _c, _vp, _vp, _d, _vp, _vp, _d, _vp, _vp, _i, _i, _i, _vp]
        L.vbatched_dtrsm.argtypes = [_c, _c, _c, _c, _vp, _vp, _d, _vp, _vp, _vp, _vp, _i, _i, _i,
                                     _vp]
        L.vbatched_dpotrs.argtypes = [_c, _vp, _vp, _vp, _vp, _vp, _vp, _i, _i, _i, _vp]
        L.vbatched_dposv.argtypes = [_c, _vp, _vp, _vp, _vp, _vp, _vp, _vp, _i, _i, _i, _vp]
        L.vbatched_partition_lpt.argtypes = [_vp, _i, _i, _vp]
        L.vbatched_version.restype = ctypes.c_char_p
        L.vbatched_dpotrf_kernel_launches.argtypes = [_i]
        L.vbatched_dpotrf_kernel_launches.restype = _i
        L.vbatched_dpotrf_kernel_names.argtypes = [_i]
        L.vbatched_dpotrf_kernel_names.restype = ctypes.c_char_p
        L.vbatched_zpotrf.argtypes = [_c, _vp, _vp, _vp, _vp, _i, _i, _vp]
        L.vbatched_cpotrf.argtypes = [_c, _vp, _vp, _vp, _vp, _i, _i, _vp]
        L.vbatched_dgeqrf.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _i, _i, _i, _vp]
        L.vbatched_dgetrf.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _i, _i, _i, _vp]
        L.vbatched_release_host_staging.argtypes = []
        L.vbatched_release_host_staging.restype = _i
        L.vbatched_host_alloc.argtypes = [ctypes.c_size_t]
        L.vbatched_host_alloc.restype = _vp
        L.vbatched_host_free.argtypes = [_vp]
        for name in ("vbatched_dpotrf", "vbatched_dpotrf_nomax", "vbatched_dpotrf_host",
                     "vbatched_spotrf", "vbatched_spotrf_nomax",
                     "vbatched_dpotrf_scan", "vbatched_dpotrf_factor",
                     "vbatched_dgemm", "vbatched_dsyrk", "vbatched_dtrsm",
                     "vbatched_dpotrs", "vbatched_dposv",
                     "vbatched_partition_lpt", "vbatched_host_free"):
            getattr(L, name).restype = _i
        _lib = L
    return _lib


def _ptr(x):
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if hasattr(x, "ctypes"):  # numpy
        return x.ctypes.data
    raise TypeError(f"cannot take a pointer of {type(x)}")


def _stream(s):
    if s is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(s, int):
        return s
    return s.cuda_stream


def _ch(c: str) -> bytes:
    return c.encode() if isinstance(c, str) else c


def _check(rc: int, name: str) -> int:
    if rc != 0:
        raise VBatchedError(f"{name} returned {rc} "
                            f"({'invalid argument #%d' % -rc if rc < 0 else 'CUDA error'})")
    return rc


def vbatched_dpotrf(uplo, n, dA_array, ldda, info, batchCount, max_n, stream=None, check=True):
    rc = lib().vbatched_dpotrf(_ch(uplo), _ptr(n), _ptr(dA_array), _ptr(ldda), _ptr(info),
                               int(batchCount), int(max_n), _stream(stream))
    return _check(rc, "vbatched_dpotrf") if check else rc


def vbatched_spotrf(uplo, n, dA_array, ldda, info, batchCount, max_n, stream=None, check=True):
    rc = lib().vbatched_spotrf(_ch(uplo), _ptr(n), _ptr(dA_array), _ptr(ldda), _ptr(info),
                               int(batchCount), int(max_n), _stream(stream))
    return _check(rc, "vbatched_spotrf") if check else rc


def vbatched_spotrf_nomax(uplo, n, dA_array, ldda, info, batchCount, stream=None, check=True):
    rc = lib().vbatched_spotrf_nomax(_ch(uplo), _ptr(n), _ptr(dA_array), _ptr(ldda), _ptr(info),
                                     int(batchCount), _stream(stream))
    return _check(rc, "vbatched_spotrf_nomax") if check else rc


def vbatched_dpotrf_nomax(uplo, n, dA_array, ldda, info, batchCount, stream=None, check=True):
    rc = lib().vbatched_dpotrf_nomax(_ch(uplo), _ptr(n), _ptr(dA_array), _ptr(ldda), _ptr(info),
                                     int(batchCount), _stream(stream))
    return _check(rc, "vbatched_dpotrf_nomax") if check else rc


def vbatched_dpotrf_workspace_size(batchCount) -> int:
    return int(lib().vbatched_dpotrf_workspace_size(int(batchCount)))


def vbatched_dpotrf_scan(uplo, n, ldda, info, batchCount, max_n, d_workspace, stream=None,
                         check=True):
    rc = lib().vbatched_dpotrf_scan(_ch(uplo), _ptr(n), _ptr(ldda), _ptr(info), int(batchCount),
                                    int(max_n), _ptr(d_workspace), _stream(stream))
    return _check(rc, "vbatched_dpotrf_scan") if check else rc


def vbatched_dpotrf_factor(uplo, n, dA_array, ldda, info, batchCount, max_n, d_workspace,
                           stream=None, check=True):
    rc = lib().vbatched_dpotrf_factor(_ch(uplo), _ptr(n), _ptr(dA_array), _ptr(ldda), _ptr(info),
                                      int(batchCount), int(max_n), _ptr(d_workspace),
                                      _stream(stream))
    return _check(rc, "vbatched_dpotrf_factor") if check else rc


def vbatched_dpotrf_host(uplo, h_n, hA_array, h_ldda, h_info, batchCount, max_n,
                         workspace_bytes=0, stream=0, check=True):
    """Host-memory variant (blocking). h_* are numpy arrays / host addresses."""
    rc = lib().vbatched_dpotrf_host(_ch(uplo), _ptr(h_n), _ptr(hA_array), _ptr(h_ldda),
                                    _ptr(h_info), int(batchCount), int(max_n),
                                    int(workspace_bytes), stream if isinstance(stream, int) else _stream(stream))
    return _check(rc, "vbatched_dpotrf_host") if check else rc


def vbatched_dgemm(transA, transB, m, n, k, alpha, dA_array, ldda, dB_array, lddb, beta,
                   dC_array, lddc, batchCount, max_m, max_n, max_k, stream=None, check=True):
    rc = lib().vbatched_dgemm(_ch(transA), _ch(transB), _ptr(m), _ptr(n), _ptr(k), float(alpha),
                              _ptr(dA_array), _ptr(ldda), _ptr(dB_array), _ptr(lddb), float(beta),
                              _ptr(dC_array), _ptr(lddc), int(batchCount), int(max_m), int(max_n),
                              int(max_k), _stream(stream))
    return _check(rc, "vbatched_dgemm") if check else rc


def vbatched_dsyrk(uplo, trans, n, k, alpha, dA_array, ldda, beta, dC_array, lddc, batchCount,
                   max_n, max_k, stream=None, check=True):
    rc = lib().vbatched_dsyrk(_ch(uplo), _ch(trans), _ptr(n), _ptr(k), float(alpha),
                              _ptr(dA_array), _ptr(ldda), float(beta), _ptr(dC_array), _ptr(lddc),
                              int(batchCount), int(max_n), int(max_k), _stream(stream))
    return _check(rc, "vbatched_dsyrk") if check else rc


def vbatched_dtrsm(side, uplo, transA, diag, m, n, alpha, dA_array, ldda, dB_array, lddb,
                   batchCount, max_m, max_n, stream=None, check=True):
    rc = lib().vbatched_dtrsm(_ch(side), _ch(uplo), _ch(transA), _ch(diag), _ptr(m), _ptr(n),
                              float(alpha), _ptr(dA_array), _ptr(ldda), _ptr(dB_array), _ptr(lddb),
                              int(batchCount), int(max_m), int(max_n), _stream(stream))
    return _check(rc, "vbatched_dtrsm") if check else rc


def vbatched_dpotrs(uplo, n, nrhs, dA_array, ldda, dB_array, lddb, batchCount, max_n, max_nrhs,
                    stream=None, check=True):
    rc = lib().vbatched_dpotrs(_ch(uplo), _ptr(n), _ptr(nrhs), _ptr(dA_array), _ptr(ldda),
                               _ptr(dB_array), _ptr(lddb), int(batchCount), int(max_n),
                               int(max_nrhs), _stream(stream))
    return _check(rc, "vbatched_dpotrs") if check else rc


def vbatched_dposv(uplo, n, nrhs, dA_array, ldda, dB_array, lddb, info, batchCount, max_n,
                   max_nrhs, stream=None, check=True):
    rc = lib().vbatched_dposv(_ch(uplo), _ptr(n), _ptr(nrhs), _ptr(dA_array), _ptr(ldda),
                              _ptr(dB_array), _ptr(lddb), _ptr(info), int(batchCount), int(max_n),
                              int(max_nrhs), _stream(stream))
    return _check(rc, "vbatched_dposv") if check else rc


def vbatched_zpotrf(uplo, n, dA_array, ldda, info, batchCount, max_n, stream=None, check=True):
    """vbatched complex<double> Cholesky (include/vbatched.h): matrices as complex128 tensors'
    addresses in dA_array (int64 device pointers)."""
    rc = lib().vbatched_zpotrf(_ch(uplo), _ptr(n), _ptr(dA_array), _ptr(ldda), _ptr(info),
                               int(batchCount), int(max_n), _stream(stream))
    return _check(rc, "vbatched_zpotrf") if check else rc


def vbatched_cpotrf(uplo, n, dA_array, ldda, info, batchCount, max_n, stream=None, check=True):
    """vbatched complex<float> Cholesky (FP32 storage, FP64 arithmetic)."""
    rc = lib().vbatched_cpotrf(_ch(uplo), _ptr(n), _ptr(dA_array), _ptr(ldda), _ptr(info),
                               int(batchCount), int(max_n), _stream(stream))
    return _check(rc, "vbatched_cpotrf") if check else rc


def vbatched_dgeqrf(m, n, dA_array, ldda, dtau_array, info, batchCount, max_m, max_n, stream=None,
                    check=True):
    """vbatched Householder QR (include/vbatched.h): device arrays m, n, ldda, info (int32),
    dA_array / dtau_array (int64 device pointers to the matrices / tau vectors)."""
    rc = lib().vbatched_dgeqrf(_ptr(m), _ptr(n), _ptr(dA_array), _ptr(ldda), _ptr(dtau_array),
                               _ptr(info), int(batchCount), int(max_m), int(max_n), _stream(stream))
    return _check(rc, "vbatched_dgeqrf") if check else rc


def vbatched_dgetrf(m, n, dA_array, ldda, dipiv_array, info, batchCount, max_m, max_n, stream=None,
                    check=True):
    """vbatched LU with partial pivoting (include/vbatched.h): device arrays m, n, ldda, info
    (int32), dA_array / dipiv_array (int64 device pointers)."""
    rc = lib().vbatched_dgetrf(_ptr(m), _ptr(n), _ptr(dA_array), _ptr(ldda), _ptr(dipiv_array),
                               _ptr(info), int(batchCount), int(max_m), int(max_n), _stream(stream))
    return _check(rc, "vbatched_dgetrf") if check else rc


def vbatched_partition_lpt(h_n, ngpu: int):
    """Returns owner[i] (numpy int32) — LPT on n^3/3 (pure host)."""
    import numpy as np
    h_n = np.ascontiguousarray(h_n, dtype=np.int32)
    owner = np.empty(len(h_n), dtype=np.int32)
    _check(lib().vbatched_partition_lpt(_ptr(h_n), len(h_n), int(ngpu), _ptr(owner)),
           "vbatched_partition_lpt")
    return owner


def vbatched_dpotrf_kernel_launches(max_n: int) -> int:
    return int(lib().vbatched_dpotrf_kernel_launches(int(max_n)))


def vbatched_dpotrf_kernel_names(max_n: int) -> str:
    return lib().vbatched_dpotrf_kernel_names(int(max_n)).decode()


factor_kernel_names = vbatched_dpotrf_kernel_names


def vbatched_release_host_staging() -> None:
    _check(lib().vbatched_release_host_staging(), "vbatched_release_host_staging")


def vbatched_version() -> str:
    return lib().vbatched_version().decode()


def vbatched_host_alloc(nbytes: int) -> int:
    p = lib().vbatched_host_alloc(int(nbytes))
    if not p:
        raise VBatchedError(f"cudaHostAlloc({nbytes}) failed")
    return p


def vbatched_host_free(p: int) -> None:
    _check(lib().vbatched_host_free(p), "vbatched_host_free")
