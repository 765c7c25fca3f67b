"""CPU oracle for vbatched DPOTRF — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package. The product package
(``paper_conf_ipps_abdelfattahhtd16_b200``) never imports it and shares no code with it.

Thin ctypes wrapper over ``oracle/liboracle.so`` (built from ``oracle/oracle.c`` by
``__graft_entry__.build()``); see ``oracle.c`` for the paper passages each routine follows,
plus the numpy-only helpers used by the parity gates (row-scaled difference, SURVEY.md
§8(c) reading #14). Parity status of every function is recorded in DESIGN.md §3.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")
SRC_PATH = os.path.join(_HERE, "oracle.c")

_dp = ctypes.POINTER(ctypes.c_double)
_ip = ctypes.POINTER(ctypes.c_int)


def build(force: bool = False) -> str:
    """Compile liboracle.so (no FMA contraction, no fast-math, OpenMP)."""
    if force or not os.path.exists(LIB_PATH) or os.path.getmtime(LIB_PATH) < os.path.getmtime(SRC_PATH):
        cmd = ["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-shared", "-fPIC",
               "-o", LIB_PATH, SRC_PATH, "-lm"]
        subprocess.check_call(cmd)
    return LIB_PATH


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB_PATH)
        L.oracle_dpotrf_lower.argtypes = [ctypes.c_int, _dp, ctypes.c_int]
        L.oracle_spotrf_lower.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_float), ctypes.c_int]
        L.oracle_spotrf_lower.restype = ctypes.c_int
        L.oracle_dpotrf_lower.restype = ctypes.c_int
        L.oracle_dpotrf_batch.argtypes = [ctypes.c_int, _ip, ctypes.POINTER(_dp), _ip, _ip, ctypes.c_int]
        L.oracle_dpotrf_batch.restype = None
        L.oracle_max_threads.argtypes = []
        L.oracle_max_threads.restype = ctypes.c_int
        L.oracle_dgemm.argtypes = [ctypes.c_char, ctypes.c_char, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                   ctypes.c_double, _dp, ctypes.c_int, _dp, ctypes.c_int, ctypes.c_double,
                                   _dp, ctypes.c_int]
        L.oracle_dsyrk.argtypes = [ctypes.c_char, ctypes.c_char, ctypes.c_int, ctypes.c_int, ctypes.c_double,
                                   _dp, ctypes.c_int, ctypes.c_double, _dp, ctypes.c_int]
        L.oracle_dtrsm.argtypes = [ctypes.c_char, ctypes.c_char, ctypes.c_char, ctypes.c_char, ctypes.c_int,
                                   ctypes.c_int, ctypes.c_double, _dp, ctypes.c_int, _dp, ctypes.c_int]
        L.oracle_backward_error.argtypes = [ctypes.c_int, _dp, ctypes.c_int, _dp, ctypes.c_int, ctypes.c_int]
        L.oracle_backward_error.restype = ctypes.c_double
        L.oracle_dgetrf.argtypes = [ctypes.c_int, ctypes.c_int, _dp, ctypes.c_int, _ip]
        L.oracle_dgetrf.restype = ctypes.c_int
        L.oracle_getrf_backward_error.argtypes = [ctypes.c_int, ctypes.c_int, _dp, ctypes.c_int, _dp,
                                                  ctypes.c_int, _ip]
        L.oracle_getrf_backward_error.restype = ctypes.c_double
        L.oracle_zpotrf_lower.argtypes = [ctypes.c_int, _dp, ctypes.c_int]
        L.oracle_zpotrf_lower.restype = ctypes.c_int
        L.oracle_cpotrf_lower.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_float), ctypes.c_int]
        L.oracle_cpotrf_lower.restype = ctypes.c_int
        L.oracle_zpotrf_backward_error.argtypes = [ctypes.c_int, _dp, ctypes.c_int, _dp, ctypes.c_int,
                                                   ctypes.c_int]
        L.oracle_zpotrf_backward_error.restype = ctypes.c_double
        L.oracle_dgeqrf.argtypes = [ctypes.c_int, ctypes.c_int, _dp, ctypes.c_int, _dp]
        L.oracle_dgeqrf.restype = None
        L.oracle_geqrf_errors.argtypes = [ctypes.c_int, ctypes.c_int, _dp, ctypes.c_int, _dp, ctypes.c_int,
                                          _dp, _dp, _dp]
        L.oracle_geqrf_errors.restype = None
        L.oracle_backward_error_batch.argtypes = [ctypes.c_int, _ip, ctypes.POINTER(_dp), _ip,
                                                  ctypes.POINTER(_dp), _ip, _ip, _dp, ctypes.c_int]
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(_dp)


def _fortran_block(a: np.ndarray) -> tuple[np.ndarray, int]:
    """Return (array, ld) for a Fortran-ordered 2-D float64 array (a view, not a copy)."""
    assert a.dtype == np.float64 and a.ndim == 2
    if not a.flags.f_contiguous:
        raise ValueError("expected a Fortran-ordered float64 array")
    return a, max(1, a.shape[0])


def dpotrf(a: np.ndarray) -> tuple[np.ndarray, int]:
    """Oracle Cholesky of one matrix. `a` is n x n (only its lower triangle is read).
    Returns (copy of a with L in the lower triangle, info)."""
    out = np.array(a, dtype=np.float64, order="F", copy=True)
    n = out.shape[0]
    assert out.shape == (n, n)
    info = lib().oracle_dpotrf_lower(n, _ptr(out), max(1, n))
    return out, info


def spotrf(a: np.ndarray) -> tuple[np.ndarray, int]:
    """Oracle Cholesky of one FP32 matrix (float arithmetic, same recurrence as dpotrf)."""
    out = np.array(a, dtype=np.float32, order="F", copy=True)
    n = out.shape[0]
    assert out.shape == (n, n)
    info = lib().oracle_spotrf_lower(n, out.ctypes.data_as(ctypes.POINTER(ctypes.c_float)), max(1, n))
    return out, info


def backward_error_f32(A0: np.ndarray, L: np.ndarray, info: int) -> float:
    """||A - L L^T||_F / (nb ||A||_F eps32), eps32 = 2^-24, long double (the FP32 reading of
    SURVEY.md §8(c) #13)."""
    return backward_error(np.asarray(A0, np.float64), np.asarray(L, np.float64), info) * 2.0 ** -29


def dpotrf_inplace(buf: np.ndarray, n: int, ld: int) -> int:
    """Factor the n x n matrix stored column-major with leading dim ld in the flat float64
    buffer `buf` (in place)."""
    assert buf.dtype == np.float64 and buf.flags.c_contiguous
    return lib().oracle_dpotrf_lower(n, _ptr(buf), ld)


def dpotrf_batch(arena: np.ndarray, offsets, n, ld, nthreads: int = 0) -> np.ndarray:
    """Factor a vbatched arena in place (OpenMP dynamic, one matrix per core).
    arena: flat float64 array; offsets: element offsets of each matrix."""
    n = np.ascontiguousarray(n, dtype=np.int32)
    ld = np.ascontiguousarray(ld, dtype=np.int32)
    B = len(n)
    base = arena.ctypes.data
    ptrs = (_dp * max(B, 1))(*[ctypes.cast(base + 8 * int(o), _dp) for o in offsets])
    info = np.zeros(B, dtype=np.int32)
    lib().oracle_dpotrf_batch(B, n.ctypes.data_as(_ip), ptrs, ld.ctypes.data_as(_ip),
                              info.ctypes.data_as(_ip), int(nthreads))
    return info


def max_threads() -> int:
    return lib().oracle_max_threads()


def dgemm(ta, tb, alpha, A, B, beta, C):
    C = np.array(C, dtype=np.float64, order="F", copy=True)
    A = np.asfortranarray(A, dtype=np.float64)
    B = np.asfortranarray(B, dtype=np.float64)
    m, n = C.shape
    k = A.shape[1] if ta == "N" else A.shape[0]
    lib().oracle_dgemm(ta.encode(), tb.encode(), m, n, k, alpha, _ptr(A), max(1, A.shape[0]),
                       _ptr(B), max(1, B.shape[0]), beta, _ptr(C), max(1, m))
    return C


def dsyrk(uplo, trans, alpha, A, beta, C):
    C = np.array(C, dtype=np.float64, order="F", copy=True)
    A = np.asfortranarray(A, dtype=np.float64)
    n = C.shape[0]
    k = A.shape[1] if trans == "N" else A.shape[0]
    lib().oracle_dsyrk(uplo.encode(), trans.encode(), n, k, alpha, _ptr(A), max(1, A.shape[0]), beta,
                       _ptr(C), max(1, n))
    return C


def dtrsm(side, uplo, transA, diag, alpha, A, B):
    B = np.array(B, dtype=np.float64, order="F", copy=True)
    A = np.asfortranarray(A, dtype=np.float64)
    m, n = B.shape
    lib().oracle_dtrsm(side.encode(), uplo.encode(), transA.encode(), diag.encode(), m, n, alpha,
                       _ptr(A), max(1, A.shape[0]), _ptr(B), max(1, m))
    return B


def dpotrs(uplo, F, B):
    """Solve A X = B from the Cholesky factor F of A, step by step as LAPACK DPOTRS defines it
    (SURVEY.md §8(f) NEXT-4): 'L' (F = L, A = L L^T): L Y = B, then L^T X = Y; 'U' (F = U,
    A = U^T U): U^T Y = B, then U X = Y. Each step is the oracle's plain triangular solve."""
    if uplo == "L":
        Y = dtrsm("L", "L", "N", "N", 1.0, F, B)
        return dtrsm("L", "L", "T", "N", 1.0, F, Y)
    Y = dtrsm("L", "U", "T", "N", 1.0, F, B)
    return dtrsm("L", "U", "N", "N", 1.0, F, Y)


def dposv(uplo, A, B):
    """LAPACK DPOSV: factor A (the oracle's unblocked Cholesky of the referenced triangle), then
    dpotrs; on info != 0 B is returned unchanged. Returns (X, F, info)."""
    A = np.asarray(A, dtype=np.float64)
    if uplo == "L":
        L, info = dpotrf(np.asfortranarray(A))
        F = np.tril(L)
    else:
        L, info = dpotrf(np.asfortranarray(A.T))  # U = L^T of the transposed (mirrored) view
        F = np.triu(L.T)
    if info != 0:
        return np.array(B, dtype=np.float64, copy=True), F, info
    return dpotrs(uplo, F, B), F, info


def backward_error(A0: np.ndarray, L: np.ndarray, info: int) -> float:
    """||A - L L^T||_F / (nb ||A||_F eps), eps = 2^-53, long double."""
    A0 = np.asfortranarray(A0, dtype=np.float64)
    L = np.asfortranarray(L, dtype=np.float64)
    n = A0.shape[0]
    return lib().oracle_backward_error(n, _ptr(A0), max(1, n), _ptr(L), max(1, L.shape[0]), int(info))


def rowscaled_diff(Lg: np.ndarray, Lo: np.ndarray, nb: int) -> float:
    """max_{i>=j} |Lg_ij - Lo_ij| / ||Lo(i, 0:i)||_2 over the leading nb x nb block
    (SURVEY.md §8(c) reading #14)."""
    if nb <= 0:
        return 0.0
    g = np.tril(np.asarray(Lg)[:nb, :nb])
    o = np.tril(np.asarray(Lo)[:nb, :nb])
    rn = np.sqrt(np.sum(o * o, axis=1))
    rn[rn == 0] = 1.0
    return float(np.max(np.abs(g - o) / rn[:, None]))


def dgetrf(a: np.ndarray) -> tuple[np.ndarray, np.ndarray, int]:
    """Oracle LU with partial pivoting of one m x n matrix (oracle.c: textbook unblocked
    elimination, LAPACK DGETF2 conventions). Returns (factored copy: L strictly below the
    diagonal, U on/above; ipiv (1-based, int32, min(m,n)); info)."""
    out = np.array(a, dtype=np.float64, order="F", copy=True)
    m, n = out.shape
    ipiv = np.zeros(max(1, min(m, n)), dtype=np.int32)
    info = lib().oracle_dgetrf(m, n, _ptr(out), max(1, m), ipiv.ctypes.data_as(_ip))
    return out, ipiv[: min(m, n)], info


def getrf_backward_error(A0: np.ndarray, F: np.ndarray, ipiv: np.ndarray) -> float:
    """||P A - L U||_F / (max(m,n) ||A||_F 2^-53) in long double (L unit lower from F's strict
    lower part, U = F's upper part, P from ipiv applied in order)."""
    A0 = np.asfortranarray(A0, dtype=np.float64)
    F = np.asfortranarray(F, dtype=np.float64)
    m, n = A0.shape
    ip = np.ascontiguousarray(ipiv, dtype=np.int32)
    if ip.size == 0:
        ip = np.zeros(1, np.int32)
    return lib().oracle_getrf_backward_error(m, n, _ptr(A0), max(1, m), _ptr(F), max(1, F.shape[0]),
                                             ip.ctypes.data_as(_ip))


def zpotrf(a: np.ndarray) -> tuple[np.ndarray, int]:
    """Oracle complex Cholesky A = L L^H of one Hermitian matrix (complex128; only its lower
    triangle is read, the diagonal's imaginary part ignored). Returns (copy with L in the lower
    triangle, info)."""
    out = np.array(a, dtype=np.complex128, order="F", copy=True)
    n = out.shape[0]
    info = lib().oracle_zpotrf_lower(n, out.ctypes.data_as(_dp), max(1, n))
    return out, info


def cpotrf(a: np.ndarray) -> tuple[np.ndarray, int]:
    """The same recurrence in IEEE single precision (complex64)."""
    out = np.array(a, dtype=np.complex64, order="F", copy=True)
    n = out.shape[0]
    info = lib().oracle_cpotrf_lower(n, out.ctypes.data_as(ctypes.POINTER(ctypes.c_float)), max(1, n))
    return out, info


def zpotrf_backward_error(A0: np.ndarray, L: np.ndarray, info: int) -> float:
    """||A - L L^H||_F / (nb ||A||_F 2^-53), long double (complex; SURVEY §8(c) #13 extended)."""
    A0 = np.asfortranarray(A0, dtype=np.complex128)
    L = np.asfortranarray(L, dtype=np.complex128)
    n = A0.shape[0]
    return lib().oracle_zpotrf_backward_error(n, A0.ctypes.data_as(_dp), max(1, n), L.ctypes.data_as(_dp),
                                              max(1, L.shape[0]), int(info))


def dgeqrf(a: np.ndarray) -> tuple[np.ndarray, np.ndarray]:
    """Oracle Householder QR (oracle.c: textbook DGEQR2 / DLARFG conventions). Returns (compact
    factor: R on/above the diagonal, v below; tau[min(m,n)])."""
    out = np.array(a, dtype=np.float64, order="F", copy=True)
    m, n = out.shape
    tau = np.zeros(max(1, min(m, n)))
    lib().oracle_dgeqrf(m, n, _ptr(out), max(1, m), _ptr(tau))
    return out, tau[: min(m, n)]


def geqrf_errors(A0: np.ndarray, F: np.ndarray, tau: np.ndarray) -> tuple[float, float]:
    """(||A - QR||_F / (max(m,n) ||A||_F eps), ||Q^T Q - I||_F / (m eps)), long double."""
    A0 = np.asfortranarray(A0, dtype=np.float64)
    F = np.asfortranarray(F, dtype=np.float64)
    m, n = A0.shape
    t = np.ascontiguousarray(tau, dtype=np.float64)
    if t.size == 0:
        t = np.zeros(1)
    b, o = ctypes.c_double(), ctypes.c_double()
    lib().oracle_geqrf_errors(m, n, _ptr(A0), max(1, m), _ptr(F), max(1, F.shape[0]), _ptr(t),
                              ctypes.byref(b), ctypes.byref(o))
    return b.value, o.value
