"""vbgen — seeded synthetic inputs for vbatched DPOTRF (shared by tests, bench and smoke).

This module holds NONE of the method's arithmetic (no factorisation, no BLAS): it only
draws matrix sizes and fills matrix entries from a counter-based hash, so that the CPU
oracle (``oracle/``) and the CUDA path (``paper_conf_ipps_abdelfattahhtd16_b200``) can be
fed bit-identical inputs without sharing code. The device-side twin of ``f1_matrix`` is
``vbgen/gen.cu`` (same hash, same formula, integer-only until the final scale, so the two
agree bit for bit; pinned by ``tests/test_generator.py``).

Recipes (SURVEY.md §8(c) readings #7-#11, §8(d)):
* sizes: uniform integers in [1, Nmax] inclusive (§IV-B) or Gaussian with
  mean 256 and sd 96 rounded to nearest and clipped to [1, 512] (PAPER.md:885-892 fixes the
  mean at Nmax/2; BASELINE.json fixes sd=96). One fresh ``numpy.random.default_rng(seed)``
  per config, used for nothing else.
* values (family F1): a_ij = a_ji = u(seed, gidx, max(i,j), min(i,j)) in [0,1) for i != j and
  a_ii = u_ii + n  (MAGMA-tester "diag += N" convention; Gershgorin gives lambda_min >= 1).
* non-SPD injection (C4: 5 %): matrices with gidx % 20 == 19 get a_kk <- -a_kk at the 1-based
  k = 1 + splitmix64(splitmix64(seed) ^ gidx ^ 0x5EED) mod n, so the k-th pivot is < -n and
  LAPACK info = k under any rounding.
"""
from __future__ import annotations

import dataclasses

import numpy as np

MASK64 = (1 << 64) - 1
NAN_POISON_BITS = 0x7FF8DEADBEEF0001  # quiet NaN with a payload; written to never-touched slots


@dataclasses.dataclass(frozen=True)
class Config:
    name: str
    batch: int
    dist: str          # "uniform" | "gauss"
    nmax: int
    seed: int
    nonspd_mod: int = 0  # 0 = none; 20 = gidx % 20 == 19 is made non-SPD (5 %)
    desc: str = ""


# BASELINE.json "configs" [0..4]
CONFIGS = {
    "C1": Config("C1", 100, "uniform", 32, 1, 0, "batchCount=100, n uniform in [1,32]"),
    "C2": Config("C2", 3000, "uniform", 128, 2, 0, "batchCount=3000, n uniform in [1,128]"),
    "C3": Config("C3", 3000, "uniform", 512, 3, 0, "batchCount=3000, n uniform in [1,512]"),
    "C4": Config("C4", 2000, "gauss", 512, 4, 20,
                 "batchCount=2000, n Gaussian(256,96) clipped to [1,512], 5% non-SPD"),
    "C5": Config("C5", 40000, "uniform", 1024, 5, 0, "batchCount=40000, n uniform in [1,1024]"),
}


def sizes(cfg: Config | str) -> np.ndarray:
    """Per-matrix sizes n[gidx] (int32) for a config; gidx is the position in this array."""
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    rng = np.random.default_rng(cfg.seed)
    if cfg.dist == "uniform":
        n = rng.integers(1, cfg.nmax + 1, cfg.batch)
    elif cfg.dist == "gauss":
        n = np.clip(np.rint(rng.normal(256, 96, cfg.batch)), 1, 512)
    else:
        raise ValueError(cfg.dist)
    return n.astype(np.int32)


def splitmix64(x):
    """SplitMix64 finaliser on uint64 numpy arrays/scalars (wrapping arithmetic)."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def _u(seed: int, gidx: int, hi, lo):
    key = (np.uint64(gidx) << np.uint64(42)) ^ (np.asarray(hi, np.uint64) << np.uint64(21)) \
        ^ np.asarray(lo, np.uint64)
    h = splitmix64(splitmix64(np.uint64(seed)) ^ key)
    return (h >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def nonspd_k(seed: int, gidx: int, n: int) -> int:
    """1-based index of the negated diagonal entry of a non-SPD matrix."""
    h = splitmix64(splitmix64(np.uint64(seed)) ^ np.uint64(gidx) ^ np.uint64(0x5EED))
    return 1 + int(h % np.uint64(n))


def is_nonspd(cfg: Config, gidx: int) -> bool:
    return cfg.nonspd_mod > 0 and gidx % cfg.nonspd_mod == cfg.nonspd_mod - 1


def f1_matrix(seed: int, gidx: int, n: int, nonspd: bool = False) -> np.ndarray:
    """Full symmetric n x n F1 matrix (float64, Fortran order)."""
    if n == 0:
        return np.zeros((0, 0), order="F")
    i = np.arange(n)[:, None]
    j = np.arange(n)[None, :]
    hi = np.maximum(i, j)
    lo = np.minimum(i, j)
    a = _u(seed, gidx, hi, lo)
    d = np.arange(n)
    a[d, d] = a[d, d] + float(n)
    if nonspd:
        k = nonspd_k(seed, gidx, n) - 1
        a[k, k] = -a[k, k]
    return np.asfortranarray(a)


def f2_matrix(seed: int, gidx: int, n: int, kappa: float = 1e4) -> np.ndarray:
    """Family F2 (SURVEY.md §8(c) reading #9, parity only): Q diag(lambda) Q^T with Q the
    orthogonal factor of a seeded Gaussian matrix and lambda log-uniform in [1, kappa]
    (endpoints included, so kappa(A) ~= kappa), symmetrised. Input generation only."""
    if n == 0:
        return np.zeros((0, 0), order="F")
    rng = np.random.default_rng([seed, gidx, n, 0xF2])
    Q, _ = np.linalg.qr(rng.standard_normal((n, n)))
    lam = 10.0 ** rng.uniform(0.0, np.log10(kappa), n)
    lam[0] = 1.0
    if n > 1:
        lam[-1] = kappa
    A = (Q * lam) @ Q.T
    return np.asfortranarray((A + A.T) / 2)


def g1_matrix(seed: int, gidx: int, m: int, n: int) -> np.ndarray:
    """General (non-symmetric) m x n matrix for the LU path: a_ij =
    2 u(seed, gidx, i, j) - 1 in [-1, 1) from the same counter hash, keyed by (i, j) — no
    symmetry. Input generation only."""
    if m == 0 or n == 0:
        return np.zeros((m, n), order="F")
    i = np.arange(m)[:, None] + np.zeros((1, n), np.int64)
    j = np.arange(n)[None, :] + np.zeros((m, 1), np.int64)
    key = (np.uint64(gidx) << np.uint64(42)) ^ (i.astype(np.uint64) << np.uint64(21)) ^ \
        j.astype(np.uint64) ^ np.uint64(0x1 << 63)
    h = splitmix64(splitmix64(np.uint64(seed)) ^ key)
    u = (h >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)
    return np.asfortranarray(2.0 * u - 1.0)


def f1c_matrix(seed: int, gidx: int, n: int, nonspd: bool = False) -> np.ndarray:
    """Complex Hermitian family F1c (complex Cholesky): a_ij = u + i v
    (i > j, u, v from the counter hash keyed by (gidx, i, j) and (gidx, i, j) ^ 2^62), a_ji =
    conj(a_ij), a_ii = u_ii + 2n (real): diagonally dominant (|a_ij| < sqrt 2), so Hermitian PD.
    nonspd negates a_kk at the same hashed k as F1. Input generation only."""
    if n == 0:
        return np.zeros((0, 0), dtype=np.complex128, order="F")
    i = np.arange(n)[:, None] + np.zeros((1, n), np.int64)
    j = np.arange(n)[None, :] + np.zeros((n, 1), np.int64)
    hi, lo = np.maximum(i, j), np.minimum(i, j)
    re = _u(seed, gidx, hi, lo)
    key = (np.uint64(gidx) << np.uint64(42)) ^ (hi.astype(np.uint64) << np.uint64(21)) ^ \
        lo.astype(np.uint64) ^ np.uint64(1 << 62)
    im = (splitmix64(splitmix64(np.uint64(seed)) ^ key) >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
    im = np.where(i > j, im, -im)
    a = re + 1j * im
    d = np.arange(n)
    a[d, d] = re[d, d] + 2.0 * n
    if nonspd:
        k = nonspd_k(seed, gidx, n) - 1
        a[k, k] = -a[k, k]
    return np.asfortranarray(a)


def config_matrix(cfg: Config | str, gidx: int, n: int | None = None) -> np.ndarray:
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    if n is None:
        n = int(sizes(cfg)[gidx])
    return f1_matrix(cfg.seed, gidx, n, is_nonspd(cfg, gidx))


def expected_flops(n: np.ndarray) -> float:
    """Headline flop count: sum of n^3/3 (BASELINE.json metric; SURVEY §8(c) reading #6)."""
    n = np.asarray(n, dtype=np.float64)
    return float(np.sum(n ** 3) / 3.0)


def algorithmic_bytes(n: np.ndarray) -> float:
    """Lower triangle read once + written once: 8*n*(n+1) bytes per matrix."""
    n = np.asarray(n, dtype=np.float64)
    return float(np.sum(8.0 * n * (n + 1)))


def ldda_for(n: np.ndarray, mode: str = "pad32") -> np.ndarray:
    """Leading dimensions: 'pad32' = roundup(n,32) (MAGMA-tester convention), 'tight' = max(1,n)."""
    n = np.asarray(n, dtype=np.int64)
    if mode == "pad32":
        return np.maximum(32, (n + 31) // 32 * 32).astype(np.int32)
    if mode == "tight":
        return np.maximum(1, n).astype(np.int32)
    if mode == "odd":  # smallest odd ldda >= max(1,n): defeats 16-byte alignment of columns
        m = np.maximum(1, n)
        return (m + (m % 2 == 0)).astype(np.int32)
    raise ValueError(mode)


def arena_layout(n: np.ndarray, ldda: np.ndarray, align_bytes: int = 256, elem_bytes: int = 8):
    """Element offsets of each matrix in one arena (each base `align_bytes`-aligned) and the
    total element count."""
    sz = ldda.astype(np.int64) * np.maximum(n.astype(np.int64), 0)
    al = align_bytes // elem_bytes
    sz_al = (sz + al - 1) // al * al
    off = np.zeros(len(n), dtype=np.int64)
    if len(n) > 1:
        off[1:] = np.cumsum(sz_al)[:-1]
    total = int(sz_al.sum()) if len(n) else 0
    return off, max(total, 1)
