"""Pins for the CPU oracle (oracle/oracle.c) against things the paper's problem and the
mathematics fix — never against the oracle itself or the CUDA path (CPU only).

PAPER.md prints no numeric worked example and no error bound (its figures are garbled),
so the pins are (SURVEY.md §8(c) "What pins each part"):
  closed forms (min(i,j), Pascal, hand-worked 2x2/3x3 golden fixtures), exact integer
  families (integer unit-lower L, power-of-two diagonals), invariants (det, reconstruction),
  library cross-checks (LAPACK dpotrf via MKL in torch; OpenBLAS via scipy), exact rational
  Sylvester pivots on tiny integer matrices, and LAPACK info conventions.
Each is chosen so a plausible oracle bug (dropped term, wrong sign/index, transposed
operand, info off by one) fails at least one test.
"""
import json
import math
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import vbgen

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _chol(A):
    return oracle.dpotrf(np.asfortranarray(np.asarray(A, dtype=np.float64)))


# ---------------------------------------------------------------- golden / closed forms
def test_handworked_golden():
    g = json.load(open(os.path.join(GOLD, "handworked.json")))
    for case in g["cases"]:
        A = np.array(case["A"], dtype=np.float64)
        L, info = _chol(A)
        assert info == case["info"], case["name"]
        if info == 0:
            Lexp = np.array([[math.sqrt(2.0) if v == "sqrt2" else float(v) for v in row] for row in case["L"]])
            assert np.array_equal(np.tril(L), Lexp), case["name"]  # bit-exact
        else:
            k = info - 1
            lead = np.array(case["L_leading"], dtype=np.float64).reshape(k, k)
            assert np.array_equal(np.tril(L[:k, :k]), lead), case["name"]
            assert L[k, k] == case["pivot"], case["name"]  # LAPACK stores the failing pivot


@pytest.mark.parametrize("n", [1, 2, 3, 7, 32, 33, 100, 200])
def test_min_ij_gives_tril_ones(n):
    i = np.arange(1, n + 1)
    A = np.minimum.outer(i, i).astype(np.float64)
    L, info = _chol(A)
    assert info == 0
    assert np.array_equal(np.tril(L), np.tril(np.ones((n, n))))


@pytest.mark.parametrize("n", [1, 5, 12, 20, 29])
def test_pascal_gives_lower_pascal(n):
    P = np.array([[math.comb(i + j, j) for j in range(n)] for i in range(n)], dtype=np.float64)
    Lp = np.array([[math.comb(i, j) if j <= i else 0 for j in range(n)] for i in range(n)], dtype=np.float64)
    L, info = _chol(P)
    assert info == 0
    assert np.array_equal(np.tril(L), Lp)


def _int_unit_lower(n, rng, diag=None):
    L = np.tril(rng.integers(-1, 2, size=(n, n)), -1).astype(np.int64)
    d = np.ones(n, dtype=np.int64) if diag is None else diag
    L[np.arange(n), np.arange(n)] = d
    return L


@pytest.mark.parametrize("n", [2, 9, 33, 128])
def test_integer_unit_lower_exact(n):
    rng = np.random.default_rng(100 + n)
    L = _int_unit_lower(n, rng)
    A = (L @ L.T).astype(np.float64)  # exact: small integers
    assert np.max(np.abs(L @ L.T)) < 2 ** 53
    Lc, info = _chol(A)
    assert info == 0
    assert np.array_equal(np.tril(Lc), L.astype(np.float64))


def test_integer_pow2_diagonal_exact():
    rng = np.random.default_rng(7)
    n = 64
    L = _int_unit_lower(n, rng, diag=rng.choice([1, 2, 4], size=n))
    A = (L @ L.T).astype(np.float64)
    Lc, info = _chol(A)
    assert info == 0
    assert np.array_equal(np.tril(Lc), L.astype(np.float64))


def test_identity_and_diagonal_and_scalar():
    for n in (1, 4, 50):
        L, info = _chol(np.eye(n))
        assert info == 0 and np.array_equal(np.tril(L), np.eye(n))
    d = 4.0 ** np.arange(10)
    L, info = _chol(np.diag(d))
    assert info == 0 and np.array_equal(np.tril(L), np.diag(2.0 ** np.arange(10)))
    for a in (2.0, 3.0, 1e-300, 7.5e300):
        L, info = _chol([[a]])
        assert info == 0 and L[0, 0] == math.sqrt(a)


def test_upper_triangle_never_read_or_written():
    n = 40
    A = vbgen.f1_matrix(9, 3, n)
    ref, info_ref = _chol(A)
    B = A.copy(order="F")
    iu = np.triu_indices(n, 1)
    B[iu] = np.nan
    L, info = _chol(B)
    assert info == info_ref == 0
    assert np.array_equal(np.tril(L), np.tril(ref))
    assert np.all(np.isnan(L[iu]))


# ---------------------------------------------------------------- info conventions
def test_info_special_cases():
    assert _chol(np.ones((5, 5)))[1] == 2
    assert _chol(np.zeros((3, 3)))[1] == 1
    assert _chol([[-1.0]])[1] == 1
    assert _chol(np.zeros((0, 0)))[1] == 0


@pytest.mark.parametrize("n", [1, 2, 17, 64, 200])
def test_info_negated_diagonal(n):
    for gidx in range(0, 60, 7):
        A = vbgen.f1_matrix(4, gidx, n, nonspd=True)
        k = vbgen.nonspd_k(4, gidx, n)
        L, info = _chol(A)
        assert info == k
        # leading block is the factor of the leading (k-1) block of A
        if k > 1:
            L2, info2 = _chol(A[: k - 1, : k - 1].copy(order="F"))
            assert info2 == 0
            assert np.array_equal(np.tril(L[: k - 1, : k - 1]), np.tril(L2))
        assert L[k - 1, k - 1] < -n  # failing pivot stored (LAPACK dpotf2 convention)


@pytest.mark.parametrize("pos", [(0, 0), (3, 3), (7, 7), (5, 2), (7, 0), (6, 5)])
def test_info_nan_positions(pos):
    """NaN at (k,k) -> info k+1; NaN at (i,j), i>j -> info i+1 (0-based positions);
    matches MKL (LAPACK DISNAN semantics), SURVEY §8(c) reading #2."""
    n = 8
    A = vbgen.f1_matrix(1, 0, n)
    i, j = pos
    A[i, j] = np.nan
    _, info = _chol(A)
    assert info == i + 1


def test_info_nan_matches_mkl():
    import torch
    n = 8
    for (i, j) in [(2, 2), (3, 1), (7, 0)]:
        A = vbgen.f1_matrix(1, 1, n)
        A[i, j] = np.nan
        A[j, i] = np.nan
        _, info_m = torch.linalg.cholesky_ex(torch.from_numpy(A))
        assert _chol(A)[1] == int(info_m)


# ---------------------------------------------------------------- exact rationals (Sylvester)
def _ldl_pivots(A):
    """Exact rational pivots d_k = det(A_k)/det(A_{k-1}) by fraction-exact elimination."""
    n = len(A)
    M = [[Fraction(int(v)) for v in row] for row in A]
    piv = []
    for k in range(n):
        d = M[k][k]
        piv.append(d)
        if d == 0:
            break
        for i in range(k + 1, n):
            f = M[i][k] / d
            for j in range(k, n):
                M[i][j] -= f * M[k][j]
    return piv


def test_exact_rational_pivots_and_info():
    rng = np.random.default_rng(11)
    checked_fail = checked_ok = 0
    for trial in range(300):
        n = int(rng.integers(1, 11))
        X = rng.integers(-3, 4, size=(n, n))
        A = X @ X.T + np.diag(rng.integers(-6, 4, size=n))
        A = (A + A.T) // 2
        piv = _ldl_pivots(A)
        k_exact = next((k + 1 for k, d in enumerate(piv) if d <= 0), 0)
        # only judge cases where all float pivots are well separated from 0
        if any(abs(float(d)) < 1e-6 for d in piv):
            continue
        L, info = _chol(A.astype(np.float64))
        assert info == k_exact
        nb = n if info == 0 else info - 1
        for q in range(nb):
            assert math.isclose(L[q, q] ** 2, float(piv[q]), rel_tol=1e-12)
        checked_fail += info > 0
        checked_ok += info == 0
    assert checked_fail > 20 and checked_ok > 20


# ---------------------------------------------------------------- invariants / library
def test_det_invariant():
    """prod l_jj^2 == det(A) with det from long-double partial-pivot LU (independent algorithm)."""
    for n in (3, 10, 25):
        A = vbgen.f1_matrix(2, n, n) / n
        L, info = _chol(A)
        assert info == 0
        M = A.astype(np.longdouble).copy()
        det = np.longdouble(1)
        for k in range(n):
            p = k + int(np.argmax(np.abs(M[k:, k])))
            if p != k:
                M[[k, p]] = M[[p, k]]
                det = -det
            det *= M[k, k]
            M[k + 1:, k:] -= np.outer(M[k + 1:, k] / M[k, k], M[k, k:])
        prod = np.prod(np.diag(L).astype(np.longdouble) ** 2)
        assert abs(prod / det - 1) < 1e-12


@pytest.mark.parametrize("n", [8, 64, 256])
def test_random_well_conditioned_L_recovered(n):
    rng = np.random.default_rng(n)
    L = np.tril(rng.uniform(-1, 1, (n, n)) / n, -1) + np.diag(rng.uniform(1, 2, n))
    A = np.asfortranarray(L @ L.T)
    Lc, info = _chol(A)
    assert info == 0
    assert np.max(np.abs(np.tril(Lc) - L)) / np.max(np.abs(L)) < 1e-13


@pytest.mark.parametrize("n", [1, 5, 40, 130, 300])
def test_matches_mkl_dpotrf(n):
    import torch
    for gidx in range(3):
        A = vbgen.f1_matrix(3, gidx, n)
        L, info = _chol(A)
        Lm, info_m = torch.linalg.cholesky_ex(torch.from_numpy(A))
        assert info == int(info_m) == 0
        assert oracle.rowscaled_diff(L, Lm.numpy(), n) < 1e-13
        assert oracle.backward_error(A, L, info) < 1.0


def test_matches_openblas_info_on_nonspd():
    from scipy.linalg import lapack
    for n in (5, 50, 120):
        for gidx in (19, 39, 59):
            A = vbgen.f1_matrix(4, gidx, n, nonspd=True)
            _, info_s = lapack.dpotrf(A, lower=1, clean=0)
            assert _chol(A)[1] == info_s


def test_ill_conditioned_backward_error():
    """F2 family: Q diag(lambda) Q^T with lambda log-uniform in [1,1e4]."""
    rng = np.random.default_rng(5)
    for n in (16, 64, 128):
        Q, _ = np.linalg.qr(rng.standard_normal((n, n)))
        lam = 10 ** rng.uniform(0, 4, n)
        A = np.asfortranarray((Q * lam) @ Q.T)
        A = np.asfortranarray((A + A.T) / 2)
        L, info = _chol(A)
        assert info == 0
        assert oracle.backward_error(A, L, info) < 10


def test_backward_error_detects_wrong_factor():
    n = 20
    A = vbgen.f1_matrix(1, 2, n)
    L, info = _chol(A)
    assert oracle.backward_error(A, L, info) < 10
    L2 = L.copy(order="F")
    L2[7, 3] *= (1 + 1e-10)
    assert oracle.backward_error(A, L2, info) > 10


def test_batch_equals_single():
    n = np.array([0, 1, 5, 33, 64, 100, 2], dtype=np.int32)
    ld = vbgen.ldda_for(n, "pad32")
    off, tot = vbgen.arena_layout(n, ld)
    arena = np.zeros(tot)
    for b in range(len(n)):
        A = vbgen.f1_matrix(1, b, int(n[b]), nonspd=(b == 3))
        blk = np.zeros((ld[b], n[b]), order="F")
        blk[: n[b], :] = A
        arena[off[b]: off[b] + ld[b] * n[b]] = blk.ravel(order="F")
    ref = arena.copy()
    info = oracle.dpotrf_batch(arena, off, n, ld, nthreads=4)
    for b in range(len(n)):
        A = ref[off[b]: off[b] + ld[b] * n[b]].reshape((ld[b], n[b]), order="F")[: n[b]]
        L1, i1 = _chol(np.asfortranarray(A))
        got = arena[off[b]: off[b] + ld[b] * n[b]].reshape((ld[b], n[b]), order="F")[: n[b]]
        assert info[b] == i1
        assert np.array_equal(np.tril(got), np.tril(L1))
    assert info[3] == vbgen.nonspd_k(1, 3, 33)


# ---------------------------------------------------------------- BLAS oracles
def _rand(rng, *shape):
    return np.asfortranarray(rng.standard_normal(shape))


@pytest.mark.parametrize("ta,tb", [("N", "N"), ("N", "T"), ("T", "N"), ("T", "T")])
def test_gemm_oracle(ta, tb):
    rng = np.random.default_rng(1)
    m, n, k = 7, 5, 9
    A = _rand(rng, m, k) if ta == "N" else _rand(rng, k, m)
    B = _rand(rng, k, n) if tb == "N" else _rand(rng, n, k)
    C = _rand(rng, m, n)
    got = oracle.dgemm(ta, tb, 1.5, A, B, -0.5, C)
    opA = A if ta == "N" else A.T
    opB = B if tb == "N" else B.T
    assert np.allclose(got, 1.5 * opA @ opB - 0.5 * C, rtol=1e-13, atol=1e-13)
    # exact small-integer case
    Ai = np.asfortranarray(rng.integers(-3, 4, A.shape).astype(float))
    Bi = np.asfortranarray(rng.integers(-3, 4, B.shape).astype(float))
    Ci = np.asfortranarray(rng.integers(-3, 4, C.shape).astype(float))
    opA = Ai if ta == "N" else Ai.T
    opB = Bi if tb == "N" else Bi.T
    assert np.array_equal(oracle.dgemm(ta, tb, 1.0, Ai, Bi, 1.0, Ci), opA @ opB + Ci)


@pytest.mark.parametrize("uplo,trans", [("L", "N"), ("L", "T"), ("U", "N"), ("U", "T")])
def test_syrk_oracle(uplo, trans):
    rng = np.random.default_rng(2)
    n, k = 6, 4
    A = _rand(rng, n, k) if trans == "N" else _rand(rng, k, n)
    C = _rand(rng, n, n)
    got = oracle.dsyrk(uplo, trans, -1.0, A, 1.0, C)
    full = -(A @ A.T if trans == "N" else A.T @ A) + C
    tri = np.tril if uplo == "L" else np.triu
    other = np.triu if uplo == "L" else np.tril
    assert np.allclose(tri(got), tri(full), rtol=1e-13, atol=1e-13)
    assert np.array_equal(other(got, 1 if uplo == "L" else -1), other(C, 1 if uplo == "L" else -1))


@pytest.mark.parametrize("side", ["L", "R"])
@pytest.mark.parametrize("uplo", ["L", "U"])
@pytest.mark.parametrize("ta", ["N", "T"])
@pytest.mark.parametrize("diag", ["N", "U"])
def test_trsm_oracle(side, uplo, ta, diag):
    from scipy.linalg import solve_triangular
    rng = np.random.default_rng(3)
    m, n = 6, 5
    na = m if side == "L" else n
    A = _rand(rng, na, na) + 4 * np.eye(na)
    A = np.asfortranarray(A)
    B = _rand(rng, m, n)
    X = oracle.dtrsm(side, uplo, ta, diag, 2.0, A, B)
    T = np.tril(A) if uplo == "L" else np.triu(A)
    if diag == "U":
        np.fill_diagonal(T, 1.0)
    opT = T if ta == "N" else T.T
    if side == "L":
        ref = solve_triangular(opT, 2.0 * B, lower=np.allclose(opT, np.tril(opT)))
        assert np.allclose(opT @ X, 2.0 * B, rtol=1e-12, atol=1e-12)
    else:
        ref = solve_triangular(opT.T, (2.0 * B).T, lower=np.allclose(opT.T, np.tril(opT.T))).T
        assert np.allclose(X @ opT, 2.0 * B, rtol=1e-12, atol=1e-12)
    assert np.allclose(X, ref, rtol=1e-12, atol=1e-12)


# ---- NEXT-4: the solve (LAPACK DPOTRS / DPOSV) ------------------------------------------------
@pytest.mark.parametrize("uplo", ["L", "U"])
@pytest.mark.parametrize("n,nrhs", [(1, 1), (7, 3), (33, 5), (128, 1), (200, 17)])
def test_potrs_oracle_exact_integer_family(uplo, n, nrhs):
    """A = L L^T with integer unit-lower L (entries -1/0/1) and B = A X0 with integer X0:
    every intermediate of both triangular solves is an integer below 2^53 and every division
    is by 1, so the oracle must return X0 exactly (and the factor L exactly)."""
    rng = np.random.default_rng(100 + n)
    L = np.tril(rng.integers(-1, 2, size=(n, n)), -1).astype(np.int64) + np.eye(n, dtype=np.int64)
    A = (L @ L.T).astype(np.float64)
    X0 = rng.integers(-3, 4, size=(n, nrhs)).astype(np.int64)
    B = (L @ (L.T @ X0)).astype(np.float64)
    X, F, info = oracle.dposv(uplo, A, B)
    assert info == 0
    if uplo == "L":
        assert np.array_equal(F, L.astype(np.float64))
    else:
        assert np.array_equal(F, L.T.astype(np.float64))
    assert np.array_equal(X, X0.astype(np.float64))


@pytest.mark.parametrize("uplo", ["L", "U"])
def test_potrs_oracle_residual_and_library(uplo):
    """F1 matrices: the solution matches numpy's LAPACK solve (dgesv) to 1e-12 relative and the
    residual ||A X - B|| is at rounding level."""
    rng = np.random.default_rng(7)
    for n, nrhs in [(5, 2), (64, 8), (257, 3)]:
        A = vbgen.f1_matrix(9, n, n)
        B = rng.standard_normal((n, nrhs))
        X, _, info = oracle.dposv(uplo, A, B)
        assert info == 0
        ref = np.linalg.solve(A, B)
        assert np.max(np.abs(X - ref)) <= 1e-12 * np.max(np.abs(ref))
        assert np.linalg.norm(A @ X - B) <= 1e-13 * np.linalg.norm(A) * np.linalg.norm(X)


def test_posv_oracle_failure_keeps_b():
    A = vbgen.f1_matrix(9, 3, 40)
    A[9, 9] = -A[9, 9]
    B = np.arange(80, dtype=np.float64).reshape(40, 2)
    X, _, info = oracle.dposv("L", A, B)
    assert info == 10 and np.array_equal(X, B)


# ---- NEXT-3: the FP32 oracle (oracle_spotrf_lower) --------------------------------------------
def test_spotrf_oracle_exact_families():
    """min(i,j) -> tril(ones) and integer unit-lower L (entries -1/0/1, A = L L^T below 2^24):
    every operation is exact in FP32 too, so the factor must be bit-exact."""
    n = 120
    i = np.arange(1, n + 1)
    L, info = oracle.spotrf(np.minimum.outer(i, i).astype(np.float32))
    assert info == 0 and np.array_equal(np.tril(L), np.tril(np.ones((n, n), np.float32)))
    rng = np.random.default_rng(41)
    for n in (17, 64, 100):
        Li = np.tril(rng.integers(-1, 2, size=(n, n)), -1).astype(np.int64) + np.eye(n, dtype=np.int64)
        A = (Li @ Li.T)
        assert np.abs(A).max() < 2 ** 24
        L, info = oracle.spotrf(A.astype(np.float32))
        assert info == 0 and np.array_equal(np.tril(L), Li.astype(np.float32))


def test_spotrf_oracle_vs_fp64_and_lapack():
    """On F1 matrices (kappa ~ 1.6) the FP32 factor is within a small multiple of n eps32 of the
    FP64 oracle's (row-scaled) and of numpy's float32 LAPACK Cholesky; the FP32 backward error
    ratio stays <= 10; an injected negative pivot gives the same info as FP64."""
    for n in (5, 64, 300):
        A = vbgen.f1_matrix(13, n, n)
        A32 = A.astype(np.float32)
        L32, info = oracle.spotrf(A32)
        L64, info64 = oracle.dpotrf(A32.astype(np.float64))
        assert info == info64 == 0
        rs = oracle.rowscaled_diff(L32.astype(np.float64), L64, n)
        assert rs <= 4 * n * 2.0 ** -24, (n, rs)
        Ln = np.linalg.cholesky(A32)
        assert oracle.rowscaled_diff(L32.astype(np.float64), Ln.astype(np.float64), n) <= 4 * n * 2.0 ** -24
        assert oracle.backward_error_f32(A32, np.tril(L32), info) <= 10.0
    A = vbgen.f1_matrix(13, 7, 90).astype(np.float32)
    A[40, 40] = -A[40, 40]
    assert oracle.spotrf(A)[1] == 41


# ---------------------------------------------------------------- the parity gates themselves
# The two gate functions every GPU parity test relies on are pinned here against closed forms
# computed independently (exact rationals / hand arithmetic), so that a gate that returned 0,
# used eps = 2^-52 instead of 2^-53, dropped the factor n, or read the wrong triangle would fail.
def _bwd_closed_form(A, Lg, nb, eps):
    """||A - Lg Lg^T||_F / (nb ||A||_F eps) on the leading nb block, exact rational sums
    (Fractions) and one final float sqrt: independent of the oracle's long-double loop."""
    Af = [[Fraction(float(A[max(i, j), min(i, j)])) for j in range(nb)] for i in range(nb)]
    Lf = [[Fraction(float(Lg[i, k])) if k <= i else Fraction(0) for k in range(nb)]
          for i in range(nb)]
    num = Fraction(0)
    den = Fraction(0)
    for i in range(nb):
        for j in range(nb):
            s = sum((Lf[i][k] * Lf[j][k] for k in range(nb)), Fraction(0))
            d = Af[i][j] - s
            num += d * d
            den += Af[i][j] * Af[i][j]
    return math.sqrt(num) / (nb * math.sqrt(den) * eps)


def _int_spd(n, seed):
    rng = np.random.default_rng(seed)
    L = np.tril(rng.integers(-3, 4, size=(n, n)), -1).astype(np.float64)
    L[np.arange(n), np.arange(n)] = rng.integers(1, 5, size=n)
    return L, np.asfortranarray(L @ L.T)  # exact small integers


def test_backward_error_gate_closed_form():
    """oracle_backward_error on an exact A = L L^T with a known perturbation of L: equals the
    closed form ||A - Lg Lg^T||_F / (n ||A||_F 2^-53) to 1e-9 relative."""
    L, A = _int_spd(7, 41)
    assert oracle.backward_error(A, np.asfortranarray(L), 0) == 0.0  # exact factor -> 0
    for (p, q, d) in [(3, 1, 2.0 ** -40), (6, 6, -(2.0 ** -37)), (0, 0, 2.0 ** -45)]:
        Lg = np.asfortranarray(L.copy())
        Lg[p, q] += d
        got = oracle.backward_error(A, Lg, 0)
        exp = _bwd_closed_form(A, Lg, 7, 2.0 ** -53)
        assert got == pytest.approx(exp, rel=1e-9), (p, q, got, exp)
        # the same number by hand for a single perturbed entry: Delta = d (l_q e_p^T + e_p l_q^T)
        # + d^2 e_p e_p^T with l_q = column q of L (row p's own entry included)
        lq = L[:, q].copy()
        D = d * (np.outer(lq, np.eye(7)[p]) + np.outer(np.eye(7)[p], lq))
        D[p, p] += d * d
        hand = np.sqrt(np.sum(D * D)) / (7 * np.sqrt(np.sum(A * A)) * 2.0 ** -53)
        assert got == pytest.approx(hand, rel=1e-6)
    # eps = 2^-52 or a dropped n would be off by exactly 2x / 7x
    Lg = np.asfortranarray(L.copy())
    Lg[4, 2] += 2.0 ** -40
    got = oracle.backward_error(A, Lg, 0)
    assert got != pytest.approx(_bwd_closed_form(A, Lg, 7, 2.0 ** -52), rel=0.1)
    assert got != pytest.approx(_bwd_closed_form(A, Lg, 7, 2.0 ** -53) * 7, rel=0.1)


def test_backward_error_gate_triangles_and_leading_block():
    """Only A's lower triangle and Lg's lower triangle are read; on info > 0 only the leading
    (info-1) block counts (SURVEY §8(c) readings #3, #13)."""
    L, A = _int_spd(6, 43)
    Ab = np.asfortranarray(A.copy())
    Ab[np.triu_indices(6, 1)] = np.nan  # strict upper of A: never read
    Lg = np.asfortranarray(L.copy())
    Lg[np.triu_indices(6, 1)] = np.nan  # strict upper of the factor: taken as zero
    Lg[2, 1] += 2.0 ** -40
    got = oracle.backward_error(Ab, Lg, 0)
    assert got == pytest.approx(_bwd_closed_form(A, Lg, 6, 2.0 ** -53), rel=1e-9)
    # info = 4: the leading 3x3 block only; a perturbation in row 4 does not count
    Lg2 = np.asfortranarray(L.copy())
    Lg2[4, 1] += 1.0
    assert oracle.backward_error(A, Lg2, 4) == 0.0
    Lg2[1, 0] += 2.0 ** -40
    assert oracle.backward_error(A, Lg2, 4) == pytest.approx(
        _bwd_closed_form(A, Lg2, 3, 2.0 ** -53), rel=1e-9)


def test_backward_error_f32_gate_closed_form():
    """backward_error_f32 is the same ratio with eps32 = 2^-24."""
    L, A = _int_spd(5, 47)
    Lg = np.asfortranarray(L.copy())
    Lg[3, 2] += 2.0 ** -20
    assert oracle.backward_error_f32(A, Lg, 0) == pytest.approx(
        _bwd_closed_form(A, Lg, 5, 2.0 ** -24), rel=1e-9)


def test_rowscaled_gate_closed_form():
    """rowscaled_diff = max_{i>=j} |Lg_ij - Lo_ij| / ||Lo(i, 0:i)||_2 on the leading nb block
    (SURVEY §8(c) reading #14), on hand-built rows with norms 3, 5, 3, 13."""
    Lo = np.array([[3.0, 0, 0, 0],
                   [3.0, 4.0, 0, 0],
                   [1.0, 2.0, 2.0, 0],
                   [3.0, 4.0, 12.0, 0.0]])  # row norms 3, 5, 3, 13
    assert oracle.rowscaled_diff(Lo, Lo, 4) == 0.0
    Lg = Lo.copy()
    Lg[1, 0] += 1e-6       # 1e-6 / 5
    assert oracle.rowscaled_diff(Lg, Lo, 4) == pytest.approx(2e-7, rel=1e-12)
    Lg[2, 2] -= 3e-5       # 3e-5 / 3 = 1e-5 (the max)
    assert oracle.rowscaled_diff(Lg, Lo, 4) == pytest.approx(1e-5, rel=1e-9)
    Lg[3, 2] = -12.0       # sign flip: 24 / 13
    assert oracle.rowscaled_diff(Lg, Lo, 4) == pytest.approx(24 / 13, rel=1e-12)
    # the strict upper triangle and rows/cols beyond nb are not compared
    Lh = Lo.copy()
    Lh[0, 3] = 1e9
    Lh[3, 3] = 7.0
    assert oracle.rowscaled_diff(Lh, Lo, 3) == 0.0
    assert oracle.rowscaled_diff(Lh, Lo, 4) == pytest.approx(7 / 13, rel=1e-12)
    # a zero row of the oracle's factor scales by 1 (absolute difference)
    Z = np.zeros((2, 2))
    Zg = Z.copy()
    Zg[1, 0] = 2.5e-3
    assert oracle.rowscaled_diff(Zg, Z, 2) == pytest.approx(2.5e-3, rel=1e-12)
    # a NaN in the compared part must fail the gate (compare_with_oracle uses <= 1e-10)
    Ln = Lo.copy()
    Ln[2, 1] = np.nan
    assert not (oracle.rowscaled_diff(Ln, Lo, 4) <= 1e-10)


# ---------------------------------------------------------------- LU
def _apply_ipiv(A, ipiv):
    """P A for LAPACK interchanges ipiv (1-based), applied in order."""
    B = np.array(A, dtype=np.float64, copy=True)
    for k, p in enumerate(ipiv):
        if p - 1 != k:
            B[[k, p - 1], :] = B[[p - 1, k], :]
    return B


def _split_lu(F):
    m, n = F.shape
    k = min(m, n)
    L = np.tril(F[:, :k], -1) + np.eye(m, k)
    U = np.triu(F[:k, :])
    return L, U


def test_lu_handworked_golden():
    g = json.load(open(os.path.join(GOLD, "lu_handworked.json")))
    for c in g["cases"]:
        F, ipiv, info = oracle.dgetrf(np.array(c["A"], dtype=np.float64))
        assert np.array_equal(F, np.array(c["F"], dtype=np.float64)), c["name"]
        assert list(ipiv) == c["ipiv"] and info == c["info"], c["name"]


@pytest.mark.parametrize("m,n", [(1, 1), (5, 5), (33, 33), (64, 40), (40, 64), (130, 130)])
def test_lu_exact_family(m, n):
    """A = P0 L U with unit-lower L (|l_ik| <= 1/2, dyadic) and integer U whose pivots dominate:
    partial pivoting must select exactly the rows P0 moved, and L, U come back bit-exactly."""
    rng = np.random.default_rng(1000 + 7 * m + n)
    k = min(m, n)
    L = np.tril(rng.choice([-0.5, -0.25, 0.0, 0.25, 0.5], size=(m, k)), -1) + np.eye(m, k)
    U = np.triu(rng.integers(-3, 4, size=(k, n)).astype(np.float64), 1)
    U[np.arange(k), np.arange(k)] = rng.choice([-8.0, -4.0, 4.0, 8.0], size=k)
    A = L @ U  # exact: dyadic products, small sums
    perm = rng.permutation(m)
    A0 = A[perm]
    F, ipiv, info = oracle.dgetrf(A0)
    assert info == 0
    Lg, Ug = _split_lu(F)
    assert np.array_equal(Ug, U)
    # the k pivot rows are A's first k rows in order (their l = 1 entries dominate), so L's top
    # k rows come back exactly; the rows below are a row permutation of L's (order set by the
    # interchanges), and P A0 = L U holds bit-exactly
    assert np.array_equal(Lg[:k], L[:k])
    key = lambda M: M[np.lexsort(M.T[::-1])]  # noqa: E731
    assert np.array_equal(key(Lg[k:]), key(L[k:]))
    assert np.array_equal(_apply_ipiv(A0, ipiv), Lg @ Ug)


@pytest.mark.parametrize("m,n", [(7, 7), (64, 64), (100, 37), (37, 100), (257, 257)])
def test_lu_matches_lapack(m, n):
    """ipiv bit-exact and the factors within 1e-12 of LAPACK DGETRF (OpenBLAS via scipy, MKL via
    torch) on the general random family."""
    import scipy.linalg
    import torch
    A = vbgen.g1_matrix(11, m * 1000 + n, m, n)
    F, ipiv, info = oracle.dgetrf(A)
    lu, piv = scipy.linalg.lu_factor(A, check_finite=False)
    k = min(m, n)
    assert info == 0
    assert np.array_equal(ipiv, (piv[:k] + 1).astype(np.int32))
    assert np.max(np.abs(F - lu)) <= 1e-12 * max(1.0, np.max(np.abs(lu)))
    LU_t, piv_t = torch.linalg.lu_factor(torch.from_numpy(np.array(A)))
    assert np.array_equal(ipiv, piv_t.numpy()[:k].astype(np.int32))
    assert np.max(np.abs(F - LU_t.numpy())) <= 1e-12 * max(1.0, np.max(np.abs(lu)))


def test_lu_singular_info():
    A = np.ones((6, 6))
    _, _, info = oracle.dgetrf(A)
    assert info == 2  # second pivot exactly zero (rows all equal)
    B = vbgen.g1_matrix(3, 5, 8, 8)
    B[:, 3] = 0.0
    _, ipiv, info = oracle.dgetrf(B)
    assert info == 4 and ipiv[3] == 4  # zero column: no interchange, info = first zero pivot
    Z = np.zeros((3, 5))
    F, ipiv, info = oracle.dgetrf(Z)
    assert info == 1 and list(ipiv) == [1, 2, 3] and not F.any()


def test_lu_det_invariant_exact_rational():
    """det(A) = (-1)^(#swaps) prod u_kk, against an exact rational determinant (Bareiss-free
    Fraction elimination) of small integer matrices."""
    rng = np.random.default_rng(77)
    for n in (2, 3, 5, 8):
        A = rng.integers(-9, 10, size=(n, n)).astype(np.float64)
        M = [[Fraction(int(x)) for x in row] for row in A]
        det = Fraction(1)
        for k in range(n):
            p = next((i for i in range(k, n) if M[i][k] != 0), None)
            if p is None:
                det = Fraction(0)
                break
            if p != k:
                M[k], M[p] = M[p], M[k]
                det = -det
            det *= M[k][k]
            for i in range(k + 1, n):
                f = M[i][k] / M[k][k]
                for j in range(k, n):
                    M[i][j] -= f * M[k][j]
        F, ipiv, info = oracle.dgetrf(A)
        sign = (-1) ** sum(1 for k, p in enumerate(ipiv) if p - 1 != k)
        got = sign * np.prod(np.diag(F))
        assert got == pytest.approx(float(det), rel=1e-12, abs=1e-12)


def test_lu_backward_error_gate_closed_form():
    """oracle_getrf_backward_error: 0 on an exact factorisation; equals the Fraction closed form
    ||P A - L U||_F / (max(m,n) ||A||_F 2^-53) for a known perturbation of U; dgetrf's own
    factors of a random matrix stay far below 10."""
    m, n = 6, 4
    rng = np.random.default_rng(5)
    L = np.tril(rng.choice([-0.5, 0.25, 0.5], size=(m, n)), -1) + np.eye(m, n)
    U = np.triu(rng.integers(-3, 4, size=(n, n)).astype(np.float64), 1) + np.diag([8.0, -8, 4, 4])
    A = L @ U
    F, ipiv, info = oracle.dgetrf(A)
    assert info == 0 and oracle.getrf_backward_error(A, F, ipiv) == 0.0
    F2 = F.copy(order="F")
    F2[1, 2] += 2.0 ** -30
    Lf, Uf = _split_lu(F2)
    PA = [[Fraction(float(x)) for x in row] for row in _apply_ipiv(A, ipiv)]
    LfF = [[Fraction(float(x)) for x in row] for row in Lf]
    UfF = [[Fraction(float(x)) for x in row] for row in Uf]
    num = sum((PA[i][j] - sum((LfF[i][k] * UfF[k][j] for k in range(n)), Fraction(0))) ** 2
              for i in range(m) for j in range(n))
    den = sum(x * x for row in PA for x in row)
    exp = math.sqrt(num) / (max(m, n) * math.sqrt(den) * 2.0 ** -53)
    assert oracle.getrf_backward_error(A, F2, ipiv) == pytest.approx(exp, rel=1e-9)
    G = vbgen.g1_matrix(2, 9, 200, 200)
    FG, ipg, _ = oracle.dgetrf(G)
    assert oracle.getrf_backward_error(G, FG, ipg) < 10


# ---------------------------------------------------------------- complex Cholesky (NEXT-3)
def test_zpotrf_handworked():
    """[[4, .], [2+2i, 6]] -> l21 = 1+i, l22 = sqrt(6 - |1+i|^2) = 2 (exact); the strict upper
    triangle is never read or written; the diagonal's imaginary part is ignored."""
    A = np.array([[4 + 5j, np.nan], [2 + 2j, 6 - 3j]], dtype=np.complex128)
    L, info = oracle.zpotrf(A)
    assert info == 0
    assert L[0, 0] == 2 and L[1, 0] == 1 + 1j and L[1, 1] == 2
    assert np.isnan(L[0, 1])


@pytest.mark.parametrize("n", [1, 7, 33, 100])
def test_zpotrf_gaussian_integer_family_exact(n):
    """L with real diagonal in {1,2,4} and Gaussian-integer entries in {-1,0,1} + i{-1,0,1}:
    A = L L^H is exact, so chol(A) = L bit for bit (double and single precision)."""
    rng = np.random.default_rng(300 + n)
    L = np.tril(rng.integers(-1, 2, (n, n)) + 1j * rng.integers(-1, 2, (n, n)), -1)
    L[np.arange(n), np.arange(n)] = rng.choice([1.0, 2.0, 4.0], n)
    A = L @ L.conj().T
    Lz, info = oracle.zpotrf(A)
    assert info == 0 and np.array_equal(np.tril(Lz), L)
    if n <= 33:
        Lc, info = oracle.cpotrf(A.astype(np.complex64))
        assert info == 0 and np.array_equal(np.tril(Lc), L.astype(np.complex64))


def test_zpotrf_real_case_equals_real_oracle():
    """With zero imaginary parts the complex recurrence performs the real one's operations."""
    A = vbgen.f1_matrix(3, 4, 60)
    Lr, ir = oracle.dpotrf(A)
    Lz, iz = oracle.zpotrf(A.astype(np.complex128))
    assert ir == iz == 0
    assert np.array_equal(np.tril(Lz).real, np.tril(Lr)) and not np.tril(Lz).imag.any()


@pytest.mark.parametrize("n", [5, 64, 200])
def test_zpotrf_matches_lapack_and_backward_error(n):
    import torch
    A = vbgen.f1c_matrix(9, n, n)
    L, info = oracle.zpotrf(A)
    assert info == 0
    ref = np.linalg.cholesky(A)  # LAPACK ZPOTRF (numpy's bundled OpenBLAS)
    assert np.max(np.abs(np.tril(L) - ref)) <= 1e-13 * np.max(np.abs(ref))
    Lt, it = torch.linalg.cholesky_ex(torch.from_numpy(A))  # MKL
    assert int(it) == 0 and np.max(np.abs(np.tril(L) - Lt.numpy())) <= 1e-13 * np.max(np.abs(ref))
    assert oracle.zpotrf_backward_error(A, np.tril(L), 0) < 10
    Lc, infoc = oracle.cpotrf(A.astype(np.complex64))
    assert infoc == 0 and np.max(np.abs(np.tril(Lc) - ref)) <= 8 * n * 2.0 ** -24 * np.max(np.abs(ref))


def test_zpotrf_info_and_backward_error_gate():
    A = vbgen.f1c_matrix(4, 19, 40, nonspd=True)
    k = vbgen.nonspd_k(4, 19, 40)
    L, info = oracle.zpotrf(A)
    assert info == k
    # closed-form gate: a perturbation d of one entry of an exact factor
    rng = np.random.default_rng(2)
    n = 5
    Le = np.tril(rng.integers(-1, 2, (n, n)) + 1j * rng.integers(-1, 2, (n, n)), -1)
    Le[np.arange(n), np.arange(n)] = 2.0
    Ae = Le @ Le.conj().T
    assert oracle.zpotrf_backward_error(Ae, Le, 0) == 0.0
    Lp = Le.copy()
    Lp[3, 1] += 2.0 ** -40 * 1j
    D = Ae - Lp @ Lp.conj().T  # exact in double: entries are Gaussian integers +- 2^-40 terms
    exp = np.sqrt(np.sum(np.abs(D) ** 2)) / (n * np.sqrt(np.sum(np.abs(Ae) ** 2)) * 2.0 ** -53)
    assert oracle.zpotrf_backward_error(Ae, Lp, 0) == pytest.approx(exp, rel=1e-9)


# ---------------------------------------------------------------- QR
def test_qr_handworked_golden():
    g = json.load(open(os.path.join(GOLD, "qr_handworked.json")))
    for c in g["cases"]:
        F, tau = oracle.dgeqrf(np.array(c["A"], dtype=np.float64))
        Fx, tx = np.array(c["F"], dtype=np.float64), np.array(c["tau"], dtype=np.float64)
        assert np.all(np.abs(F - Fx) <= 4 * 2.0 ** -52 * np.maximum(np.abs(Fx), 1e-300)), c["name"]
        assert np.all(np.abs(tau - tx) <= 4 * 2.0 ** -52 * np.abs(tx)), c["name"]


@pytest.mark.parametrize("m,n", [(1, 1), (2, 5), (7, 7), (50, 30), (30, 50), (130, 130), (257, 100)])
def test_qr_matches_lapack_and_gates(m, n):
    """Compact factor and tau within 1e-12 of LAPACK DGEQRF (OpenBLAS via scipy, MKL via torch);
    reconstruction and orthogonality gates far below 10."""
    import scipy.linalg
    import torch
    A = vbgen.g1_matrix(21, m * 1000 + n, m, n)
    F, tau = oracle.dgeqrf(A)
    (qr, tq), _ = scipy.linalg.qr(A, mode="raw")
    scale = max(1.0, np.max(np.abs(qr)))
    assert np.max(np.abs(F - qr)) <= 1e-12 * scale and np.max(np.abs(tau - tq[: len(tau)])) <= 1e-13
    Ft, tt = torch.geqrf(torch.from_numpy(np.array(A)))
    assert np.max(np.abs(F - Ft.numpy())) <= 1e-12 * scale
    assert np.max(np.abs(tau - tt.numpy()[: len(tau)])) <= 1e-13
    bwd, orth = oracle.geqrf_errors(A, F, tau)
    assert bwd < 10 and orth < 10


def test_qr_triangular_input_and_zero_columns():
    """A column that is already zero below the diagonal: tau = 0, H = I, the column unchanged."""
    A = np.triu(vbgen.g1_matrix(5, 1, 6, 6))
    F, tau = oracle.dgeqrf(A)
    assert np.array_equal(F, A) and not tau.any()
    Z = np.zeros((4, 3))
    F, tau = oracle.dgeqrf(Z)
    assert not F.any() and not tau.any()


def test_qr_gate_closed_form():
    """Orthogonality gate: a single reflector for x = (3, 4) with tau perturbed by d gives
    Q^T Q - I = (2 tau v^T v - 2) d v v^T + O(d^2) = 2 d v v^T (v = (1, 1/2)), so the gate reads
    2 d ||v||^2 / (2 eps) = 2.5 d / (2 eps)."""
    A = np.array([[3.0], [4.0]])
    F, tau = oracle.dgeqrf(A)
    b0, o0 = oracle.geqrf_errors(A, F, tau)
    assert b0 < 1 and o0 < 1
    d = 2.0 ** -40
    _, o = oracle.geqrf_errors(A, F, tau + d)
    assert o == pytest.approx(2.5 * d / (2 * 2.0 ** -53), rel=1e-3)
