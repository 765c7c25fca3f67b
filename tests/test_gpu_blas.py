"""GPU parity of the standalone vbatched BLAS (vbatched_dgemm / dsyrk / dtrsm) against the
oracle's plain-loop BLAS definitions, on variable sizes including 0 and ragged tiles."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ipps_abdelfattahhtd16_b200 as vb

pytestmark = pytest.mark.gpu


class Mats:
    """Variable-size batch of column-major matrices in one device arena."""

    def __init__(self, shapes, rng, kind="randn"):
        self.shapes = shapes
        self.ld = [max(1, r + (i % 3)) for i, (r, c) in enumerate(shapes)]  # ld >= rows, ragged
        sizes = [ld * c for ld, (r, c) in zip(self.ld, shapes)]
        self.off = np.concatenate([[0], np.cumsum(sizes)]).astype(np.int64)
        self.host = np.zeros(max(1, int(self.off[-1])))
        for i, (r, c) in enumerate(shapes):
            blk = rng.standard_normal((self.ld[i], c)) if kind == "randn" else np.zeros((self.ld[i], c))
            self.host[self.off[i]: self.off[i] + self.ld[i] * c] = blk.ravel(order="F")
        self.dev = torch.from_numpy(self.host.copy()).cuda()
        self.ptrs = torch.from_numpy(self.dev.data_ptr() + 8 * self.off[:-1]).cuda()
        self.d_ld = torch.tensor(self.ld, dtype=torch.int32, device="cuda")

    def get(self, i, src=None):
        r, c = self.shapes[i]
        a = self.host if src is None else src
        return a[self.off[i]: self.off[i] + self.ld[i] * c].reshape((self.ld[i], c), order="F")[:r].copy(order="F")

    def result(self):
        return self.dev.cpu().numpy()


def _ints(x):
    return torch.tensor(x, dtype=torch.int32, device="cuda")


SIZES = [(0, 5, 3), (1, 1, 1), (5, 7, 0), (64, 64, 64), (65, 63, 17), (130, 70, 200), (7, 129, 33),
         (200, 1, 65), (33, 33, 100)]


@pytest.mark.parametrize("ta,tb", [("N", "N"), ("N", "T"), ("T", "N"), ("T", "T")])
def test_gemm(ta, tb):
    rng = np.random.default_rng(1)
    m = [s[0] for s in SIZES]
    n = [s[1] for s in SIZES]
    k = [s[2] for s in SIZES]
    A = Mats([(mi, ki) if ta == "N" else (ki, mi) for mi, ki in zip(m, k)], rng)
    B = Mats([(ki, ni) if tb == "N" else (ni, ki) for ni, ki in zip(n, k)], rng)
    C = Mats(list(zip(m, n)), rng)
    alpha, beta = 1.25, -0.5
    vb.vbatched_dgemm(ta, tb, _ints(m), _ints(n), _ints(k), alpha, A.ptrs, A.d_ld, B.ptrs, B.d_ld,
                      beta, C.ptrs, C.d_ld, len(m), max(m), max(n), max(k))
    torch.cuda.synchronize()
    out = C.result()
    for i in range(len(m)):
        ref = oracle.dgemm(ta, tb, alpha, A.get(i), B.get(i), beta, C.get(i))
        got = C.get(i, out)
        scale = max(1.0, np.max(np.abs(ref)) if ref.size else 1.0)
        assert got.shape == ref.shape
        if ref.size:
            assert np.max(np.abs(got - ref)) / scale < 1e-13 * max(1, k[i]), (i, ta, tb)


@pytest.mark.parametrize("uplo,trans", [("L", "N"), ("L", "T"), ("U", "N"), ("U", "T")])
def test_syrk(uplo, trans):
    rng = np.random.default_rng(2)
    n = [s[0] for s in SIZES]
    k = [s[2] for s in SIZES]
    A = Mats([(ni, ki) if trans == "N" else (ki, ni) for ni, ki in zip(n, k)], rng)
    C = Mats([(ni, ni) for ni in n], rng)
    alpha, beta = -1.0, 1.0
    vb.vbatched_dsyrk(uplo, trans, _ints(n), _ints(k), alpha, A.ptrs, A.d_ld, beta, C.ptrs, C.d_ld,
                      len(n), max(n), max(k))
    torch.cuda.synchronize()
    out = C.result()
    for i in range(len(n)):
        ref = oracle.dsyrk(uplo, trans, alpha, A.get(i), beta, C.get(i))
        got = C.get(i, out)
        if ref.size:
            scale = max(1.0, np.max(np.abs(ref)))
            assert np.max(np.abs(got - ref)) / scale < 1e-13 * max(1, k[i]), (i, uplo, trans)
            # other triangle untouched (bitwise)
            other = np.triu(np.ones_like(ref, bool), 1) if uplo == "L" else np.tril(np.ones_like(ref, bool), -1)
            assert np.array_equal(got[other], C.get(i)[other])


@pytest.mark.parametrize("side", ["R", "L"])
@pytest.mark.parametrize("uplo", ["L", "U"])
@pytest.mark.parametrize("ta", ["N", "T"])
@pytest.mark.parametrize("diag", ["N", "U"])
def test_trsm(side, uplo, ta, diag):
    rng = np.random.default_rng(3)
    mn = [(0, 4), (1, 1), (5, 0), (70, 33), (64, 64), (130, 97), (3, 200), (257, 65)]
    m = [a for a, _ in mn]
    n = [b for _, b in mn]
    na = n if side == "R" else m  # order of the triangular A
    A = Mats([(ni, ni) for ni in na], rng)
    # well-conditioned triangular: boost the diagonal
    for i, ni in enumerate(na):
        if ni:
            blk = A.get(i)
            blk += 4 * np.eye(ni)
            full = A.host[A.off[i]: A.off[i] + A.ld[i] * ni].reshape((A.ld[i], ni), order="F")
            full[:ni] = blk
    A.dev.copy_(torch.from_numpy(A.host))
    B = Mats(list(zip(m, n)), rng)
    alpha = 0.75
    vb.vbatched_dtrsm(side, uplo, ta, diag, _ints(m), _ints(n), alpha, A.ptrs, A.d_ld, B.ptrs, B.d_ld,
                      len(m), max(m), max(n))
    torch.cuda.synchronize()
    out = B.result()
    for i in range(len(m)):
        ref = oracle.dtrsm(side, uplo, ta, diag, alpha, A.get(i), B.get(i))
        got = B.get(i, out)
        if ref.size:
            scale = max(1.0, np.max(np.abs(ref)))
            assert np.max(np.abs(got - ref)) / scale < 1e-12, (i, side, uplo, ta, diag)


def test_blas_argument_errors():
    z = _ints([1])
    assert vb.vbatched_dgemm("X", "N", z, z, z, 1, 0, z, 0, z, 0, 0, z, 1, 1, 1, 1, check=False) == -1
    assert vb.vbatched_dgemm("N", "Q", z, z, z, 1, 0, z, 0, z, 0, 0, z, 1, 1, 1, 1, check=False) == -2
    assert vb.vbatched_dgemm("N", "N", z, z, z, 1, 0, z, 0, z, 0, 0, z, -1, 1, 1, 1, check=False) == -14
    assert vb.vbatched_dsyrk("Q", "N", z, z, 1, 0, z, 0, 0, z, 1, 1, 1, check=False) == -1
    assert vb.vbatched_dtrsm("X", "L", "T", "N", z, z, 1, 0, z, 0, z, 1, 1, 1, check=False) == -1
    assert vb.vbatched_dtrsm("R", "L", "T", "N", z, z, 1, 0, z, 0, z, 0, 1, 1, check=False) == 0
