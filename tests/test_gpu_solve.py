"""GPU parity of the vbatched solve: vbatched_dpotrs / vbatched_dposv
against the oracle's LAPACK-DPOTRS/DPOSV composition (oracle.dposv), uplo 'L' and 'U', sizes on
every factorisation path, ragged right-hand sides (including 0), a non-SPD matrix (B must stay
unchanged) and an exact integer family (X bit-exact)."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ipps_abdelfattahhtd16_b200 as vb
import vbgen
from harness import DeviceBatch

pytestmark = pytest.mark.gpu

SIZES = [1, 7, 32, 33, 100, 128, 129, 300, 513, 64]
NRHS = [1, 3, 0, 5, 2, 16, 1, 8, 4, 6]
FAIL = {4: 50}  # slot -> failing pivot


def _rhs(nrhs_list, n_list, rng, x0=None):
    ld = [max(1, n + 1) for n in n_list]  # ragged, odd leading dimensions
    off = np.concatenate([[0], np.cumsum([l * r for l, r in zip(ld, nrhs_list)])]).astype(np.int64)
    host = np.zeros(max(1, int(off[-1])))
    blocks = []
    for i, (n, r) in enumerate(zip(n_list, nrhs_list)):
        b = rng.standard_normal((ld[i], r)) if x0 is None else x0[i]
        if x0 is not None:
            b = np.vstack([b, np.zeros((ld[i] - n, r))])
        host[off[i]: off[i] + ld[i] * r] = b.ravel(order="F")
        blocks.append(b[:n].copy())
    dev = torch.from_numpy(host.copy()).cuda()
    ptrs = torch.from_numpy(dev.data_ptr() + 8 * off[:-1]).cuda()
    d_ld = torch.tensor(ld, dtype=torch.int32, device="cuda")
    get = lambda i, a: a[off[i]: off[i] + ld[i] * nrhs_list[i]].reshape((ld[i], nrhs_list[i]), order="F")
    return dev, ptrs, d_ld, blocks, get


@pytest.mark.parametrize("uplo", ["L", "U"])
def test_posv_matches_oracle(uplo):
    rng = np.random.default_rng(11)
    n = np.array(SIZES, dtype=np.int32)
    db = DeviceBatch(n, seed=31)
    mats = {}
    for i, ni in enumerate(SIZES):
        A = vbgen.f1_matrix(31, i, ni)
        if i in FAIL:
            k = FAIL[i]
            A[k - 1, k - 1] = -A[k - 1, k - 1]
        mats[i] = A
        db.set_matrix(i, A, uplo=uplo)
    dev, ptrs, d_ld, B, get = _rhs(NRHS, SIZES, rng)
    before = dev.cpu().numpy()
    nrhs = torch.tensor(NRHS, dtype=torch.int32, device="cuda")
    vb.vbatched_dposv(uplo, db.d_n, nrhs, db.d_ptrs, db.d_ldda, ptrs, d_ld, db.d_info, len(SIZES),
                      max(SIZES), max(NRHS))
    torch.cuda.synchronize()
    after = dev.cpu().numpy()
    info = db.info()
    for i, ni in enumerate(SIZES):
        X, _, info_o = oracle.dposv(uplo, mats[i], B[i])
        assert info[i] == info_o == FAIL.get(i, 0), i
        got = get(i, after)
        if info_o != 0 or NRHS[i] == 0:  # untouched, including the padding row
            assert np.array_equal(got.view(np.uint64), get(i, before).view(np.uint64)), i
            continue
        assert np.max(np.abs(got[:ni] - X)) <= 1e-12 * max(1.0, np.max(np.abs(X))), i
        assert np.array_equal(got[ni:].view(np.uint64), get(i, before)[ni:].view(np.uint64)), i


@pytest.mark.parametrize("uplo", ["L", "U"])
def test_potrs_exact_integer_family(uplo):
    """A = L L^T, L integer unit-lower, B = A X0 (integers): the factor and every substitution
    step are exact, so X must equal X0 bit for bit (dpotrf then dpotrs as separate calls)."""
    rng = np.random.default_rng(5)
    sizes = [3, 40, 96, 160, 300]
    nrhs_l = [2, 4, 1, 3, 5]
    n = np.array(sizes, dtype=np.int32)
    db = DeviceBatch(n, seed=5)
    x0s = []
    for i, ni in enumerate(sizes):
        L = np.tril(rng.integers(-1, 2, size=(ni, ni)), -1).astype(np.int64) + np.eye(ni, dtype=np.int64)
        db.set_matrix(i, (L @ L.T).astype(np.float64), uplo=uplo)
        X0 = rng.integers(-3, 4, size=(ni, nrhs_l[i])).astype(np.int64)
        x0s.append(((L @ (L.T @ X0)).astype(np.float64), X0.astype(np.float64)))
    dev, ptrs, d_ld, _, get = _rhs(nrhs_l, sizes, rng, x0=[b for b, _ in x0s])
    db.dpotrf(uplo=uplo)
    nrhs = torch.tensor(nrhs_l, dtype=torch.int32, device="cuda")
    vb.vbatched_dpotrs(uplo, db.d_n, nrhs, db.d_ptrs, db.d_ldda, ptrs, d_ld, len(sizes), max(sizes),
                       max(nrhs_l))
    torch.cuda.synchronize()
    assert np.all(db.info() == 0)
    out = dev.cpu().numpy()
    for i, ni in enumerate(sizes):
        assert np.array_equal(get(i, out)[:ni], x0s[i][1]), i


def test_solve_argument_errors():
    z = torch.zeros(1, dtype=torch.int32, device="cuda")
    assert vb.vbatched_dpotrs("X", z, z, z, z, z, z, 1, 1, 1, check=False) == -1
    assert vb.vbatched_dpotrs("L", z, z, z, z, z, z, -1, 1, 1, check=False) == -8
    assert vb.vbatched_dposv("L", z, z, z, z, z, z, z, 1, -1, 1, check=False) == -10
    assert vb.vbatched_dposv("U", z, z, z, z, z, z, z, 0, 1, 1, check=False) == 0
