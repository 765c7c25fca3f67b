"""GPU parity of vbatched_zpotrf / vbatched_cpotrf (complex precisions,
PAPER.md:859-863) against the CPU oracle (oracle_zpotrf_lower / oracle_cpotrf_lower): info
exact; complex backward error <= 10; row-scaled difference <= 1e-10 (Z) / 8 n eps32 (C);
Gaussian-integer family bit-exact; the unreferenced triangle and padding untouched."""
import numpy as np
import pytest
import torch

import vbgen
from harness import ZBatch, compare_zpotrf_with_oracle

pytestmark = pytest.mark.gpu
SIZES = [1, 2, 7, 15, 16, 17, 31, 32, 33, 47, 48, 49, 64, 100, 127, 128, 129, 200, 256, 300, 511, 512, 700]


def _check(zb, uplo="L", idxs=None):
    torch.cuda.synchronize()
    info = zb.info()
    bad = []
    for i in (range(zb.B) if idxs is None else idxs):
        n = int(zb.n[i])
        blk = zb.block(i)
        G = blk[:n, :n] if uplo == "L" else blk[:n, :n].T.conj()
        r = compare_zpotrf_with_oracle(zb.inputs[i], G, info[i], single=zb.single)
        if not r["ok"]:
            bad.append((i, r))
        other = np.triu(np.ones((n, n), bool), 1) if uplo == "L" else np.tril(np.ones((n, n), bool), -1)
        assert np.all(np.isnan(blk[:n, :n][other])), i
        if blk.shape[0] > n:
            assert np.all(np.isnan(blk[n:])), i
    assert not bad, bad[:4]
    return info


@pytest.mark.parametrize("single", [False, True])
@pytest.mark.parametrize("uplo", ["L", "U"])
def test_zpotrf_sizes(single, uplo):
    n = np.array(SIZES, np.int32)
    zb = ZBatch(n, seed=51, single=single, ldda=n + 3).fill(uplo=uplo)
    zb.potrf(uplo=uplo)
    info = _check(zb, uplo)
    assert np.all(info == 0)


def test_zpotrf_gaussian_integer_family_bit_exact():
    rng = np.random.default_rng(61)
    sizes = [16, 33, 100, 257]
    zb = ZBatch(np.array(sizes, np.int32), seed=1)
    Ls = {}
    for i, n in enumerate(sizes):
        L = np.tril(rng.integers(-1, 2, (n, n)) + 1j * rng.integers(-1, 2, (n, n)), -1)
        L[np.arange(n), np.arange(n)] = rng.choice([1.0, 2.0, 4.0], n)
        Ls[i] = L
        zb.set_matrix(i, L @ L.conj().T)
    zb.potrf()
    torch.cuda.synchronize()
    assert np.all(zb.info() == 0)
    for i, n in enumerate(sizes):
        assert np.array_equal(np.tril(zb.block(i)[:n, :n]), Ls[i]), i


def test_zpotrf_nonspd_mixed_batch():
    """A C4-like mixed batch (Gaussian sizes, 5 % non-HPD at the hashed k) in both precisions."""
    n = vbgen.sizes("C4")[:300]
    for single in (False, True):
        zb = ZBatch(n, seed=4, single=single, nonspd_mod=20).fill()
        zb.potrf()
        info = _check(zb, idxs=range(0, 300, 2))
        exp = [vbgen.nonspd_k(4, i, int(n[i])) if i % 20 == 19 else 0 for i in range(300)]
        assert list(info) == exp
