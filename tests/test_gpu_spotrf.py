"""GPU parity of vbatched_spotrf (FP32 storage, FP64 arithmetic on the
DMMA tensor cores) against the FP32 oracle (oracle_spotrf_lower): info exact (robust injected
failures), factor within 8 n eps32 (row-scaled) of the oracle's, FP32 backward error <= 10,
exact integer families bit-exact, the unreferenced triangle and padding untouched."""
import numpy as np
import pytest
import torch

import oracle
import vbgen
from harness import DeviceBatch

pytestmark = pytest.mark.gpu
POISON32 = np.uint32(0x7FC0BEEF)
EDGE = [1, 2, 31, 32, 33, 64, 65, 127, 128, 129, 192, 255, 256, 257, 320, 511, 512, 513, 700, 1024]


def _check(db, i, A32, uplo="L"):
    n = int(db.n[i])
    blk = db.block(i)
    info = int(db.info()[i])
    L32, info_o = oracle.spotrf(A32)
    assert info == info_o, (i, n, info, info_o)
    k = n if info == 0 else info - 1
    G = blk[:n, :n] if uplo == "L" else blk[:n, :n].T
    if k:
        rs = oracle.rowscaled_diff(G.astype(np.float64), L32.astype(np.float64), k)
        assert rs <= 8 * max(k, 1) * 2.0 ** -24, (i, n, rs)
        assert oracle.backward_error_f32(A32, np.tril(G[:n, :n]), info) <= 10.0
    other = np.triu(np.ones((n, n), bool), 1) if uplo == "L" else np.tril(np.ones((n, n), bool), -1)
    assert np.all(blk[:n, :n].view(np.uint32)[other] == POISON32), i
    if blk.shape[0] > n:
        assert np.all(blk[n:].view(np.uint32) == POISON32), i


@pytest.mark.parametrize("ldda_mode", ["pad32", "tight"])
@pytest.mark.parametrize("uplo", ["L", "U"])
def test_spotrf_edge_sizes_and_failures(ldda_mode, uplo):
    n = np.array(EDGE, dtype=np.int32)
    db = DeviceBatch(n, seed=17, ldda_mode=ldda_mode, dtype="f32")
    fail = {5: 20, 9: 129, 14: 300, 18: 650}
    inputs = {}
    for i, ni in enumerate(EDGE):
        A = vbgen.f1_matrix(17, i, ni)
        if i in fail:
            k = fail[i]
            A[k - 1, k - 1] = -A[k - 1, k - 1]
        inputs[i] = A.astype(np.float32)
        db.set_matrix(i, inputs[i], uplo=uplo)
    db.dpotrf(uplo=uplo)
    torch.cuda.synchronize()
    assert list(db.info()) == [fail.get(i, 0) for i in range(len(EDGE))]
    for i in range(len(EDGE)):
        _check(db, i, inputs[i], uplo)


def test_spotrf_c3_sample_device_generated():
    """First 500 matrices of C4 (Gaussian sizes, 5 % non-SPD) generated on the device in FP32."""
    cfg = vbgen.CONFIGS["C4"]
    n = vbgen.sizes(cfg)[:500]
    db = DeviceBatch(n, seed=cfg.seed, nonspd_mod=cfg.nonspd_mod, dtype="f32").fill(poison=True)
    db.dpotrf()
    torch.cuda.synchronize()
    info = db.info()
    assert (info > 0).sum() == 25
    for i in range(0, 500, 9):
        A = db.host_matrix_input(i).astype(np.float32)
        _check(db, i, A)


def test_spotrf_exact_family():
    sizes = [40, 130, 300]
    n = np.array(sizes, dtype=np.int32)
    db = DeviceBatch(n, seed=2, dtype="f32")
    for i, ni in enumerate(sizes):
        j = np.arange(1, ni + 1)
        db.set_matrix(i, np.minimum.outer(j, j).astype(np.float32))
    db.dpotrf()
    torch.cuda.synchronize()
    assert np.all(db.info() == 0)
    for i, ni in enumerate(sizes):
        assert np.array_equal(np.tril(db.block(i)[:ni, :ni]), np.tril(np.ones((ni, ni), np.float32)))


def test_spotrf_nomax_equals_max_given():
    import paper_conf_ipps_abdelfattahhtd16_b200 as vb
    n = vbgen.sizes("C3")[:300]
    a = DeviceBatch(n, seed=3, nonspd_mod=20, dtype="f32").fill(poison=True)
    b = DeviceBatch(n, seed=3, nonspd_mod=20, dtype="f32").fill(poison=True)
    a.dpotrf()
    vb.vbatched_spotrf_nomax("L", b.d_n, b.d_ptrs, b.d_ldda, b.d_info, b.B)
    torch.cuda.synchronize()
    assert np.array_equal(a.info(), b.info())
    ha, hb = a.arena.cpu().numpy(), b.arena.cpu().numpy()
    for i in range(a.B):  # the matrices' blocks (the arenas' alignment gaps are never written)
        sl = slice(int(a.off[i]), int(a.off[i]) + int(a.ldda[i]) * max(int(n[i]), 0))
        assert np.array_equal(ha[sl].view(np.uint32), hb[sl].view(np.uint32)), i
