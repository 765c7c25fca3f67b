"""GPU parity of vbatched_dgeqrf (the QR extension of PAPER.md:2279-2285)
against the CPU oracle (oracle_dgeqrf): reconstruction and orthogonality gates <= 10, compact
factor and tau within 1e-10 of the oracle's, triangular inputs untouched (tau = 0), padding rows
untouched, invalid arguments reported and their matrices untouched."""
import numpy as np
import pytest
import torch

import vbgen
from harness import QRBatch, compare_qr_with_oracle

pytestmark = pytest.mark.gpu
POISON = np.uint64(vbgen.NAN_POISON_BITS)
SHAPES = [(1, 1), (2, 2), (5, 3), (3, 5), (15, 15), (16, 16), (17, 17), (32, 31), (31, 32), (48, 16),
          (16, 48), (64, 64), (65, 65), (100, 37), (37, 100), (128, 128), (129, 129), (200, 200),
          (256, 256), (257, 257), (300, 120), (120, 300), (512, 512), (700, 650), (1024, 1024)]


def _check(qb, idxs=None):
    torch.cuda.synchronize()
    assert np.all(qb.info()[list(idxs) if idxs is not None else slice(None)] == 0)
    bad = []
    for i in (range(qb.B) if idxs is None else idxs):
        m, n = int(qb.m[i]), int(qb.n[i])
        r = compare_qr_with_oracle(qb.inputs[i], qb.block(i), qb.tau_of(i))
        if not r["ok"]:
            bad.append((i, r))
        blk = qb.block(i)
        if blk.shape[0] > m:
            assert np.all(blk[m:].view(np.uint64) == POISON), i
    assert not bad, bad[:4]


@pytest.mark.parametrize("pad", [0, 3])
def test_geqrf_shapes(pad):
    m = np.array([s[0] for s in SHAPES], np.int32)
    n = np.array([s[1] for s in SHAPES], np.int32)
    qb = QRBatch(m, n, seed=71, ldda=m + pad).fill()
    qb.geqrf()
    _check(qb)


def test_geqrf_triangular_and_invalid():
    shapes = [(20, 20), (40, 30), (9, 9), (6, 6), (300, 300)]
    m = np.array([s[0] for s in shapes], np.int32)
    n = np.array([s[1] for s in shapes], np.int32)
    qb = QRBatch(m, n, seed=72).fill()
    T0 = np.triu(vbgen.g1_matrix(72, 0, 20, 20))
    qb.set_matrix(0, T0)
    before = {i: qb.block(i).copy() for i in (2, 3, 4)}
    bad_m, bad_ld = qb.d_m.clone(), qb.d_ldda.clone()
    bad_m[2] = -1
    bad_ld[3] = 5
    from paper_conf_ipps_abdelfattahhtd16_b200 import vbatched_dgeqrf
    vbatched_dgeqrf(bad_m, qb.d_n, qb.d_ptrs, bad_ld, qb.d_tau, qb.d_info, qb.B, 200, 200)
    torch.cuda.synchronize()
    assert list(qb.info()) == [0, 0, -1, -4, -9]
    for i in (2, 3, 4):
        assert np.array_equal(qb.block(i).view(np.uint64), before[i].view(np.uint64)), i
    assert np.array_equal(qb.block(0), T0) and not qb.tau_of(0).any()  # H = I for every column
    _check(qb, idxs=[0, 1])


def test_geqrf_mixed_batch():
    rng = np.random.default_rng(5)
    n = rng.integers(1, 400, 300).astype(np.int32)
    m = n.copy()
    m[::4] = np.minimum(1024, n[::4] * 2)
    qb = QRBatch(m, n, seed=73).fill()
    qb.geqrf()
    _check(qb, idxs=range(0, 300, 4))


# the two-level blocking's edges (16-column steps inside 64-column blocks): block boundaries in m,
# n and min(m, n); a last block narrower than 64 with trailing columns (wide), a full block with no
# rows below it, tall matrices ending on a block
BLOCK_EDGES = [(63, 63), (64, 200), (200, 64), (65, 130), (130, 65), (70, 130), (130, 70),
               (127, 129), (129, 127), (191, 192), (192, 193), (193, 191), (250, 70), (70, 250)]


@pytest.mark.parametrize("pad", [0, 3])
def test_geqrf_block_edges(pad):
    m = np.array([s[0] for s in BLOCK_EDGES], np.int32)
    n = np.array([s[1] for s in BLOCK_EDGES], np.int32)
    qb = QRBatch(m, n, seed=44, ldda=np.maximum(1, m) + pad).fill()
    qb.geqrf()
    _check(qb)


def test_geqrf_sliced_batch():
    """More matrices than one ~4 GiB workspace slice at the declared bounds (1024 x 1024): the
    batch runs as several slices, every matrix still factored (sampled against the oracle)."""
    rng = np.random.default_rng(45)
    n = rng.integers(1, 40, 3000).astype(np.int32)
    m = (n + rng.integers(0, 20, 3000)).astype(np.int32)
    qb = QRBatch(m, n, seed=46).fill()
    qb.geqrf(max_m=1024, max_n=1024)
    _check(qb, idxs=list(range(0, 3000, 97)) + [2599, 2600, 2601, 2999])
