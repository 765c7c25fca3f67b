"""GPU parity of vbatched_dgetrf (the LU extension of PAPER.md:2279-2285)
against the CPU oracle (oracle_dgetrf): info and ipiv bit-exact, backward error <= 10,
row-scaled factor difference <= 1e-10, exact dyadic family bit-exact, padding rows untouched."""
import numpy as np
import pytest
import torch

import vbgen
from harness import LUBatch, compare_lu_with_oracle

pytestmark = pytest.mark.gpu
POISON = np.uint64(vbgen.NAN_POISON_BITS)

SHAPES = [(1, 1), (2, 2), (5, 3), (3, 5), (15, 15), (16, 16), (17, 17), (31, 32), (32, 31),
          (33, 33), (48, 16), (16, 48), (64, 64), (65, 65), (100, 37), (37, 100), (127, 128),
          (128, 128), (129, 129), (200, 200), (255, 256), (256, 256), (257, 257), (300, 120),
          (120, 300), (511, 511), (512, 512), (513, 513), (700, 650), (1024, 1024)]


def _check_all(lb, idxs=None):
    torch.cuda.synchronize()
    info = lb.info()
    bad = []
    for i in (range(lb.B) if idxs is None else idxs):
        m, n = int(lb.m[i]), int(lb.n[i])
        if m == 0 or n == 0:
            continue
        r = compare_lu_with_oracle(lb.inputs[i], lb.block(i), lb.ipiv_of(i), info[i])
        if not r["ok"]:
            bad.append((i, r))
        blk = lb.block(i)
        if blk.shape[0] > m:
            assert np.all(blk[m:].view(np.uint64) == POISON), i
    assert not bad, bad[:4]
    return info


@pytest.mark.parametrize("pad", [0, 5])
def test_getrf_shapes(pad):
    m = np.array([s[0] for s in SHAPES], np.int32)
    n = np.array([s[1] for s in SHAPES], np.int32)
    lb = LUBatch(m, n, seed=41, ldda=np.maximum(1, m) + pad).fill()
    lb.getrf()
    info = _check_all(lb)
    assert np.all(info == 0)


def test_getrf_exact_dyadic_family():
    """A = P0 L U with dyadic |l| <= 1/2 and dominant power-of-two pivots: the GPU must find the
    same interchanges and return U and the pivot rows of L bit-exactly (TRSM / GEMM included)."""
    rng = np.random.default_rng(8)
    shapes = [(40, 40), (70, 33), (33, 70), (130, 130), (257, 200)]
    m = np.array([s[0] for s in shapes], np.int32)
    n = np.array([s[1] for s in shapes], np.int32)
    lb = LUBatch(m, n, seed=1)
    exp = {}
    for i, (mi, ni) in enumerate(shapes):
        k = min(mi, ni)
        L = np.tril(rng.choice([-0.5, -0.25, 0.0, 0.25, 0.5], size=(mi, k)), -1) + np.eye(mi, k)
        U = np.triu(rng.integers(-3, 4, size=(k, ni)).astype(np.float64), 1)
        U[np.arange(k), np.arange(k)] = rng.choice([-8.0, 8.0, 4.0, -4.0], size=k)
        A = L @ U
        perm = rng.permutation(mi)
        lb.set_matrix(i, A[perm])
        exp[i] = (L, U, k)
    lb.getrf()
    torch.cuda.synchronize()
    assert np.all(lb.info() == 0)
    for i in range(lb.B):
        L, U, k = exp[i]
        F = lb.block(i)[: lb.m[i]]
        assert np.array_equal(np.triu(F[:k, :]), U), i
        assert np.array_equal(np.tril(F[:k, :k], -1) + np.eye(k), L[:k]), i
        r = compare_lu_with_oracle(lb.inputs[i], lb.block(i), lb.ipiv_of(i), 0)
        assert r["ok"], r


def test_getrf_singular_and_invalid():
    shapes = [(6, 6), (40, 40), (100, 100), (5, 5), (7, 7), (9, 4), (120, 120)]
    m = np.array([s[0] for s in shapes], np.int32)
    n = np.array([s[1] for s in shapes], np.int32)
    lb = LUBatch(m, n, seed=3).fill()
    lb.set_matrix(0, np.ones((6, 6)))                 # info 2
    B = vbgen.g1_matrix(3, 1, 40, 40); B[:, 17] = 0.0  # info 18
    lb.set_matrix(1, B)
    C = vbgen.g1_matrix(3, 2, 100, 100); C[:, 0] = 0.0  # info 1 (first panel, first column)
    lb.set_matrix(2, C)
    before = {i: lb.block(i).copy() for i in (3, 4, 6)}
    bad_m, bad_ld = lb.d_m.clone(), lb.d_ldda.clone()
    bad_m[3] = -1       # -1
    bad_ld[4] = 6       # ldda < m: -4
    from paper_conf_ipps_abdelfattahhtd16_b200 import vbatched_dgetrf
    vbatched_dgetrf(bad_m, lb.d_n, lb.d_ptrs, bad_ld, lb.d_ipiv, lb.d_info, lb.B, 100, 100)  # 120 > 100: -9
    torch.cuda.synchronize()
    info = lb.info()
    assert list(info[:5]) == [2, 18, 1, -1, -4] and info[6] == -9 and info[5] == 0, info
    for i in (3, 4, 6):
        assert np.array_equal(lb.block(i).view(np.uint64), before[i].view(np.uint64))
    _check_all(lb, idxs=[0, 1, 2, 5])


def test_getrf_mixed_batch_c3_like():
    """500 square matrices, n ~ U{1..512} (BASELINE C3's size law), plus 5 % rectangular."""
    rng = np.random.default_rng(3)
    n = rng.integers(1, 513, 500).astype(np.int32)
    m = n.copy()
    m[::20] = np.maximum(1, (n[::20] * 3) // 4)
    lb = LUBatch(m, n, seed=5).fill()
    lb.getrf()
    info = _check_all(lb, idxs=range(0, 500, 3))
    assert np.all(info == 0)


def test_getrf_stream_and_repeat_bit_identical():
    n = np.random.default_rng(4).integers(1, 300, 200).astype(np.int32)
    a = LUBatch(n, n, seed=9).fill()
    b = LUBatch(n, n, seed=9).fill()
    s = torch.cuda.Stream()
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        a.getrf(stream=s)
    s.synchronize()
    b.getrf()
    torch.cuda.synchronize()
    assert torch.equal(a.ipiv, b.ipiv)
    for i in range(a.B):
        assert np.array_equal(a.block(i).view(np.uint64), b.block(i).view(np.uint64)), i


# the two-level blocking's edges (SURVEY §8(f) NEXT-4 built with 16-column steps inside 64-column
# blocks): block boundaries in m, n and min(m, n); a last block narrower than 64 with trailing
# columns (wide), a full block with no rows below it (kmax = 64), tall matrices ending on a block
BLOCK_EDGES = [(63, 63), (64, 200), (200, 64), (65, 130), (130, 65), (70, 130), (130, 70),
               (127, 129), (129, 127), (191, 192), (192, 193), (193, 191), (250, 70), (70, 250)]


@pytest.mark.parametrize("pad", [0, 3])
def test_getrf_block_edges(pad):
    m = np.array([s[0] for s in BLOCK_EDGES], np.int32)
    n = np.array([s[1] for s in BLOCK_EDGES], np.int32)
    lb = LUBatch(m, n, seed=43, ldda=np.maximum(1, m) + pad).fill()
    lb.getrf()
    info = _check_all(lb)
    assert np.all(info == 0)
