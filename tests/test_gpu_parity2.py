"""GPU parity, round 2 coverage (VERDICT r01 "What's missing" #3-#4, "What's weak" #2):

* F2 matrices (SURVEY.md §8(c) reading #9: Q diag(lambda) Q^T, lambda log-uniform in
  [1, 1e4], so kappa = 1e4) through every kernel path — warp (n <= 32), small (32 < n <= 128),
  blocked (n > 128) — and both storage triangles, at north_star's gates: info exact, backward
  error <= 10, row-scaled difference to the oracle's L <= 1e-10 (kappa <= 1e4 clause).
* the LAPACK-like interface without max_n (vbatched_dpotrf_nomax, vbatched_spotrf_nomax)
  compared with the oracle itself, not only with the max-given call.
* an independent GPU backward-error checker (harness.gpu_backward_errors: torch FP64 bmm),
  validated against the long-double oracle; the all-matrix C5 use is in test_gpu_potrf.
"""
import numpy as np
import pytest
import torch

import oracle
import vbgen
from harness import DeviceBatch, compare_with_oracle, gpu_backward_errors

pytestmark = pytest.mark.gpu

F2_SIZES = [1, 2, 5, 16, 17, 31, 32, 33, 48, 64, 65, 96, 127, 128, 129, 160, 192, 256, 257,
            384, 512, 513, 700, 1024]


@pytest.mark.parametrize("uplo", ["L", "U"])
def test_f2_kappa_1e4_all_paths(uplo):
    sizes = [n for n in F2_SIZES for _ in range(2)]
    n = np.array(sizes, dtype=np.int32)
    db = DeviceBatch(n, seed=31)
    inputs = {}
    for i, ni in enumerate(sizes):
        inputs[i] = vbgen.f2_matrix(31, i, ni)
        db.set_matrix(i, inputs[i], uplo=uplo)
    db.dpotrf(uplo=uplo)
    torch.cuda.synchronize()
    info = db.info()
    worst = {"bwd": 0.0, "rowscaled": 0.0}
    for i, ni in enumerate(sizes):
        blk = db.block(i)
        G = blk[:ni, :ni] if uplo == "L" else blk[:ni, :ni].T.copy()
        r = compare_with_oracle(inputs[i], G, info[i])
        assert r["ok"], (i, ni, r)
        worst["bwd"] = max(worst["bwd"], r["bwd"])
        worst["rowscaled"] = max(worst["rowscaled"], r["rowscaled"])
    assert np.all(info == 0)
    print("F2", uplo, worst)


def test_f2_kappa_1e4_device_batch_mixed():
    """A C3-like mixed batch (300 matrices, U{1..512}) of F2 matrices in one call, so the three
    kernels run concurrently as in the bench."""
    rng = np.random.default_rng(77)
    sizes = rng.integers(1, 513, 300).astype(np.int32)
    db = DeviceBatch(sizes, seed=32)
    inputs = {}
    for i, ni in enumerate(sizes):
        inputs[i] = vbgen.f2_matrix(32, i, int(ni))
        db.set_matrix(i, inputs[i])
    db.dpotrf()
    torch.cuda.synchronize()
    info = db.info()
    for i in range(db.B):
        r = compare_with_oracle(inputs[i], db.block(i), info[i])
        assert r["ok"], (i, r)


@pytest.mark.parametrize("cfg,count", [("C2", 600), ("C4", 400)])
def test_nomax_against_oracle(cfg, count):
    import paper_conf_ipps_abdelfattahhtd16_b200 as vb
    c = vbgen.CONFIGS[cfg]
    n = vbgen.sizes(c)[:count]
    db = DeviceBatch(n, seed=c.seed, nonspd_mod=c.nonspd_mod).fill(poison=True)
    vb.vbatched_dpotrf_nomax("L", db.d_n, db.d_ptrs, db.d_ldda, db.d_info, db.B)
    torch.cuda.synchronize()
    info = db.info()
    for i in range(db.B):
        r = compare_with_oracle(db.host_matrix_input(i), db.block(i), info[i])
        assert r["ok"], (i, r)
    if c.nonspd_mod:
        assert (info > 0).sum() == count // 20


def test_spotrf_nomax_against_oracle():
    import paper_conf_ipps_abdelfattahhtd16_b200 as vb
    c = vbgen.CONFIGS["C4"]
    n = vbgen.sizes(c)[:300]
    db = DeviceBatch(n, seed=c.seed, nonspd_mod=c.nonspd_mod, dtype="f32").fill(poison=True)
    vb.vbatched_spotrf_nomax("L", db.d_n, db.d_ptrs, db.d_ldda, db.d_info, db.B)
    torch.cuda.synchronize()
    info = db.info()
    for i in range(0, db.B, 3):
        ni = int(n[i])
        A32 = db.host_matrix_input(i).astype(np.float32)
        L32, info_o = oracle.spotrf(A32)
        assert info[i] == info_o, i
        k = ni if info_o == 0 else info_o - 1
        if k:
            G = db.block(i)[:ni, :ni].astype(np.float64)
            assert oracle.rowscaled_diff(G, L32.astype(np.float64), k) <= 8 * k * 2.0 ** -24
            assert oracle.backward_error_f32(A32, np.tril(G), int(info[i])) <= 10.0


def test_gpu_backward_error_checker_matches_oracle():
    """The torch checker used for the all-matrix C5 gate agrees with the long-double oracle's
    backward error (absolute 0.5 on ratios that are O(0.1)), and flags a perturbed factor."""
    n = np.concatenate([vbgen.sizes("C3")[:150], np.array([1, 2, 1000, 1024], np.int32)])
    db = DeviceBatch(n, seed=3, nonspd_mod=20).fill()
    db.dpotrf()
    torch.cuda.synchronize()
    info = db.info()
    gb = gpu_backward_errors(db)
    assert np.all(np.isnan(gb[info != 0])) and np.all(np.isfinite(gb[(info == 0) & (n > 0)]))
    for i in range(0, db.B, 5):
        if info[i] != 0:
            continue
        ob = oracle.backward_error(db.host_matrix_input(i), db.block(i)[: n[i], : n[i]].copy(order="F"), 0)
        assert abs(ob - gb[i]) <= 0.5, (i, ob, gb[i])
    # a 1e-6 relative perturbation of one entry (L[5,0] of the n = 1024 factor) must push the
    # ratio far above 10 (about 2 |dL| ||l_0|| / (n ||A||_F eps) ~ 1e2)
    j = int(np.argmax(n))
    db.arena[int(db.off[j]) + 5] *= 1 + 1e-6
    gb2 = gpu_backward_errors(db)
    assert gb2[j] > 10 and np.nanmax(np.delete(gb2, j)) <= 10


def test_stream_successor_sees_all_chained_grids():
    """The factorisation grids are PDL-chained (blocked -> small -> warp); a stream-ordered
    successor enqueued right after the call (no host sync) must see every grid's results:
    the chained grids wait for their upstream before exiting (transitive
    completion). The copies are taken by torch kernels on the same stream."""
    n = np.concatenate([np.full(40, 1024, np.int32), vbgen.sizes("C2")[:600]])
    db = DeviceBatch(n, seed=9, nonspd_mod=7).fill()
    s = torch.cuda.Stream()
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        db.dpotrf(stream=s)
        info_copy = db.d_info.clone()
        arena_copy = db.arena.clone()
    s.synchronize()
    assert torch.equal(info_copy, db.d_info)
    assert torch.equal(arena_copy.view(torch.int64), db.arena.view(torch.int64))
    assert (db.info() > 0).sum() == sum(1 for g in range(len(n)) if g % 7 == 6)


def test_release_host_staging_and_reuse():
    import paper_conf_ipps_abdelfattahhtd16_b200 as vb
    n = vbgen.sizes("C3")[:100]
    dev = DeviceBatch(n, seed=3).fill()
    torch.cuda.synchronize()
    host0 = dev.arena.cpu().numpy().copy()
    outs = []
    for _ in range(2):
        host = host0.copy()
        ptrs = (host.ctypes.data + 8 * dev.off).astype(np.int64)
        info = np.full(dev.B, -99, dtype=np.int32)
        vb.vbatched_dpotrf_host("L", dev.n, ptrs, dev.ldda, info, dev.B, int(n.max()))
        assert np.all(info == 0)
        outs.append(host)
        vb.vbatched_release_host_staging()
    assert np.array_equal(outs[0].view(np.uint64), outs[1].view(np.uint64))
