"""Input generator (vbgen) pins: seeded size anchors, distribution shape (§IV-B),
F1 properties, non-SPD injection. CPU only; the device twin is pinned in test_gpu_paths.py."""
import json
import os

import numpy as np
import pytest

import vbgen

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_splitmix64_known_values():
    # Reference values of the SplitMix64 finaliser applied to 0 and 1 (standard test vectors:
    # the first outputs of the SplitMix64 generator seeded with 0 are mix(0+gamma), ...).
    assert int(vbgen.splitmix64(np.uint64(0))) == 0xE220A8397B1DCDAF
    assert int(vbgen.splitmix64(np.uint64(0x9E3779B97F4A7C15))) == 0x6E789E6AA1B965F4


@pytest.mark.parametrize("name,nmin,nmax,sumf,tol", [
    ("C1", 1, 32, 0.29e6, 0.02), ("C2", 1, 128, 0.5444e9, 2e-4), ("C3", 1, 512, 33.331e9, 2e-5),
    ("C4", 1, 512, 15.862e9, 5e-5), ("C5", 1, 1024, 3609.47e9, 5e-6)])
def test_seeded_size_anchors(name, nmin, nmax, sumf, tol):
    """Regression anchors recorded in SURVEY.md §8(d) 'Seeded actuals'."""
    n = vbgen.sizes(name)
    cfg = vbgen.CONFIGS[name]
    assert len(n) == cfg.batch and n.dtype == np.int32
    assert n.min() >= nmin and n.max() <= nmax
    assert abs(vbgen.expected_flops(n) / sumf - 1) < tol  # tol = half a unit of the anchor's last digit


def test_uniform_histogram_shape():
    g = json.load(open(os.path.join(GOLD, "e1_histogram.json")))
    cfg = vbgen.Config("E1", g["batch"], "uniform", g["nmax"], 123)
    n = vbgen.sizes(cfg)
    cnt = np.bincount(n, minlength=g["nmax"] + 1)[1:]
    assert np.mean(cnt == 0) <= g["frac_unseen_max"]
    assert np.mean((cnt >= 1) & (cnt <= 5)) >= g["frac_1_to_5_min"]


def test_gauss_sizes():
    n = vbgen.sizes("C4")
    assert abs(n.mean() - 256) < 10 and 80 < n.std() < 110
    assert n.min() >= 1 and n.max() <= 512


def test_f1_symmetric_spd_and_distinct():
    for n in (1, 2, 33, 100):
        A = vbgen.f1_matrix(5, 7, n)
        assert np.array_equal(A, A.T)
        off = A[~np.eye(n, dtype=bool)]
        if n > 1:
            assert off.min() >= 0 and off.max() < 1
        assert np.all(np.diag(A) >= n) and np.all(np.diag(A) < n + 1)
        assert np.linalg.eigvalsh(A).min() >= 1 - 1e-9
    assert not np.array_equal(vbgen.f1_matrix(5, 7, 10), vbgen.f1_matrix(5, 8, 10))
    assert not np.array_equal(vbgen.f1_matrix(5, 7, 10), vbgen.f1_matrix(6, 7, 10))


def test_nonspd_selection():
    cfg = vbgen.CONFIGS["C4"]
    sel = [g for g in range(cfg.batch) if vbgen.is_nonspd(cfg, g)]
    assert len(sel) == 100
    n = vbgen.sizes(cfg)
    ks = [vbgen.nonspd_k(cfg.seed, g, int(n[g])) for g in sel]
    assert all(1 <= k <= n[g] for k, g in zip(ks, sel))
    A = vbgen.config_matrix(cfg, 19)
    k = vbgen.nonspd_k(cfg.seed, 19, int(n[19]))
    assert A[k - 1, k - 1] < 0


def test_arena_layout_alignment():
    n = vbgen.sizes("C2")
    ld = vbgen.ldda_for(n)
    off, tot = vbgen.arena_layout(n, ld)
    assert np.all(off % 32 == 0)
    assert np.all(ld >= n) and np.all(ld % 32 == 0)
    assert tot >= int(np.sum(ld.astype(np.int64) * n))
    odd = vbgen.ldda_for(n, "odd")
    assert np.all(odd % 2 == 1) and np.all(odd >= n)
