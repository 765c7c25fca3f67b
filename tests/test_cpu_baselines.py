"""The bench's CPU library baselines (MKL / scipy's OpenBLAS dpotrf one core per matrix,
cpu_baselines/) agree with the oracle on info and to rounding on L (it is a reported baseline, so this only checks
that the number it produces comes from correct factorisations)."""
import numpy as np
import pytest

import cpu_baselines
import oracle
import vbgen


@pytest.mark.parametrize("which", ["mkl", "openblas"])
def test_lapack_batch_matches_oracle(which):
    lib_path = None
    if which == "openblas":
        lib_path = cpu_baselines.openblas_path()
        if lib_path is None:
            pytest.skip("scipy's bundled OpenBLAS not present")
    n = np.array([0, 1, 5, 33, 100, 257, 64], dtype=np.int32)
    ld = vbgen.ldda_for(n)
    off, tot = vbgen.arena_layout(n, ld)
    arena = np.zeros(tot)
    for j, nn in enumerate(n.tolist()):
        if nn:
            blk = arena[off[j]: off[j] + int(ld[j]) * nn].reshape((int(ld[j]), nn), order="F")
            blk[:nn, :] = vbgen.f1_matrix(11, j, nn, j == 4)
    a_or = arena.copy()
    _, info = cpu_baselines.dpotrf_batch(arena, off, n, ld, 2, lib_path=lib_path)
    info_or = oracle.dpotrf_batch(a_or, off, n, ld, 2)
    assert np.array_equal(info, info_or) and info[4] == vbgen.nonspd_k(11, 4, 100)
    for j, nn in enumerate(n.tolist()):
        if nn == 0 or info[j]:
            continue
        b1 = arena[off[j]: off[j] + int(ld[j]) * nn].reshape((int(ld[j]), nn), order="F")[:nn]
        b2 = a_or[off[j]: off[j] + int(ld[j]) * nn].reshape((int(ld[j]), nn), order="F")[:nn]
        assert np.allclose(np.tril(b1), np.tril(b2), rtol=0, atol=1e-12 * nn)
        assert np.array_equal(np.triu(b1, 1), np.triu(b2, 1))  # upper never written
