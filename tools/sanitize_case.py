"""Workloads for compute-sanitizer (tools/sanitize.sh): small enough for the tools' replay
overhead, covering every kernel and protocol of one vbatched_dpotrf call.

  c1     BASELINE C1 (100 x U{1..32}): the direct warp kernel.
  mixed  200 matrices spanning all three factorisation kernels (n in 1..700), 'L' and 'U',
         roundup-32 and odd ldda (the cp.async gather instead of TMA bulk copies), failing
         pivots (-> early termination, the TMA ring drain, the look-ahead barrier exits).
  lu     vbatched_dgetrf on 40 general matrices (square and rectangular, n < 300).
  qr     vbatched_dgeqrf on 40 general matrices (square, wide and tall).
  host   vbatched_dpotrf_host on pinned memory in several chunks (staircase transfers).
  z      vbatched_zpotrf / vbatched_cpotrf with non-HPD matrices.
Each case checks info against the expected values so a silent corruption also fails.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbgen  # noqa: E402
from harness import DeviceBatch  # noqa: E402


def c1():
    n = vbgen.sizes("C1")
    db = DeviceBatch(n, seed=1).fill(poison=True)
    db.dpotrf(max_n=32)
    torch.cuda.synchronize()
    assert np.all(db.info() == 0)


def mixed_gather():
    """The mixed batch with odd ldda only: every chunk of the blocked kernel goes through the
    8-byte cp.async gather (generic-proxy writes racecheck can follow) instead of TMA."""
    rng = np.random.default_rng(201)
    n = np.concatenate([rng.integers(33, 129, 30), rng.integers(129, 501, 40)]).astype(np.int32)
    for uplo in ("L", "U"):
        db = DeviceBatch(n, seed=202, nonspd_mod=9, ldda_mode="odd").fill(poison=True, uplo=uplo)
        db.dpotrf(uplo=uplo)
        torch.cuda.synchronize()
        exp = np.array([vbgen.nonspd_k(202, g, int(n[g])) if g % 9 == 8 else 0 for g in range(len(n))])
        assert np.array_equal(db.info(), exp), uplo


def mixed(scale=1):
    rng = np.random.default_rng(200)
    n = np.concatenate([rng.integers(1, 33, 60 // scale), rng.integers(33, 129, 80 // scale),
                        rng.integers(129, 701, 60 // scale)]).astype(np.int32)
    for uplo in ("L", "U"):
        for mode in ("pad32", "odd"):
            db = DeviceBatch(n, seed=201, nonspd_mod=9, ldda_mode=mode).fill(poison=True, uplo=uplo)
            db.dpotrf(uplo=uplo)
            torch.cuda.synchronize()
            info = db.info()
            exp = np.array([vbgen.nonspd_k(201, g, int(n[g])) if g % 9 == 8 else 0 for g in range(len(n))])
            assert np.array_equal(info, exp), (uplo, mode)
    print("mixed ok")


def lu():
    from harness import LUBatch
    rng = np.random.default_rng(7)
    n = rng.integers(1, 300, 40).astype(np.int32)
    m = n.copy()
    m[::5] = np.maximum(1, n[::5] // 2)
    lb = LUBatch(m, n, seed=3).fill()
    lb.getrf()
    torch.cuda.synchronize()
    assert np.all(lb.info() == 0)


def qr():
    from harness import QRBatch
    rng = np.random.default_rng(9)
    n = rng.integers(1, 300, 40).astype(np.int32)
    m = n.copy()
    m[::5] = np.maximum(1, n[::5] // 2)
    m[1::5] = n[1::5] + 37
    qb = QRBatch(m, n, seed=4).fill()
    qb.geqrf()
    torch.cuda.synchronize()
    assert np.all(qb.info() == 0)


def host():
    """vbatched_dpotrf_host on pinned memory, chunked: staircase and whole-block transfers."""
    import ctypes

    import paper_conf_ipps_abdelfattahhtd16_b200 as vb
    rng = np.random.default_rng(11)
    n = np.concatenate([rng.integers(1, 128, 30), rng.integers(128, 400, 20)]).astype(np.int32)
    dev = DeviceBatch(n, seed=12, nonspd_mod=7).fill(poison=True)
    torch.cuda.synchronize()
    src = dev.arena.cpu().numpy()
    hp = vb.vbatched_host_alloc(src.nbytes)
    try:
        host = np.ctypeslib.as_array((ctypes.c_double * src.size).from_address(hp))
        host[:] = src
        info = np.zeros(dev.B, np.int32)
        vb.vbatched_dpotrf_host("L", dev.n, (hp + 8 * dev.off).astype(np.int64), dev.ldda, info,
                                dev.B, int(n.max()), workspace_bytes=3 * 4 << 20)
        exp = np.array([vbgen.nonspd_k(12, g, int(n[g])) if g % 7 == 6 else 0 for g in range(len(n))])
        assert np.array_equal(info, exp)
    finally:
        vb.vbatched_host_free(hp)


def z():
    from harness import ZBatch
    n = np.array([1, 5, 16, 17, 40, 100, 200], np.int32)
    for single in (False, True):
        zb = ZBatch(n, seed=5, single=single, nonspd_mod=3).fill()
        zb.potrf()
        torch.cuda.synchronize()
        exp = [vbgen.nonspd_k(5, i, int(n[i])) if i % 3 == 2 else 0 for i in range(len(n))]
        assert list(zb.info()) == exp


if __name__ == "__main__":
    {"c1": c1, "mixed": mixed, "mixed_small": lambda: mixed(4), "mixed_gather": mixed_gather, "lu": lu, "qr": qr, "host": host, "z": z}[sys.argv[1]]()
    print("case ok", sys.argv[1])
