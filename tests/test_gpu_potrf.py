"""GPU parity of vbatched_dpotrf (through the C ABI) against the CPU oracle.

Gates (BASELINE.json north_star): info[] bit-exact; backward error
||A - L L^T||_F / (n ||A||_F eps) <= 10 (eps = 2^-53); row-scaled difference to the
oracle's L <= 1e-10 (kappa <= 1e4). Exact integer families must be bit-exact. The strict
upper triangle and padding rows must be bit-identical afterwards (NaN sentinels).
"""
import os

import numpy as np
import pytest
import torch

import vbgen
from harness import DeviceBatch, compare_with_oracle

pytestmark = pytest.mark.gpu

POISON = np.uint64(vbgen.NAN_POISON_BITS)


def _check_batch(db: DeviceBatch, idxs=None, exact_inputs=None):
    torch.cuda.synchronize()
    info = db.info()
    bad = []
    idxs = range(db.B) if idxs is None else idxs
    for i in idxs:
        n = int(db.n[i])
        blk = db.block(i)
        if n == 0:
            assert info[i] == 0
            continue
        A = db.host_matrix_input(i) if exact_inputs is None else exact_inputs[i]
        r = compare_with_oracle(A, blk, info[i])
        if not r["ok"]:
            bad.append((i, r))
    assert not bad, bad[:5]
    return info


def _check_sentinels(db: DeviceBatch, idxs=None):
    for i in (range(db.B) if idxs is None else idxs):
        n, ld = int(db.n[i]), int(db.ldda[i])
        if n <= 0:
            continue
        blk = db.block(i).view(np.uint64)
        mask = np.ones((ld, n), bool)
        mask[:n, :n] = np.triu(np.ones((n, n), bool), 1)  # strict upper of the n x n part
        mask[n:, :] = True
        assert np.all(blk[mask] == POISON), f"matrix {i} (n={n}, ld={ld}) touched outside lower"


def test_generator_device_matches_numpy():
    n = np.array([1, 2, 5, 33, 64, 130], dtype=np.int32)
    db = DeviceBatch(n, seed=7, nonspd_mod=3).fill(poison=True)
    torch.cuda.synchronize()
    for i in range(db.B):
        blk = db.block(i)
        A = db.host_matrix_input(i)
        low = np.tril(np.ones((n[i], n[i]), bool))
        assert np.array_equal(blk[: n[i]][low].view(np.uint64), A[low].view(np.uint64))
    _check_sentinels(db)


def test_c1_full_parity():
    n = vbgen.sizes("C1")
    db = DeviceBatch(n, seed=1).fill(poison=True)
    db.dpotrf(max_n=32)
    info = _check_batch(db)
    assert np.all(info == 0)
    _check_sentinels(db)


EDGE = [1, 2, 3, 7, 8, 15, 16, 17, 31, 32, 33, 34, 47, 48, 63, 64, 65, 96, 127, 128, 129, 130,
        159, 160, 161, 191, 255, 256, 257, 300, 383, 384, 385, 511, 512, 513]


@pytest.mark.parametrize("ldda_mode", ["pad32", "tight", "odd"])
def test_edge_sizes(ldda_mode):
    n = np.array(EDGE, dtype=np.int32)
    db = DeviceBatch(n, seed=11, ldda_mode=ldda_mode).fill(poison=True)
    db.dpotrf()
    info = _check_batch(db)
    assert np.all(info == 0)
    _check_sentinels(db)


def test_large_sizes():
    n = np.array([640, 767, 1000, 1023, 1024, 1025], dtype=np.int32)
    db = DeviceBatch(n, seed=12).fill(poison=True)
    db.dpotrf()
    _check_batch(db)
    _check_sentinels(db)


def test_nonspd_info_positions():
    """Non-SPD by negating a_kk at block boundaries and ends."""
    cases = []
    for n in (1, 5, 32, 33, 64, 65, 100, 200, 300):
        for k in sorted({min(n, v) for v in (1, 2, 31, 32, 33, 64, 65)} | {n}):
            cases.append((n, k))
    n_arr = np.array([c[0] for c in cases], dtype=np.int32)
    db = DeviceBatch(n_arr, seed=3)
    inputs = {}
    for i, (n, k) in enumerate(cases):
        A = vbgen.f1_matrix(3, i, n)
        A[k - 1, k - 1] = -A[k - 1, k - 1]
        inputs[i] = A
        db.set_matrix(i, A)
    db.dpotrf()
    info = _check_batch(db, exact_inputs=inputs)
    assert list(info) == [k for _, k in cases]
    _check_sentinels(db)


def test_nonspd_large_and_ring_recovery():
    """Failures inside the NB=64 blocked kernel (n > 128): failing pivots in the first and
    second 32-column halves of a 64-wide diagonal block, at panel starts and at n; the TMA ring
    must stay consistent for the matrices the same CTA factors afterwards (checked by parity of
    healthy matrices in the same batch; subprocess so that a ring hang cannot wedge the run)."""
    import subprocess
    import sys
    code = f"""
import os, sys
sys.path.insert(0, {repr(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))})
import numpy as np, torch, vbgen
from harness import DeviceBatch, compare_with_oracle
cases = [(700, 1), (700, 33), (700, 64), (700, 65), (700, 129), (700, 700), (1024, 511),
         (1024, 1024), (600, 0), (800, 0), (513, 513), (900, 0), (1000, 97), (129, 129),
         (130, 65), (200, 0), (256, 193), (255, 0), (192, 64), (160, 1)]
n_arr = np.array([c[0] for c in cases], dtype=np.int32)
db = DeviceBatch(n_arr, seed=8)
inputs = {{}}
for i, (n, k) in enumerate(cases):
    A = vbgen.f1_matrix(8, i, n)
    if k:
        A[k - 1, k - 1] = -A[k - 1, k - 1]
    inputs[i] = A
    db.set_matrix(i, A)
db.dpotrf()
torch.cuda.synchronize()
info = db.info()
assert list(info) == [k for _, k in cases], (list(info), cases)
for i in range(db.B):
    r = compare_with_oracle(inputs[i], db.block(i), info[i])
    assert r["ok"], (i, r)
print("OK")
"""
    out = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=600)
    assert out.returncode == 0 and "OK" in out.stdout, out.stdout[-2000:] + out.stderr[-3000:]


def test_small_kernel_c2_sizes_and_failures():
    """The small-matrix kernel (32 < n <= 128) on C2 sizes plus failing pivots in every 8-column
    sub-block (subprocess, so that a hang in the look-ahead barriers cannot wedge the run)."""
    import subprocess
    import sys
    code = f"""
import os, sys
sys.path.insert(0, {repr(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))})
import numpy as np, torch, vbgen
from harness import DeviceBatch, compare_with_oracle
n = np.concatenate([vbgen.sizes("C2")[:400], np.array([33, 40, 64, 65, 97, 128, 128, 100], np.int32)])
fail = {{400: 1, 401: 9, 402: 17, 403: 40, 404: 70, 405: 128, 406: 100, 407: 33}}
db = DeviceBatch(n, seed=12)
inputs = {{}}
for i in range(len(n)):
    A = vbgen.f1_matrix(12, i, int(n[i]))
    if i in fail:
        k = fail[i]; A[k - 1, k - 1] = -A[k - 1, k - 1]
    inputs[i] = A
    db.set_matrix(i, A)
db.dpotrf()
torch.cuda.synchronize()
info = db.info()
for i in range(len(n)):
    assert info[i] == fail.get(i, 0), (i, info[i])
    r = compare_with_oracle(inputs[i], db.block(i), info[i])
    assert r["ok"], (i, r)
print("OK")
"""
    out = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=600)
    assert out.returncode == 0 and "OK" in out.stdout, out.stdout[-2000:] + out.stderr[-3000:]


def test_nan_info():
    cases = [(8, (2, 2)), (8, (5, 1)), (40, (33, 33)), (40, (39, 10)), (100, (70, 64)),
             (100, (0, 0)), (100, (99, 99)), (700, (40, 40)), (700, (300, 200)),
             (1024, (1000, 999)), (600, (64, 3))]
    n_arr = np.array([c[0] for c in cases], dtype=np.int32)
    db = DeviceBatch(n_arr, seed=4)
    for i, (n, (r, c)) in enumerate(cases):
        A = vbgen.f1_matrix(4, i, n)
        A[r, c] = np.nan
        A[c, r] = np.nan
        db.set_matrix(i, A)
    db.dpotrf()
    torch.cuda.synchronize()
    assert list(db.info()) == [r + 1 for _, (r, c) in cases]  # MKL/LAPACK DISNAN convention


def test_exact_families_bit_exact():
    """min(i,j) -> tril(ones); integer unit-lower L -> L; power-of-two diagonals."""
    rng = np.random.default_rng(0)
    mats, Ls = [], []
    for n in (5, 32, 33, 100, 200, 300):
        i = np.arange(1, n + 1)
        mats.append(np.minimum.outer(i, i).astype(np.float64))
        Ls.append(np.tril(np.ones((n, n))))
    for n in (33, 128, 257, 400):
        L = np.tril(rng.integers(-1, 2, (n, n)), -1).astype(np.int64)
        L[np.arange(n), np.arange(n)] = rng.choice([1, 2, 4], size=n)
        mats.append((L @ L.T).astype(np.float64))
        Ls.append(L.astype(np.float64))
    n_arr = np.array([m.shape[0] for m in mats], dtype=np.int32)
    db = DeviceBatch(n_arr)
    for i, A in enumerate(mats):
        db.set_matrix(i, A)
    db.dpotrf()
    torch.cuda.synchronize()
    assert np.all(db.info() == 0)
    for i, L in enumerate(Ls):
        n = L.shape[0]
        got = np.tril(db.block(i)[:n])
        assert np.array_equal(got, L), f"case {i} n={n}: max diff {np.max(np.abs(got - L))}"
    _check_sentinels(db)


@pytest.mark.parametrize("cfg", ["C2", "C3", "C4"])
def test_config_full_parity(cfg):
    c = vbgen.CONFIGS[cfg]
    n = vbgen.sizes(c)
    db = DeviceBatch(n, seed=c.seed, nonspd_mod=c.nonspd_mod).fill(poison=(cfg == "C2"))
    db.dpotrf(max_n=c.nmax)
    info = _check_batch(db)
    if c.nonspd_mod:
        for i in range(db.B):
            expect = vbgen.nonspd_k(c.seed, i, int(n[i])) if vbgen.is_nonspd(c, i) else 0
            assert info[i] == expect
    else:
        assert np.all(info == 0)
    if cfg == "C2":
        _check_sentinels(db)


def test_c5_full_size_sampled():
    """C5 at BASELINE size (40000 x U{1..1024}, 112 GB) in the bench launch configuration;
    every info must be 0; a deterministic sample is compared with the oracle element by
    element, and EVERY matrix's backward error is checked (<= 10, north_star) by the
    independent torch FP64 checker (harness.gpu_backward_errors)."""
    free, _ = torch.cuda.mem_get_info()
    c = vbgen.CONFIGS["C5"]
    n = vbgen.sizes(c)
    need = vbgen.arena_layout(n, vbgen.ldda_for(n))[1] * 8
    if need > free * 0.9:
        pytest.skip("not enough device memory for full C5")
    db = DeviceBatch(n, seed=c.seed).fill()
    db.dpotrf(max_n=c.nmax)
    torch.cuda.synchronize()
    assert np.all(db.info() == 0)
    order = np.argsort(-n, kind="stable")
    sample = list(order[:4]) + list(range(0, db.B, 4001)) + list(order[-3:])
    _check_batch(db, idxs=sample)
    from harness import gpu_backward_errors
    be = gpu_backward_errors(db)
    assert np.all(np.isfinite(be)), int(np.sum(~np.isfinite(be)))
    print(f"C5 all-matrix backward error: max {be.max():.3f}, mean {be.mean():.4f}, "
          f"p99 {np.percentile(be, 99):.3f} over {db.B} matrices")
    assert be.max() <= 10.0, (int(np.argmax(be)), float(be.max()))
    del db
    torch.cuda.empty_cache()


def test_nomax_equals_max():
    n = vbgen.sizes("C2")[:500]
    a = DeviceBatch(n, seed=2).fill(poison=True)
    b = DeviceBatch(n, seed=2).fill(poison=True)
    a.dpotrf(max_n=128)
    from paper_conf_ipps_abdelfattahhtd16_b200 import vbatched_dpotrf_nomax
    vbatched_dpotrf_nomax("L", b.d_n, b.d_ptrs, b.d_ldda, b.d_info, b.B)
    torch.cuda.synchronize()
    ha, hb = a.arena.cpu().numpy(), b.arena.cpu().numpy()
    for i in range(a.B):  # bitwise over each matrix's block (the alignment gaps are never written)
        sl = slice(int(a.off[i]), int(a.off[i]) + int(a.ldda[i]) * int(n[i]))
        assert np.array_equal(ha[sl].view(np.uint64), hb[sl].view(np.uint64)), i
    assert np.array_equal(a.info(), b.info())


def test_invalid_matrices_untouched():
    """n<0 -> -2, ldda<max(1,n) -> -4, n>max_n -> -7; those matrices are not touched."""
    n = np.array([10, 40, 50, 3, 0, 70], dtype=np.int32)
    ld = np.array([32, 64, 64, 32, 1, 96], dtype=np.int32)
    db = DeviceBatch(n, ldda=ld, seed=5).fill(poison=True)
    before = db.host_arena().copy()
    bad_n = db.d_n.clone()
    bad_n[3] = -1
    bad_ld = db.d_ldda.clone()
    bad_ld[1] = 39
    from paper_conf_ipps_abdelfattahhtd16_b200 import vbatched_dpotrf
    vbatched_dpotrf("L", bad_n, db.d_ptrs, bad_ld, db.d_info, db.B, 60)
    torch.cuda.synchronize()
    info = db.info()
    assert list(info) == [0, -4, 0, -2, 0, -7]
    after = db.host_arena()
    for i in (1, 3, 5):
        s = slice(db.off[i], db.off[i] + int(ld[i]) * max(int(n[i]), 0))
        assert np.array_equal(before[s].view(np.uint64), after[s].view(np.uint64))
    _check_batch(db, idxs=[0, 2])


def test_direct_warp_path_validation():
    """max_n <= 32 takes the scan-free direct warp kernel: it must validate like the scan
    (-2 / -4 / -7, matrices untouched) and factor the rest."""
    n = np.array([10, 30, 25, 3, 0, 31, 32], dtype=np.int32)
    ld = np.array([32, 32, 32, 32, 1, 32, 32], dtype=np.int32)
    db = DeviceBatch(n, ldda=ld, seed=6).fill(poison=True)
    before = db.host_arena().copy()
    bad_n = db.d_n.clone()
    bad_n[3] = -1
    bad_ld = db.d_ldda.clone()
    bad_ld[1] = 29
    from paper_conf_ipps_abdelfattahhtd16_b200 import vbatched_dpotrf
    vbatched_dpotrf("L", bad_n, db.d_ptrs, bad_ld, db.d_info, db.B, 30)
    torch.cuda.synchronize()
    assert list(db.info()) == [0, -4, 0, -2, 0, -7, -7]
    after = db.host_arena()
    for i in (1, 3, 5, 6):
        sl = slice(db.off[i], db.off[i] + int(ld[i]) * max(int(n[i]), 0))
        assert np.array_equal(before[sl].view(np.uint64), after[sl].view(np.uint64))
    _check_batch(db, idxs=[0, 2])
    _check_sentinels(db, idxs=[0, 2])


def test_argument_errors_and_empty():
    from paper_conf_ipps_abdelfattahhtd16_b200 import vbatched_dpotrf
    db = DeviceBatch(np.array([4], dtype=np.int32)).fill()
    assert vbatched_dpotrf("X", db.d_n, db.d_ptrs, db.d_ldda, db.d_info, 1, 4, check=False) == -1
    assert vbatched_dpotrf("X", db.d_n, db.d_ptrs, db.d_ldda, db.d_info, 1, 4, check=False) == -1
    assert vbatched_dpotrf("L", db.d_n, db.d_ptrs, db.d_ldda, db.d_info, -1, 4, check=False) == -6
    assert vbatched_dpotrf("L", db.d_n, db.d_ptrs, db.d_ldda, db.d_info, 1, -1, check=False) == -7
    assert vbatched_dpotrf("L", 0, 0, 0, 0, 0, 0, check=False) == 0


def test_stream_semantics():
    """Work is enqueued on the given stream; nothing happens on another stream's timeline."""
    n = vbgen.sizes("C3")[:300]
    db = DeviceBatch(n, seed=3).fill(poison=True)
    ref = DeviceBatch(n, seed=3).fill(poison=True)
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        db.dpotrf(stream=s)
    s.synchronize()
    ref.dpotrf()
    torch.cuda.synchronize()
    ha, hb = db.arena.cpu().numpy(), ref.arena.cpu().numpy()  # deterministic across streams / runs
    for i in range(db.B):  # bitwise per matrix block (alignment gaps are never written)
        sl = slice(int(db.off[i]), int(db.off[i]) + int(db.ldda[i]) * int(n[i]))
        assert np.array_equal(ha[sl].view(np.uint64), hb[sl].view(np.uint64)), i


@pytest.mark.parametrize("uplo", ["L", "U"])
def test_host_api_chunked(uplo):
    """vbatched_dpotrf_host: host buffers, small workspace -> many chunks; bit-identical to the
    device API on the same inputs (both storage triangles)."""
    from paper_conf_ipps_abdelfattahhtd16_b200 import vbatched_dpotrf_host
    n = vbgen.sizes("C3")[:400]
    dev = DeviceBatch(n, seed=3, nonspd_mod=20).fill(poison=True, uplo=uplo)
    torch.cuda.synchronize()
    host = dev.arena.cpu().numpy().copy()
    dev.dpotrf(uplo=uplo)
    torch.cuda.synchronize()
    ptrs = (host.ctypes.data + 8 * dev.off).astype(np.int64)
    info = np.full(dev.B, -99, dtype=np.int32)
    vbatched_dpotrf_host(uplo, dev.n, ptrs, dev.ldda, info, dev.B, int(n.max()),
                         workspace_bytes=3 * 48 << 20)
    assert np.array_equal(info, dev.info()) and (info > 0).sum() == 20
    assert np.array_equal(host.view(np.uint64), dev.arena.cpu().numpy().view(np.uint64))


@pytest.mark.parametrize("cfg", ["C3", "C4"])
def test_repeat_bit_identical(cfg):
    """Every matrix is factored by one CTA in a fixed order, so repeated calls on the same input
    must give bit-identical factors: any difference is a race (this caught a TMA-refill /
    in-flight-LDS race in the ring that changed ~1 C3 run in 10)."""
    c = vbgen.CONFIGS[cfg]
    n = vbgen.sizes(c)
    db = DeviceBatch(n, seed=c.seed, nonspd_mod=c.nonspd_mod)
    ref = ref_info = None
    scramble = torch.empty(1 << 27, dtype=torch.uint8, device="cuda")
    for _ in range(15):
        db.fill()
        scramble.random_(0, 256)
        db.dpotrf(max_n=c.nmax)
        torch.cuda.synchronize()
        out = db.arena.clone().view(torch.int64)
        info = db.info()
        if ref is None:
            ref, ref_info = out, info
            continue
        assert torch.equal(out, ref) and np.array_equal(info, ref_info)


@pytest.mark.parametrize("ldda_mode", ["pad32", "tight"])
def test_uplo_upper_matches_lower_bitwise(ldda_mode):
    """uplo='U' (LAPACK DPOTRF): A = U^T U with only the upper triangle
    referenced. The kernels run the same arithmetic on the transposed view, so U^T must equal
    the 'L' run's factor bit for bit (info too); the strict lower triangle and the padding rows
    stay untouched (NaN poison), and the factor passes the oracle gates."""
    sizes = [1, 2, 7, 16, 31, 32, 33, 40, 64, 65, 96, 127, 128, 129, 160, 192, 255, 256, 257,
             300, 384, 511, 513, 640, 700, 1024]
    fail = {3: 5, 10: 60, 17: 200, 21: 129, 24: 650}  # slot -> failing pivot (1-based)
    n = np.array(sizes, dtype=np.int32)
    dl = DeviceBatch(n, seed=21, ldda_mode=ldda_mode)
    du = DeviceBatch(n, seed=21, ldda_mode=ldda_mode)
    inputs = {}
    for i, ni in enumerate(sizes):
        A = vbgen.f1_matrix(21, i, ni)
        if i in fail:
            k = fail[i]
            A[k - 1, k - 1] = -A[k - 1, k - 1]
        inputs[i] = A
        dl.set_matrix(i, A, uplo="L")
        du.set_matrix(i, A, uplo="U")
    dl.dpotrf(uplo="L")
    du.dpotrf(uplo="U")
    torch.cuda.synchronize()
    il, iu = dl.info(), du.info()
    assert list(il) == list(iu) == [fail.get(i, 0) for i in range(len(sizes))]
    for i, ni in enumerate(sizes):
        bl, bu = dl.block(i), du.block(i)
        k = ni if il[i] == 0 else il[i] - 1  # defined leading block
        low = np.tril(np.ones((k, k), bool))
        Lb = bl[:k, :k].view(np.uint64)
        Ub = bu[:k, :k].T.view(np.uint64)
        assert np.array_equal(Lb[low], Ub[low]), i
        # strict lower triangle and padding rows of the 'U' storage: never touched
        strict_low = np.tril(np.ones((ni, ni), bool), -1)
        assert np.all(bu[:ni, :ni].view(np.uint64)[strict_low] == POISON), i
        if bu.shape[0] > ni:
            assert np.all(bu[ni:, :].view(np.uint64) == POISON), i
        r = compare_with_oracle(inputs[i], bu[:ni, :ni].T.copy(), iu[i])
        assert r["ok"], (i, r)


def test_uplo_upper_device_generated_c3_sample():
    """uplo='U' on device-generated upper storage (vbgen poison bit 1): the first 600 matrices of
    C3 with 5 % non-SPD; info and U^T bitwise equal to the 'L' run, lower triangle untouched."""
    n = vbgen.sizes("C3")[:600]
    dl = DeviceBatch(n, seed=3, nonspd_mod=20).fill(poison=True)
    du = DeviceBatch(n, seed=3, nonspd_mod=20).fill(poison=True, uplo="U")
    dl.dpotrf(uplo="L")
    du.dpotrf(uplo="U")
    torch.cuda.synchronize()
    il, iu = dl.info(), du.info()
    assert np.array_equal(il, iu) and (il > 0).sum() == 30
    for i in range(0, 600, 7):
        ni = int(n[i])
        k = ni if il[i] == 0 else il[i] - 1
        low = np.tril(np.ones((k, k), bool))
        bl, bu = dl.block(i), du.block(i)
        assert np.array_equal(bl[:k, :k].view(np.uint64)[low], bu[:k, :k].T.view(np.uint64)[low]), i
        strict_low = np.tril(np.ones((ni, ni), bool), -1)
        assert np.all(bu[:ni, :ni].view(np.uint64)[strict_low] == POISON), i


@pytest.mark.parametrize("uplo", ["L", "U"])
def test_two_phase_api_equals_single_call(uplo):
    """vbatched_dpotrf_scan + vbatched_dpotrf_factor on caller workspace (the split bench.py's
    roofline pass times) give exactly the single call's result, both storage triangles."""
    import paper_conf_ipps_abdelfattahhtd16_b200 as vb
    n = vbgen.sizes("C4")[:500]
    a = DeviceBatch(n, seed=4, nonspd_mod=20).fill(poison=True, uplo=uplo)
    b = DeviceBatch(n, seed=4, nonspd_mod=20).fill(poison=True, uplo=uplo)
    mx = int(n.max())
    a.dpotrf(uplo=uplo)
    ws = torch.empty(vb.vbatched_dpotrf_workspace_size(b.B), dtype=torch.uint8, device="cuda")
    vb.vbatched_dpotrf_scan(uplo, b.d_n, b.d_ldda, b.d_info, b.B, mx, ws)
    vb.vbatched_dpotrf_factor(uplo, b.d_n, b.d_ptrs, b.d_ldda, b.d_info, b.B, mx, ws)
    torch.cuda.synchronize()
    assert np.array_equal(a.info(), b.info()) and (a.info() > 0).sum() == 25
    ha, hb = a.arena.cpu().numpy(), b.arena.cpu().numpy()
    for i in range(a.B):
        sl = slice(int(a.off[i]), int(a.off[i]) + int(a.ldda[i]) * int(n[i]))
        assert np.array_equal(ha[sl].view(np.uint64), hb[sl].view(np.uint64)), i


def test_max_n_too_small_f32_and_upper():
    """n > max_n -> info -7 and the matrix untouched, for SPOTRF and for uplo 'U' too."""
    n = np.array([40, 300, 100, 700], dtype=np.int32)
    for dtype, uplo in (("f32", "L"), ("f64", "U")):
        db = DeviceBatch(n, seed=6, dtype=dtype).fill(poison=True, uplo=uplo)
        before = db.arena.cpu().numpy().copy()
        db.dpotrf(max_n=200, uplo=uplo)
        torch.cuda.synchronize()
        info = db.info()
        assert list(info[[1, 3]]) == [-7, -7] and list(info[[0, 2]]) == [0, 0], (dtype, uplo, info)
        after = db.arena.cpu().numpy()
        for i in (1, 3):
            sl = slice(int(db.off[i]), int(db.off[i]) + int(db.ldda[i]) * int(n[i]))
            assert np.array_equal(before[sl], after[sl], equal_nan=True), (dtype, uplo, i)
