"""Test/bench harness: builds vbatched device batches from vbgen recipes and compares
results with the oracle. Infrastructure only (imports oracle lazily for the comparison
helpers; the product package never imports this module)."""
from __future__ import annotations

import numpy as np
import torch

import vbgen
from vbgen import device as vbdev


class DeviceBatch:
    """A vbatched problem resident in HBM: one arena (each matrix 256 B aligned), device
    pointer array, n[], ldda[], info[] (int32), gidx[] (global matrix index for the hash)."""

    def __init__(self, n, ldda=None, seed=1, gidx=None, nonspd_mod=0, device="cuda",
                 ldda_mode="pad32", dtype="f64"):
        self.n = np.ascontiguousarray(n, dtype=np.int32)
        self.B = len(self.n)
        self.ldda = np.ascontiguousarray(vbgen.ldda_for(self.n, ldda_mode) if ldda is None else ldda,
                                         dtype=np.int32)
        self.gidx = np.arange(self.B, dtype=np.int32) if gidx is None else np.ascontiguousarray(gidx, np.int32)
        self.seed = seed
        self.nonspd_mod = nonspd_mod
        self.device = torch.device(device)
        self.f32 = dtype == "f32"
        es = 4 if self.f32 else 8
        self.off, total = vbgen.arena_layout(np.maximum(self.n, 0), self.ldda, elem_bytes=es)
        self.arena = torch.empty(total, dtype=torch.float32 if self.f32 else torch.float64,
                                 device=self.device)
        base = self.arena.data_ptr()
        self.ptrs_h = (base + es * self.off).astype(np.int64)
        self.d_ptrs = torch.from_numpy(self.ptrs_h).to(self.device)
        self.d_n = torch.from_numpy(self.n).to(self.device)
        self.d_ldda = torch.from_numpy(self.ldda).to(self.device)
        self.d_gidx = torch.from_numpy(self.gidx).to(self.device)
        self.d_info = torch.full((max(self.B, 1),), -12345, dtype=torch.int32, device=self.device)

    def fill(self, poison=False, stream=None, uplo="L"):
        s = torch.cuda.current_stream().cuda_stream if stream is None else stream
        flags = (1 if poison else 0) | (2 if uplo == "U" else 0) | (4 if self.f32 else 0)
        vbdev.fill_f1(self.seed, self.B, self.d_n.data_ptr(), self.d_ldda.data_ptr(),
                      self.d_ptrs.data_ptr(), self.d_gidx.data_ptr(), self.nonspd_mod, flags, s)
        return self

    def set_matrix(self, i, A: np.ndarray, poison=True, uplo="L"):
        """Write a host matrix into slot i: its lower ('L') or upper ('U') triangle; the other
        strict triangle and the padding rows get the NaN poison."""
        n, ld = int(self.n[i]), int(self.ldda[i])
        if self.f32:
            blk = np.full((ld, n), np.nan, dtype=np.float32)
            if poison:
                blk.view(np.uint32)[:] = np.uint32(0x7FC0BEEF)
            A = np.asarray(A, dtype=np.float32)
        else:
            blk = np.full((ld, n), np.nan)
            if poison:
                blk.view(np.uint64)[:] = np.uint64(vbgen.NAN_POISON_BITS)
        tri = np.tril(np.ones((n, n), bool)) if uplo == "L" else np.triu(np.ones((n, n), bool))
        blk[:n, :n] = np.where(tri, A, blk[:n, :n])
        t = torch.from_numpy(blk.ravel(order="F").copy())
        self.arena[self.off[i]: self.off[i] + ld * n].copy_(t)

    def block(self, i) -> np.ndarray:
        """Host copy of the full ldda x n column block of matrix i."""
        n, ld = int(self.n[i]), int(self.ldda[i])
        if n <= 0:
            return np.zeros((ld, 0))
        return self.arena[self.off[i]: self.off[i] + ld * n].cpu().numpy().reshape((ld, n), order="F")

    def host_arena(self) -> np.ndarray:
        return self.arena.cpu().numpy()

    def info(self) -> np.ndarray:
        return self.d_info[: self.B].cpu().numpy()

    def dpotrf(self, max_n=None, stream=None, uplo="L", check=True):
        """vbatched_dpotrf (or vbatched_spotrf for an FP32 batch) on the whole batch."""
        from paper_conf_ipps_abdelfattahhtd16_b200 import vbatched_dpotrf, vbatched_spotrf
        mx = int(self.n.max()) if (max_n is None and self.B) else (max_n or 0)
        fn = vbatched_spotrf if self.f32 else vbatched_dpotrf
        return fn(uplo, self.d_n, self.d_ptrs, self.d_ldda, self.d_info, self.B, mx,
                  stream=stream, check=check)

    def host_matrix_input(self, i) -> np.ndarray:
        """The matrix the generator writes for slot i (numpy twin)."""
        return vbgen.f1_matrix(self.seed, int(self.gidx[i]), int(self.n[i]),
                               self.nonspd_mod > 0 and int(self.gidx[i]) % self.nonspd_mod == self.nonspd_mod - 1)


def compare_with_oracle(A_in: np.ndarray, L_gpu: np.ndarray, info_gpu: int, kappa_ok=True):
    """Parity gates (BASELINE.json north_star):
    info bit-exact; backward error <= 10 (eps = 2^-53) on the defined leading block;
    row-scaled difference to the oracle's L <= 1e-10. Returns dict of measurements."""
    import oracle
    n = A_in.shape[0]
    Lo, info_o = oracle.dpotrf(np.asfortranarray(A_in))
    res = {"n": n, "info_oracle": info_o, "info_gpu": int(info_gpu)}
    nb = n if info_o == 0 else info_o - 1
    Lg = np.asfortranarray(L_gpu[:n, :n])
    res["bwd"] = oracle.backward_error(np.asfortranarray(A_in), Lg, info_o) if nb > 0 else 0.0
    res["rowscaled"] = oracle.rowscaled_diff(Lg, Lo, nb)
    res["ok"] = (res["info_oracle"] == res["info_gpu"] and res["bwd"] <= 10.0 and
                 (res["rowscaled"] <= 1e-10 or not kappa_ok))
    return res


def gpu_backward_errors(db: DeviceBatch, chunk_elems: int = 1 << 26) -> np.ndarray:
    """Per-matrix backward error ||A - L L^T||_F / (n ||A||_F 2^-53) of every info == 0 matrix
    of a device batch, computed on the GPU with plain torch FP64 (cuBLAS batched matmul,
    grouped by (n, ldda)) — independent of libvbatched (the all-matrix check
    of C5). A is regenerated by vbgen's device generator (F1, db's seed / gidx / non-SPD rule)
    into scratch; L is the lower triangle of db's arena. Entries for info != 0 or n == 0 are NaN.
    The FP64 rounding of L L^T adds O(1/sqrt(n)) to the ratio (validated against the
    long-double oracle on a sample by the tests)."""
    info = db.info()
    out = np.full(db.B, np.nan)
    keys = {}
    for i in np.nonzero((info == 0) & (db.n > 0))[0]:
        keys.setdefault((int(db.n[i]), int(db.ldda[i])), []).append(int(i))
    eps = 2.0 ** -53
    for (n, ld), idx in keys.items():
        per = max(1, chunk_elems // (n * n))
        for c0 in range(0, len(idx), per):
            ii = idx[c0: c0 + per]
            c = len(ii)
            # L: the stored lower triangle of each matrix ([col][row] views of the arena)
            M = torch.stack([db.arena.narrow(0, int(db.off[i]), ld * n).view(n, ld)[:, :n]
                             for i in ii]).to(torch.float64)
            L = torch.tril(M.transpose(1, 2))
            # A: regenerated (lower triangle written, column-major, ld = n) into scratch
            scratch = torch.zeros(c * n * n, dtype=torch.float64, device=db.device)
            ptrs = torch.tensor([scratch.data_ptr() + 8 * n * n * k for k in range(c)],
                                dtype=torch.int64, device=db.device)
            dn = torch.full((c,), n, dtype=torch.int32, device=db.device)
            dg = torch.tensor([int(db.gidx[i]) for i in ii], dtype=torch.int32, device=db.device)
            vbdev.fill_f1(db.seed, c, dn.data_ptr(), dn.data_ptr(), ptrs.data_ptr(), dg.data_ptr(),
                          db.nonspd_mod, 0, torch.cuda.current_stream().cuda_stream)
            Alow = torch.tril(scratch.view(c, n, n).transpose(1, 2))
            A = Alow + torch.tril(Alow, -1).transpose(1, 2)
            R = A - torch.bmm(L, L.transpose(1, 2))
            num = torch.linalg.matrix_norm(R)
            den = torch.linalg.matrix_norm(A)
            out[ii] = (num / (n * den * eps)).cpu().numpy()
    return out


class LUBatch:
    """A vbatched general-matrix problem for vbatched_dgetrf: arena of m_i x n_i column-major
    matrices (leading dims ldda_i, 256 B aligned), ipiv arena (min(m,n) int32 per matrix) and
    the device pointer arrays. Values: vbgen.g1_matrix(seed, gidx, m, n) unless set."""

    def __init__(self, m, n, seed=1, ldda=None, device="cuda"):
        self.m = np.ascontiguousarray(m, dtype=np.int32)
        self.n = np.ascontiguousarray(n, dtype=np.int32)
        self.B = len(self.m)
        self.seed = seed
        self.ldda = np.ascontiguousarray(np.maximum(1, self.m) if ldda is None else ldda, dtype=np.int32)
        self.off, total = vbgen.arena_layout(np.maximum(self.n, 0), self.ldda)
        self.arena = torch.full((total,), float("nan"), dtype=torch.float64, device=device)
        k = np.maximum(0, np.minimum(self.m, self.n)).astype(np.int64)
        self.ioff = np.concatenate([[0], np.cumsum((k + 63) // 64 * 64)[:-1]]).astype(np.int64)
        self.ipiv = torch.full((int(self.ioff[-1] + max(64, k[-1] + 64)),), -7, dtype=torch.int32,
                               device=device)
        self.d_ptrs = torch.from_numpy((self.arena.data_ptr() + 8 * self.off).astype(np.int64)).to(device)
        self.d_ipiv = torch.from_numpy((self.ipiv.data_ptr() + 4 * self.ioff).astype(np.int64)).to(device)
        self.d_m = torch.from_numpy(self.m).to(device)
        self.d_n = torch.from_numpy(self.n).to(device)
        self.d_ldda = torch.from_numpy(self.ldda).to(device)
        self.d_info = torch.full((max(self.B, 1),), -12345, dtype=torch.int32, device=device)
        self.inputs = {}

    def set_matrix(self, i, A):
        m, n, ld = int(self.m[i]), int(self.n[i]), int(self.ldda[i])
        blk = np.full((ld, n), np.nan)
        blk.view(np.uint64)[:] = np.uint64(vbgen.NAN_POISON_BITS)
        blk[:m, :] = A
        self.inputs[i] = np.asfortranarray(A)
        self.arena[self.off[i]: self.off[i] + ld * n].copy_(torch.from_numpy(blk.ravel(order="F").copy()))

    def fill(self):
        for i in range(self.B):
            if self.m[i] > 0 and self.n[i] > 0:
                self.set_matrix(i, vbgen.g1_matrix(self.seed, i, int(self.m[i]), int(self.n[i])))
        return self

    def getrf(self, max_m=None, max_n=None, stream=None, check=True):
        from paper_conf_ipps_abdelfattahhtd16_b200 import vbatched_dgetrf
        mm = int(self.m.max()) if max_m is None else max_m
        mn = int(self.n.max()) if max_n is None else max_n
        return vbatched_dgetrf(self.d_m, self.d_n, self.d_ptrs, self.d_ldda, self.d_ipiv, self.d_info,
                               self.B, mm, mn, stream=stream, check=check)

    def block(self, i):
        m, n, ld = int(self.m[i]), int(self.n[i]), int(self.ldda[i])
        return self.arena[self.off[i]: self.off[i] + ld * n].cpu().numpy().reshape((ld, n), order="F")

    def ipiv_of(self, i):
        k = max(0, min(int(self.m[i]), int(self.n[i])))
        return self.ipiv[int(self.ioff[i]): int(self.ioff[i]) + k].cpu().numpy()

    def info(self):
        return self.d_info[: self.B].cpu().numpy()


def compare_lu_with_oracle(A_in, F_gpu, ipiv_gpu, info_gpu):
    """LU parity gates (DESIGN.md readings): info and ipiv bit-exact;
    backward error ||P A - L U||_F / (max(m,n) ||A||_F eps) <= 10; every entry of the factored
    matrix within 1e-10 of the oracle's, scaled by the norm of the oracle's row."""
    import oracle
    m, n = A_in.shape
    Fo, ipo, info_o = oracle.dgetrf(A_in)
    Fg = np.asfortranarray(F_gpu[:m, :n])
    res = {"m": m, "n": n, "info_oracle": info_o, "info_gpu": int(info_gpu),
           "ipiv_equal": bool(np.array_equal(np.asarray(ipiv_gpu), ipo))}
    res["bwd"] = oracle.getrf_backward_error(A_in, Fg, np.asarray(ipiv_gpu, np.int32)) if m and n else 0.0
    rn = np.sqrt(np.sum(Fo * Fo, axis=1))
    rn[rn == 0] = 1.0
    res["rowscaled"] = float(np.max(np.abs(Fg - Fo) / rn[:, None])) if m and n else 0.0
    res["ok"] = (res["info_oracle"] == res["info_gpu"] and res["ipiv_equal"] and res["bwd"] <= 10.0
                 and res["rowscaled"] <= 1e-10)
    return res


class ZBatch:
    """A vbatched complex Hermitian problem for vbatched_zpotrf (complex128) / vbatched_cpotrf
    (complex64): arena of interleaved complex matrices (leading dims ldda, 256 B aligned), the
    referenced triangle from vbgen.f1c_matrix (or set_matrix), NaN-payload poison elsewhere."""

    def __init__(self, n, seed=1, single=False, ldda=None, nonspd_mod=0, device="cuda"):
        self.n = np.ascontiguousarray(n, dtype=np.int32)
        self.B = len(self.n)
        self.seed, self.single, self.nonspd_mod = seed, single, nonspd_mod
        self.dt = torch.complex64 if single else torch.complex128
        self.np_dt = np.complex64 if single else np.complex128
        es = 8 if single else 16
        self.ldda = np.ascontiguousarray(np.maximum(1, self.n) if ldda is None else ldda, dtype=np.int32)
        self.off, total = vbgen.arena_layout(np.maximum(self.n, 0), self.ldda, elem_bytes=es)
        self.arena = torch.zeros(total, dtype=self.dt, device=device)
        self.d_ptrs = torch.from_numpy((self.arena.data_ptr() + es * self.off).astype(np.int64)).to(device)
        self.d_n = torch.from_numpy(self.n).to(device)
        self.d_ldda = torch.from_numpy(self.ldda).to(device)
        self.d_info = torch.full((max(self.B, 1),), -12345, dtype=torch.int32, device=device)
        self.inputs = {}

    def set_matrix(self, i, A, uplo="L"):
        n, ld = int(self.n[i]), int(self.ldda[i])
        blk = np.full((ld, n), complex(np.nan, np.nan), dtype=self.np_dt)
        tri = np.tril(np.ones((n, n), bool)) if uplo == "L" else np.triu(np.ones((n, n), bool))
        blk[:n, :n] = np.where(tri, np.asarray(A, dtype=self.np_dt), blk[:n, :n])
        self.inputs[i] = np.asfortranarray(np.asarray(A, dtype=self.np_dt))
        self.arena[self.off[i]: self.off[i] + ld * n].copy_(torch.from_numpy(blk.ravel(order="F").copy()))

    def fill(self, uplo="L"):
        for i in range(self.B):
            if self.n[i] > 0:
                ns = self.nonspd_mod > 0 and i % self.nonspd_mod == self.nonspd_mod - 1
                self.set_matrix(i, vbgen.f1c_matrix(self.seed, i, int(self.n[i]), ns), uplo)
        return self

    def potrf(self, uplo="L", max_n=None, stream=None, check=True):
        import paper_conf_ipps_abdelfattahhtd16_b200 as vb
        fn = vb.vbatched_cpotrf if self.single else vb.vbatched_zpotrf
        mx = int(self.n.max()) if max_n is None else max_n
        return fn(uplo, self.d_n, self.d_ptrs, self.d_ldda, self.d_info, self.B, mx, stream=stream,
                  check=check)

    def block(self, i):
        n, ld = int(self.n[i]), int(self.ldda[i])
        return self.arena[self.off[i]: self.off[i] + ld * n].cpu().numpy().reshape((ld, n), order="F")

    def info(self):
        return self.d_info[: self.B].cpu().numpy()


def compare_zpotrf_with_oracle(A_in, L_gpu, info_gpu, single=False):
    """Complex Cholesky gates: info exact; complex backward error <= 10 (eps = 2^-53; FP32
    storage: the same ratio with eps32, i.e. x 2^-29); row-scaled difference to the oracle's L
    <= 1e-10 (Z, F1c kappa ~ 1) or 8 n eps32 (C, vs the single-precision oracle)."""
    import oracle
    n = A_in.shape[0]
    if single:
        Lo, info_o = oracle.cpotrf(A_in.astype(np.complex64))
    else:
        Lo, info_o = oracle.zpotrf(A_in)
    nb = n if info_o == 0 else info_o - 1
    Lg = np.tril(np.asarray(L_gpu[:n, :n], dtype=np.complex128))
    res = {"n": n, "info_oracle": info_o, "info_gpu": int(info_gpu)}
    bwd = oracle.zpotrf_backward_error(np.asarray(A_in, np.complex128), Lg, info_o) if nb else 0.0
    res["bwd"] = bwd * (2.0 ** -29 if single else 1.0)
    if nb:
        o = np.tril(np.asarray(Lo, np.complex128)[:nb, :nb])
        rn = np.sqrt(np.sum(np.abs(o) ** 2, axis=1))
        rn[rn == 0] = 1.0
        res["rowscaled"] = float(np.max(np.abs(Lg[:nb, :nb] - o) / rn[:, None]))
    else:
        res["rowscaled"] = 0.0
    tol = 8 * max(nb, 1) * 2.0 ** -24 if single else 1e-10
    res["ok"] = res["info_oracle"] == res["info_gpu"] and res["bwd"] <= 10.0 and res["rowscaled"] <= tol
    return res


class QRBatch(LUBatch):
    """A vbatched general-matrix problem for vbatched_dgeqrf: LUBatch's arena plus a tau arena
    (min(m, n) doubles per matrix) and its device pointer array."""

    def __init__(self, m, n, seed=1, ldda=None, device="cuda"):
        super().__init__(m, n, seed=seed, ldda=ldda, device=device)
        k = np.maximum(0, np.minimum(self.m, self.n)).astype(np.int64)
        self.toff = np.concatenate([[0], np.cumsum((k + 31) // 32 * 32)[:-1]]).astype(np.int64)
        self.tau = torch.full((int(self.toff[-1] + max(32, k[-1] + 32)),), float("nan"),
                              dtype=torch.float64, device=device)
        self.d_tau = torch.from_numpy((self.tau.data_ptr() + 8 * self.toff).astype(np.int64)).to(device)

    def geqrf(self, max_m=None, max_n=None, stream=None, check=True):
        from paper_conf_ipps_abdelfattahhtd16_b200 import vbatched_dgeqrf
        mm = int(self.m.max()) if max_m is None else max_m
        mn = int(self.n.max()) if max_n is None else max_n
        return vbatched_dgeqrf(self.d_m, self.d_n, self.d_ptrs, self.d_ldda, self.d_tau, self.d_info,
                               self.B, mm, mn, stream=stream, check=check)

    def tau_of(self, i):
        k = max(0, min(int(self.m[i]), int(self.n[i])))
        return self.tau[int(self.toff[i]): int(self.toff[i]) + k].cpu().numpy()


def compare_qr_with_oracle(A_in, F_gpu, tau_gpu):
    """QR parity gates (DESIGN.md readings): reconstruction
    ||A - QR||_F / (max(m,n) ||A||_F eps) <= 10 and orthogonality ||Q^T Q - I||_F / (m eps) <= 10
    of the GPU's own factor (Q rebuilt from its v and tau), every entry of the compact factor
    within 1e-10 of the oracle's scaled by the oracle row norm, tau within 1e-10."""
    import oracle
    m, n = A_in.shape
    Fo, to = oracle.dgeqrf(A_in)
    Fg = np.asfortranarray(F_gpu[:m, :n])
    tg = np.asarray(tau_gpu, dtype=np.float64)
    res = {"m": m, "n": n}
    res["bwd"], res["orth"] = oracle.geqrf_errors(A_in, Fg, tg) if m and n else (0.0, 0.0)
    rn = np.sqrt(np.sum(Fo * Fo, axis=1))
    rn[rn == 0] = 1.0
    res["rowscaled"] = float(np.max(np.abs(Fg - Fo) / rn[:, None])) if m and n else 0.0
    res["tau_diff"] = float(np.max(np.abs(tg - to))) if len(to) else 0.0
    res["ok"] = (res["bwd"] <= 10 and res["orth"] <= 10 and res["rowscaled"] <= 1e-10
                 and res["tau_diff"] <= 1e-10)
    return res
