"""Standalone vbatched BLAS throughput (DGEMM / DSYRK / DTRSM as
workloads of their own, against the measured FP64 DMMA peak): python tools/blas_bench.py [count]

Batches of `count` (default 4000) matrices with sizes uniform in [1, 512] (seeded), the shapes
the factorisation's updates have; flops: GEMM 2mnk, SYRK n(n+1)k, TRSM (side R) m n^2 / (side L)
n m^2. One JSON line per routine with GFLOP/s and the fraction of 37.07 TF/s."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_abdelfattahhtd16_b200 as vb  # noqa: E402

PEAK = 37.07e12
count = int(sys.argv[1]) if len(sys.argv) > 1 else 4000
rng = np.random.default_rng(77)
dev = torch.device("cuda")


def arena(shapes):
    ld = [max(1, (r + 31) // 32 * 32) for r, c in shapes]
    sz = [l * c for l, (r, c) in zip(ld, shapes)]
    off = np.concatenate([[0], np.cumsum(sz)]).astype(np.int64)
    buf = torch.rand(max(1, int(off[-1])), dtype=torch.float64, device=dev)
    ptrs = torch.from_numpy(buf.data_ptr() + 8 * off[:-1]).to(dev)
    return buf, ptrs, torch.tensor(ld, dtype=torch.int32, device=dev)


def timed(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) / 1e3)
    return best


def ints(x):
    return torch.tensor(x, dtype=torch.int32, device=dev)


m = rng.integers(1, 513, count)
n = rng.integers(1, 513, count)
k = rng.integers(1, 513, count)
out = []
# GEMM N,T (the panel-update shape): C(m x n) -= A(m x k) B(n x k)^T
A, pA, lA = arena(list(zip(m, k)))
B, pB, lB = arena(list(zip(n, k)))
C, pC, lC = arena(list(zip(m, n)))
t = timed(lambda: vb.vbatched_dgemm("N", "T", ints(m), ints(n), ints(k), -1.0, pA, lA, pB, lB, 1.0,
                                    pC, lC, count, int(m.max()), int(n.max()), int(k.max())))
fl = float(np.sum(2.0 * m * n * k))
out.append({"routine": "dgemm N,T", "gflops": fl / t / 1e9, "frac_fp64_peak": fl / t / PEAK, "ms": t * 1e3})
# SYRK L,N: C(n x n) -= A(n x k) A^T
A2, pA2, lA2 = arena(list(zip(n, k)))
C2, pC2, lC2 = arena(list(zip(n, n)))
t = timed(lambda: vb.vbatched_dsyrk("L", "N", ints(n), ints(k), -1.0, pA2, lA2, 1.0, pC2, lC2, count,
                                    int(n.max()), int(k.max())))
fl = float(np.sum(1.0 * n * (n + 1) * k))
out.append({"routine": "dsyrk L,N", "gflops": fl / t / 1e9, "frac_fp64_peak": fl / t / PEAK, "ms": t * 1e3})
# TRSM R,L,T,N (the Cholesky panel solve) and L,L,N,N: well-conditioned triangles
for side in ("R", "L"):
    na = n if side == "R" else m
    # unit-diagonal solves (diag 'U'): the timing does not depend on the values; the strictly
    # lower entries are scaled down so that the solution stays bounded
    T, pT, lT = arena(list(zip(na, na)))
    T.mul_(1.0 / 512)
    Bm, pBm, lBm = arena(list(zip(m, n)))
    fl = float(np.sum(1.0 * m * n * (n if side == "R" else m)))
    t = timed(lambda: vb.vbatched_dtrsm(side, "L", "T" if side == "R" else "N", "U", ints(m), ints(n),
                                        1.0, pT, lT, pBm, lBm, count, int(m.max()), int(n.max())))
    out.append({"routine": f"dtrsm {side},L,{'T' if side == 'R' else 'N'},U", "gflops": fl / t / 1e9,
                "frac_fp64_peak": fl / t / PEAK, "ms": t * 1e3})
for o in out:
    o["count"] = count
    o["sizes"] = "m, n, k uniform in [1, 512] (numpy default_rng(77))"
    print(json.dumps(o))
