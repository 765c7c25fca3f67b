"""vbatched_dgetrf / vbatched_dgeqrf throughput: one JSON line per
workload. python tools/getrf_bench.py [count] [nmax] ...  (square matrices, n ~ U{1..nmax});
OP=qr selects vbatched_dgeqrf (LAPACK DGEQRF flops for m = n: 4n^3/3 + n^2 + 14n/3... ~ 4n^3/3).
GFLOP/s counts the LAPACK DGETRF flops of each matrix (m n^2 - n^3/3 - n^2/2 + 5n/6 for m = n:
2n^3/3 - n^2/2 + 5n/6); timing: CUDA events around the call, inputs restored and L2 flushed
before each of 10 timed reps (3 warm-up). The roofline denominator is the measured FP64 DMMA
peak (profiles/peaks_fp64.json). The oracle (plain LU) is timed on a bounded sample."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from harness import LUBatch, QRBatch  # noqa: E402

QR = os.environ.get("OP") == "qr"


def flops(n):
    n = n.astype(np.float64)
    if QR:
        return float(np.sum(4 * n ** 3 / 3 + n ** 2 + 14 * n / 3))
    return float(np.sum(2 * n ** 3 / 3 - n ** 2 / 2 + 5 * n / 6))


args = sys.argv[1:] or ["3000", "512"]
peak = json.load(open(os.path.join(os.path.dirname(__file__), "..", "profiles", "peaks_fp64.json")))["fp64_tflops"]
for cnt, nmax in zip(args[0::2], args[1::2]):
    cnt, nmax = int(cnt), int(nmax)
    n = np.random.default_rng(nmax).integers(1, nmax + 1, cnt).astype(np.int32)
    lb = (QRBatch if QR else LUBatch)(n, n, seed=13).fill()
    pristine = lb.arena.clone()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    times = []
    for rep in range(13):
        lb.arena.copy_(pristine)
        flush.fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        lb.geqrf() if QR else lb.getrf()
        e1.record()
        torch.cuda.synchronize()
        if rep >= 3:
            times.append(e0.elapsed_time(e1) / 1e3)
    assert np.all(lb.info() == 0)
    t = float(np.median(times))
    fl = flops(n)
    import oracle
    idx = np.arange(0, cnt, max(1, cnt // 100))
    t0 = time.perf_counter()
    for i in idx:
        (oracle.dgeqrf if QR else oracle.dgetrf)(lb.inputs[int(i)])
    tc = time.perf_counter() - t0
    line = {"op": "vbatched_dgeqrf" if QR else "vbatched_dgetrf", "workload": f"{cnt} x U{{1..{nmax}}} square, g1 values",
            "value": fl / t / 1e9, "unit": "GFLOP/s", "ms": t * 1e3, "best_ms": min(times) * 1e3,
            "roofline": {"bound": "tensor", "achieved": fl / t / 1e12, "peak": peak,
                         "frac": fl / t / 1e12 / peak, "unit": "TFLOP/s"},
            "cpu_oracle": {"value": flops(n[idx]) / tc / 1e9, "unit": "GFLOP/s", "cores": 1,
                           "sample": f"every {max(1, cnt // 100)}th matrix ({len(idx)})"}}
    print(json.dumps(line), flush=True)
