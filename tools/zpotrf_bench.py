"""vbatched_zpotrf / vbatched_cpotrf throughput: one JSON line per
workload. python tools/zpotrf_bench.py [z|c] [count] [nmax] ...  (n ~ U{1..nmax}, F1c values)
GFLOP/s counts 4 n^3/3 real flops per matrix (a complex multiply-add is 4 real ones, LAPACK's
ZPOTRF count); CUDA events around the call, inputs restored + L2 flushed before each of 10
timed reps (3 warm-up). Roofline denominator: the measured FP64 DMMA peak."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from harness import ZBatch  # noqa: E402

args = sys.argv[1:] or ["z", "3000", "512"]
peak = json.load(open(os.path.join(os.path.dirname(__file__), "..", "profiles", "peaks_fp64.json")))["fp64_tflops"]
for prec, cnt, nmax in zip(args[0::3], args[1::3], args[2::3]):
    cnt, nmax = int(cnt), int(nmax)
    n = np.random.default_rng(nmax).integers(1, nmax + 1, cnt).astype(np.int32)
    zb = ZBatch(n, seed=17, single=(prec == "c")).fill()
    pristine = zb.arena.clone()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    times = []
    for rep in range(13):
        zb.arena.copy_(pristine)
        flush.fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        zb.potrf()
        e1.record()
        torch.cuda.synchronize()
        if rep >= 3:
            times.append(e0.elapsed_time(e1) / 1e3)
    assert np.all(zb.info() == 0)
    t = float(np.median(times))
    fl = float(np.sum(4.0 * n.astype(np.float64) ** 3 / 3))
    print(json.dumps({"op": f"vbatched_{prec}potrf", "workload": f"{cnt} x U{{1..{nmax}}}, F1c values",
                      "value": fl / t / 1e9, "unit": "GFLOP/s (4n^3/3 real flops per matrix)",
                      "ms": t * 1e3, "best_ms": min(times) * 1e3,
                      "roofline": {"bound": "tensor", "achieved": fl / t / 1e12, "peak": peak,
                                   "frac": fl / t / 1e12 / peak, "unit": "TFLOP/s"}}), flush=True)
