"""Factorisation throughput on uniform-size batches (dev tool): python tools/uniform_bench.py n count"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from harness import DeviceBatch  # noqa: E402

for arg in sys.argv[1:]:
    n, cnt = (int(x) for x in arg.split("x"))
    db = DeviceBatch(np.full(cnt, n, dtype=np.int32), seed=3)
    ts = []
    for it in range(4):
        db.fill()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        db.dpotrf()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    ms = min(ts[1:])
    gf = cnt * n ** 3 / 3 / (ms * 1e-3) / 1e9
    gb = cnt * 8 * n * (n + 1) / (ms * 1e-3) / 1e9
    assert np.all(db.info() == 0)
    print(f"n={n:5d} x {cnt:6d}: {ms:8.3f} ms  {gf:9.1f} GFLOP/s  {gb:8.1f} GB/s(alg)")
