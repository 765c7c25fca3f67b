"""Measure the FP64 roofline denominators on the GPU box: cuBLAS DGEMM (torch.matmul float64),
host core count / memory. Tool only (not part of the library). Writes one JSON line per measurement."""
import json
import os
import time

import torch


def dgemm_peak(n=8192, reps=10):
    a = torch.randn(n, n, dtype=torch.float64, device="cuda")
    b = torch.randn(n, n, dtype=torch.float64, device="cuda")
    for _ in range(2):
        torch.matmul(a, b)
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        torch.matmul(a, b)
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return 2.0 * n ** 3 / (best * 1e-3) / 1e12, best


def main():
    import psutil
    print(json.dumps({"host_cores": len(os.sched_getaffinity(0)),
                      "host_mem_gb": psutil.virtual_memory().total / 2**30,
                      "host_mem_avail_gb": psutil.virtual_memory().available / 2**30}))
    for n in (4096, 8192):
        tf, ms = dgemm_peak(n)
        print(json.dumps({"kernel": "cublas_dgemm", "n": n, "ms": ms, "tflops": tf}))
    # sustained: back to back for ~3 s
    n = 8192
    a = torch.randn(n, n, dtype=torch.float64, device="cuda")
    b = torch.randn(n, n, dtype=torch.float64, device="cuda")
    torch.cuda.synchronize()
    t0 = time.time()
    cnt = 0
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    while time.time() - t0 < 3.0:
        torch.matmul(a, b)
        cnt += 1
        if cnt % 4 == 0:
            torch.cuda.synchronize()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    print(json.dumps({"kernel": "cublas_dgemm_sustained", "n": n, "count": cnt,
                      "tflops": 2.0 * n ** 3 * cnt / (ms * 1e-3) / 1e12}))


if __name__ == "__main__":
    main()
