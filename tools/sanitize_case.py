"""Workloads for compute-sanitizer (tools/sanitize.sh): small enough for the tools' replay
overhead, covering every kernel and protocol of one vbatched_dpotrf call.

  c1     BASELINE C1 (100 x U{1..32}): the direct warp kernel.
  mixed  200 matrices spanning all three factorisation kernels (n in 1..700), 'L' and 'U',
         roundup-32 and odd ldda (the cp.async gather instead of TMA bulk copies), failing
         pivots (-> early termination, the TMA ring drain, the look-ahead barrier exits).
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


def mixed():
    rng = np.random.default_rng(200)
    n = np.concatenate([rng.integers(1, 33, 60), rng.integers(33, 129, 80), rng.integers(129, 701, 60)]).astype(np.int32)
    for uplo in ("L", "U"):
        for mode in ("pad32", "odd"):
            db = DeviceBatch(n, seed=201, nonspd_mod=9, ldda_mode=mode).fill(poison=True, uplo=uplo)
            db.dpotrf(uplo=uplo)
            torch.cuda.synchronize()
            info = db.info()
            exp = np.array([vbgen.nonspd_k(201, g, int(n[g])) if g % 9 == 8 else 0 for g in range(len(n))])
            assert np.array_equal(info, exp), (uplo, mode)
    print("mixed ok")


if __name__ == "__main__":
    {"c1": c1, "mixed": mixed}[sys.argv[1]]()
    print("case ok", sys.argv[1])
