"""Time vbatched_dpotrf on configs / uniform batches (dev tool; no L2 flush beyond the in-place
regeneration): python tools/cfgtime.py C3 C4 u512x2000 ...  -> best/median ms and GFLOP/s"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbgen  # noqa: E402
from harness import DeviceBatch  # noqa: E402

reps = int(os.environ.get("REPS", "5"))
tag = os.environ.get("TAG", "")
uplo = os.environ.get("UPLO", "L")
dtype = os.environ.get("DTYPE", "f64")
for cfg in sys.argv[1:]:
    if "x" in cfg and cfg.startswith("C"):  # e.g. C2x4: config C2's distribution, 4x the batch
        base, mult = cfg.split("x")
        c0 = vbgen.CONFIGS[base]
        c = vbgen.Config(cfg, c0.batch * int(mult), c0.dist, c0.nmax, c0.seed, c0.nonspd_mod)
        n, seed, mod = vbgen.sizes(c), c.seed, c.nonspd_mod
    elif cfg.startswith("u"):
        nn, cnt = (int(x) for x in cfg[1:].split("x"))
        n, seed, mod = np.full(cnt, nn, dtype=np.int32), 3, 0
    else:
        c = vbgen.CONFIGS[cfg]
        n, seed, mod = vbgen.sizes(cfg), c.seed, c.nonspd_mod
    db = DeviceBatch(n, seed=seed, nonspd_mod=mod, dtype=dtype)
    ts = []
    for it in range(reps + 1):
        db.fill(uplo=uplo)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        db.dpotrf(uplo=uplo)
        e1.record()
        torch.cuda.synchronize()
        if it:
            ts.append(e0.elapsed_time(e1))
    info = db.info()
    ok = info == 0
    fl = float(np.sum(n[ok].astype(np.float64) ** 3 / 3))
    b, m = min(ts), float(np.median(ts))
    print(f"{tag} {cfg:10s} best {b:9.3f} ms  med {m:9.3f} ms  {fl / (b * 1e-3) / 1e9:9.1f} GFLOP/s (best)"
          f"  nonzero info {int((~ok).sum())}", flush=True)
    del db
    torch.cuda.empty_cache()
