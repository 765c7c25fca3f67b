"""Predict multi-GPU strong scaling on one GPU: time the LPT shard of rank 0 (and the largest
shard by flops) of C5 for N = 1, 2, 4, 8 ranks, each shard generated from the global matrix
indices exactly as bench.py does. python tools/shard_time.py [config]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbgen  # noqa: E402
from harness import DeviceBatch  # noqa: E402
from paper_conf_ipps_abdelfattahhtd16_b200 import shard  # noqa: E402

cfg = vbgen.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C5"]
n_all = vbgen.sizes(cfg)
flops_all = float(np.sum(n_all.astype(np.float64) ** 3 / 3))
t1 = None
for world in (1, 2, 4, 8):
    worst = 0.0
    loads = []
    for rank in range(world):
        mine = shard.shard_indices(n_all, world, rank)
        loads.append(float(np.sum(n_all[mine].astype(np.float64) ** 3 / 3)))
    rank = int(np.argmax(loads))  # the most loaded rank sets the makespan
    mine = shard.shard_indices(n_all, world, rank)
    db = DeviceBatch(n_all[mine], seed=cfg.seed, gidx=mine, nonspd_mod=cfg.nonspd_mod)
    ts = []
    for it in range(4):
        db.fill()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        db.dpotrf()
        e1.record()
        torch.cuda.synchronize()
        if it:
            ts.append(e0.elapsed_time(e1))
    t = min(ts)
    if world == 1:
        t1 = t
    print(f"N={world}: most loaded rank {rank}: {len(mine)} matrices, {loads[rank] / 1e9:.1f} GFLOP "
          f"(imbalance {max(loads) / (flops_all / world) - 1:.2e}), {t:.2f} ms -> predicted "
          f"{flops_all / (t * 1e-3) / 1e12:.2f} TF/s total, speed-up {t1 / t:.2f}x", flush=True)
    del db
    torch.cuda.empty_cache()
