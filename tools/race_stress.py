"""Race stress (dev tool): factor the same batch repeatedly and require bit-identical results
(every matrix is factored by one CTA in a fixed order, so any difference is a race).
python tools/race_stress.py CFG [reps]"""
import os
import sys

sys.path.insert(0, os.getcwd())
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbgen  # noqa: E402
from harness import DeviceBatch  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
if cfg.startswith("u"):
    nn, cnt = (int(x) for x in cfg[1:].split("x"))
    n = np.full(cnt, nn, dtype=np.int32)
    seed, mod = 3, 0
else:
    c = vbgen.CONFIGS[cfg]
    n = vbgen.sizes(c)
    seed, mod = c.seed, c.nonspd_mod
db = DeviceBatch(n, seed=seed, nonspd_mod=mod)
ref = None
bad = 0
junk = torch.empty(1 << 28, dtype=torch.uint8, device="cuda")
for r in range(reps):
    db.fill()
    junk.random_(0, 256)  # scramble L2 / leave arbitrary bits around
    db.dpotrf(max_n=int(n.max()))
    torch.cuda.synchronize()
    out = db.arena.clone()
    info = db.info()
    if ref is None:
        ref, ref_info = out, info
        continue
    if not torch.equal(out.view(torch.int64), ref.view(torch.int64)) or not np.array_equal(info, ref_info):
        bad += 1
        diff = (out.view(torch.int64) != ref.view(torch.int64)).nonzero().flatten()
        first = int(diff[0]) if len(diff) else -1
        mi = int(np.searchsorted(db.off, first, side="right") - 1) if first >= 0 else -1
        print(f"rep {r}: {len(diff)} differing doubles, first at {first} (matrix {mi}, n={n[mi] if mi>=0 else -1})", flush=True)
        if mi >= 0:
            ld = int(db.ldda[mi])
            loc = diff.cpu().numpy() - int(db.off[mi])
            loc = loc[(loc >= 0) & (loc < ld * int(n[mi]))]
            rows, cols = loc % ld, loc // ld
            j0 = (cols.min() // 64) * 64
            sel = cols < j0 + 32
            print("   panel j0", j0, "rows wrong in panel cols 0..31:", np.unique(rows[sel]).tolist()[:40], flush=True)
            print("   rows", rows.min(), rows.max(), "cols", cols.min(), cols.max(),
                  "col hist", np.unique(cols // 16, return_counts=True), flush=True)
            a = out[int(db.off[mi]) + loc[:5]].cpu().numpy(); b = ref[int(db.off[mi]) + loc[:5]].cpu().numpy()
            print("   vals", a, b, flush=True)
print(f"{cfg}: {reps} reps, {bad} differing", flush=True)
