"""Host-buffer pipeline probe (dev tool): vbatched_dpotrf_host on a C5 prefix vs raw copies."""
import ctypes
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbgen  # noqa: E402
import paper_conf_ipps_abdelfattahhtd16_b200 as vb  # noqa: E402
from harness import DeviceBatch  # noqa: E402

lim = int(sys.argv[1]) if len(sys.argv) > 1 else 12000
n = vbgen.sizes("C5")[:lim]
db = DeviceBatch(n, seed=5).fill()
torch.cuda.synchronize()
nbytes = db.arena.numel() * 8
hp = vb.vbatched_host_alloc(nbytes)
host = np.ctypeslib.as_array((ctypes.c_double * (nbytes // 8)).from_address(hp))
ht = torch.from_numpy(host)
hptrs = (hp + 8 * db.off).astype(np.int64)
info = np.zeros(db.B, dtype=np.int32)
flops = vbgen.expected_flops(n)
t = time.perf_counter(); ht.copy_(db.arena); torch.cuda.synchronize(); t_d2h = time.perf_counter() - t
t = time.perf_counter(); db.arena.copy_(ht); torch.cuda.synchronize(); t_h2d = time.perf_counter() - t
print(f"{nbytes/1e9:.1f} GB: raw d2h {nbytes/t_d2h/1e9:.1f} GB/s, h2d {nbytes/t_h2d/1e9:.1f} GB/s; floor (bidir 49.5) {2*nbytes/99e9:.3f} s")
for ws in (3 << 30, 6 << 30, 12 << 30):
    for rep in range(2):
        db.fill(); torch.cuda.synchronize(); ht.copy_(db.arena); torch.cuda.synchronize()
        t = time.perf_counter()
        vb.vbatched_dpotrf_host("L", db.n, hptrs, db.ldda, info, db.B, int(n.max()), workspace_bytes=ws)
        dt = time.perf_counter() - t
        print(f"ws {ws >> 30} GiB rep {rep}: {dt:.3f} s  {flops / dt / 1e9:.0f} GFLOP/s  ({2 * nbytes / dt / 1e9:.1f} GB/s both ways)")
vb.vbatched_host_free(hp)
