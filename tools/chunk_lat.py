"""Ring latency of the blocked kernel with the matrices in HBM (debug build with -DVB_CHUNK_LAT):
python tools/chunk_lat.py <lib.so> [config|u<n>x<count>]. For the first 64 CTAs and 4096 ring
positions: how long the producer waited for a free slot, how long after issuing the copies a
chunk landed when the consumers had to wait for it, and how often they waited (SM cycles)."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["VBATCHED_LIB"] = os.path.abspath(sys.argv[1])
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbgen  # noqa: E402
import paper_conf_ipps_abdelfattahhtd16_b200 as vb  # noqa: E402
from harness import DeviceBatch  # noqa: E402

cfg = sys.argv[2] if len(sys.argv) > 2 else "u1024x600"
if cfg.startswith("u"):
    nn, cnt = (int(x) for x in cfg[1:].split("x"))
    n, seed = np.full(cnt, nn, dtype=np.int32), 3
else:
    n, seed = vbgen.sizes(cfg), vbgen.CONFIGS[cfg].seed
db = DeviceBatch(n, seed=seed).fill()
rec = torch.zeros(64 * 4096 * 8, dtype=torch.int64, device="cuda")
L = vb.lib()
L.vbatched_debug_chunk_lat.argtypes = [ctypes.c_void_p]
db.dpotrf()
torch.cuda.synchronize()
db.fill()
L.vbatched_debug_chunk_lat(ctypes.c_void_p(rec.data_ptr()))
torch.cuda.synchronize()
db.dpotrf()
torch.cuda.synchronize()
L.vbatched_debug_chunk_lat(ctypes.c_void_p(0))
r = rec.view(64, 4096, 8).cpu().numpy().astype(np.float64)
ok = (r[:, :, 0] > 0) & (r[:, :, 2] > 0) & (r[:, :, 3] > 0) & (r[:, :, 4] > 0)
r = r[ok]
empty_wait = r[:, 1] - r[:, 0]
issue = r[:, 2] - r[:, 1]
cons_wait = r[:, 4] - r[:, 3]
waited = cons_wait > 200
land = r[:, 4] - r[:, 2]  # issue done -> consumer released (the landing time when it waited)
lead = r[:, 3] - r[:, 2]  # issue done -> consumer arrived (how far ahead the producer was)
pct = lambda x: " ".join(f"p{q}={np.percentile(x, q):.0f}" for q in (10, 50, 90, 99))  # noqa: E731
print(f"{cfg}: {len(r)} chunks of 64 CTAs; consumers waited on {100 * waited.mean():.1f} % of them")
print(f"  consumer full-barrier wait      : mean {cons_wait.mean():.0f} cycles, {pct(cons_wait)}")
print(f"  producer empty-slot wait        : mean {empty_wait.mean():.0f}, {pct(empty_wait)}")
print(f"  producer issue (32 bulk copies) : mean {issue.mean():.0f}, {pct(issue)}")
print(f"  issue done -> consumer arrives  : {pct(lead)}")
print(f"  issue -> landed (waited chunks) : mean {land[waited].mean():.0f}, {pct(land[waited])}")
