"""Phase breakdown of the v2 blocked kernel (debug build with -DVB_PHASE_PROF):
python tools/phase_prof.py <lib.so> [config] [batch_limit]"""
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

cfg = sys.argv[2] if len(sys.argv) > 2 else "C5"
lim = int(sys.argv[3]) if len(sys.argv) > 3 else 0
if cfg.startswith("u"):  # uniform size: u<n>x<count>
    nn, cnt = (int(x) for x in cfg[1:].split("x"))
    n = np.full(cnt, nn, dtype=np.int32)
    seed = 3
else:
    n = vbgen.sizes(cfg)
    seed = vbgen.CONFIGS[cfg].seed
if lim:
    n = n[:lim]
db = DeviceBatch(n, seed=seed, dtype=os.environ.get("DTYPE", "f64")).fill()
L = vb.lib()
L.vbatched_debug_phases.argtypes = [ctypes.c_void_p, ctypes.c_int]
out = (ctypes.c_ulonglong * 8)()
db.dpotrf()
torch.cuda.synchronize()
L.vbatched_debug_phases(ctypes.addressof(out), 1)
db.fill()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
db.dpotrf()
e1.record()
torch.cuda.synchronize()
L.vbatched_debug_phases(ctypes.addressof(out), 1)
if os.environ.get("QUAD"):  # quad small kernel: slots 0-2 chain warp, 3-6 the 3 DMMA warps, 7 all 4
    names = ["chain:wait_tile", "chain:potf2", "chain:trtri", "dmma:pre_kloop", "dmma:wait_inv",
             "dmma:strips", "dmma:tile_build", "all:matrix"]
    scale = [1, 1, 1, 1 / 3, 1 / 3, 1 / 3, 1 / 3, 1 / 4]
    tot = out[7] / 4
    print(f"{cfg} kernel {e0.elapsed_time(e1):.3f} ms; cycles per warp of each role (sum over CTAs)")
    for i, nm in enumerate(names):
        v = out[i] * scale[i]
        print(f"  {nm:18s} {v:16.0f}  {100.0 * v / max(tot, 1):6.1f} % of matrix time")
    sys.exit(0)
names = (["gemm", "potf2", "trtri", "trsm", "matrix_total", "panel_bar"] if os.environ.get("SMALL") else
         ["kloop", "diag", "trsm+store", "panel_end", "matrix_total", "kloop_full_wait"])
tot = out[4]
print(f"{cfg} lim={lim} kernel {e0.elapsed_time(e1):.3f} ms; per-CTA-warp0 cycles (sum over CTAs):")
for i, nm in enumerate(names):
    print(f"  {nm:14s} {out[i]:16d}  {100.0 * out[i] / max(tot, 1):6.1f} %")
