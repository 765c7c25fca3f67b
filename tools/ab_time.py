"""A/B timing of vbatched_dpotrf from different builds of libvbatched.so (development tool):
python tools/ab_time.py <config> <lib.so> [<lib.so> ...] — interleaved reps, median ms each.
Minimal ctypes (only vbatched_dpotrf), so libraries from older commits load too."""
import ctypes
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbgen  # noqa: E402
from harness import DeviceBatch  # noqa: E402

cfg = vbgen.CONFIGS[sys.argv[1]]
libs = []
for p in sys.argv[2:]:
    L = ctypes.CDLL(os.path.abspath(p))
    L.vbatched_dpotrf.argtypes = [ctypes.c_char, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                  ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
    libs.append((p, L))
n = vbgen.sizes(cfg)
db = DeviceBatch(n, seed=cfg.seed, nonspd_mod=cfg.nonspd_mod)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
st = torch.cuda.current_stream().cuda_stream
times = {p: [] for p, _ in libs}
reps = int(os.environ.get("REPS", "8"))
for rep in range(reps + 2):
    for p, L in libs:
        db.fill()
        flush.fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        rc = L.vbatched_dpotrf(b"L", db.d_n.data_ptr(), db.d_ptrs.data_ptr(), db.d_ldda.data_ptr(),
                               db.d_info.data_ptr(), db.B, cfg.nmax, st)
        e1.record()
        torch.cuda.synchronize()
        assert rc == 0
        if rep >= 2:
            times[p].append(e0.elapsed_time(e1))
for p, _ in libs:
    print(f"{cfg.name} {os.path.basename(p):28s} median {statistics.median(times[p]):9.3f} ms  best {min(times[p]):9.3f}")
