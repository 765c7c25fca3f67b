"""Per-matrix timeline of one vbatched_dpotrf call (debug build with -DVB_TIMELINE):
python tools/timeline.py <lib.so> [config|u<n>x<count>] ...

Prints, per config: the call's span, per kernel the matrices, first start / last end, the
mean matrix duration per size bucket, and the concurrency profile (matrices in flight per SM
over time), which shows the tail of each persistent kernel."""
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

KIND = {30: "blocked", 20: "small", 21: "small_la", 22: "small_la2", 23: "quad", 40: "warp"}
L = vb.lib()
L.vbatched_debug_timeline.argtypes = [ctypes.c_void_p]

for cfg in sys.argv[2:] or ["C3"]:
    if cfg.startswith("u"):
        nn, cnt = (int(x) for x in cfg[1:].split("x"))
        n = np.full(cnt, nn, dtype=np.int32)
        seed = 3
    else:
        n = vbgen.sizes(cfg)
        seed = vbgen.CONFIGS[cfg].seed
    db = DeviceBatch(n, seed=seed).fill()
    tl = torch.zeros(4 * len(n), dtype=torch.int64, device="cuda")
    L.vbatched_debug_timeline(tl.data_ptr())
    db.dpotrf()
    torch.cuda.synchronize()
    db.fill()
    tl.zero_()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    db.dpotrf()
    e1.record()
    torch.cuda.synchronize()
    L.vbatched_debug_timeline(None)
    t = tl.cpu().numpy().reshape(-1, 4)
    ok = t[:, 1] > 0
    t0 = t[ok, 0].min()
    st, en = (t[:, 0] - t0) / 1e3, (t[:, 1] - t0) / 1e3  # us
    dur = en - st
    flops = float(np.sum(n.astype(np.float64) ** 3 / 3))
    print(f"== {cfg}: call {e0.elapsed_time(e1) * 1e3:.1f} us (events), matrices timed {ok.sum()}/{len(n)}, "
          f"span {en[ok].max():.1f} us, {flops / (en[ok].max() * 1e-6) / 1e9:.0f} GFLOP/s over the span")
    for k in sorted(set(t[ok, 3].tolist())):
        sel = ok & (t[:, 3] == k)
        nk = n[sel]
        kf = float(np.sum(nk.astype(np.float64) ** 3 / 3))
        print(f"  {KIND.get(k, k):7s} {sel.sum():6d} matrices n {nk.min()}..{nk.max()}: start {st[sel].min():8.1f} "
              f"last start {st[sel].max():8.1f} end {en[sel].max():8.1f} us; flops {100 * kf / flops:5.1f} %; "
              f"sum dur {dur[sel].sum():.0f} us")
        edges = np.unique(np.linspace(nk.min(), nk.max() + 1, 7).astype(int))
        for a, b in zip(edges[:-1], edges[1:]):
            s2 = sel & (n >= a) & (n < b)
            if s2.sum():
                mf = float(np.mean(n[s2].astype(np.float64) ** 3 / 3))
                print(f"      n [{a:4d},{b:4d}): {s2.sum():5d}  mean dur {dur[s2].mean():8.1f} us "
                      f"(min {dur[s2].min():7.1f} max {dur[s2].max():7.1f})  {mf / (dur[s2].mean() * 1e-6) / 1e9:7.1f} GF/s/matrix")
    # concurrency profile: matrices in flight (all kernels) sampled over the span
    T = en[ok].max()
    grid = np.linspace(0, T, 21)
    prof = []
    for x in grid[:-1] + (grid[1] - grid[0]) / 2:
        prof.append(int(np.sum(ok & (st <= x) & (en > x))))
    print("  in flight (20 slices):", prof)
