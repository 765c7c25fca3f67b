#!/usr/bin/env python
"""bench.py — vbatched DPOTRF throughput on B200 (BASELINE.json metric).

Default workload: BASELINE.json configs[4] = C5, batchCount=40000, n uniform in [1,1024]
(the configuration the metric is quoted on at 1/2/4/8 GPUs; it fits one B200: 112 GB),
flop-balanced over the ranks (LPT on n^3/3), fixed total work -> "scaling": "strong".
`--config C1..C4` selects the other BASELINE configs (parity-test sizes; not the bench line).

One step = one vbatched_dpotrf of the whole (per-rank) batch through the C ABI
(vbatched_dpotrf_scan + vbatched_dpotrf_factor = exactly what vbatched_dpotrf runs),
inputs resident in HBM. The factorisation is in place, so before every step the inputs are
regenerated in place by the seeded device generator and L2 is flushed (both untimed); the
inputs (112 GB at N=1) are also far larger than L2. Each step is timed with CUDA events on
the launching stream; K steps are bracketed by barrier + synchronize; max over ranks.

Usage:  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
        torchrun --nproc-per-node N bench.py --gpus N ...
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import vbgen  # noqa: E402

METRIC = "vbatched DPOTRF GFLOP/s & % of FP64/HBM roofline at 1/2/4/8 B200"
PEAKS_FILE = os.path.join(ROOT, "profiles", "peaks_fp64.json")
MEASURED_PEAKS = os.path.join(ROOT, "MEASURED_PEAKS.json")


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--config", default="C5", choices=list(vbgen.CONFIGS))
    p.add_argument("--batch-limit", type=int, default=0,
                   help="profiling only: keep the first B matrices of the config")
    p.add_argument("--e2e-steps", type=int, default=2)
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--graph", action="store_true",
                   help="time replays of a CUDA graph that captured one vbatched_dpotrf call "
                        "(SURVEY.md §8(d): the launch-latency-free variant for C1/C2)")
    p.add_argument("--precision", default="d", choices=["d", "s"],
                   help="d: vbatched_dpotrf (the headline); s: vbatched_spotrf (FP32 storage, "
                        "FP64 arithmetic; no e2e / CPU legs)")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--cpu-seconds", type=float, default=8.0,
                   help="target wall seconds of the bounded oracle sample")
    p.add_argument("--clock-soak", type=float, default=1.0,
                   help="seconds of untimed back-to-back steps run under the clock sampler right "
                        "before the timed region (short configs: the timed region alone is too "
                        "short for nvidia-smi to sample)")
    return p.parse_args()


# ------------------------------------------------------------------------------ clocks
class ClockSampler:
    FIELDS = ["clocks.sm", "clocks.max.sm", "power.draw", "clocks_event_reasons.active",
              "clocks_event_reasons.hw_slowdown", "clocks_event_reasons.hw_thermal_slowdown",
              "clocks_event_reasons.sw_thermal_slowdown", "clocks_event_reasons.sw_power_cap"]

    def __init__(self, device_index: int):
        self.idx = device_index
        self.lines: list[str] = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.idx), f"--query-gpu={','.join(self.FIELDS)}",
                 "--format=csv,noheader,nounits", "-lms", "20"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception as e:  # pragma: no cover
            log("clock sampler unavailable:", e)
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                smax.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------------------ oracle sample
def oracle_sample(cfg, target_seconds, cores):
    """A deterministic bounded sample of the workload for the CPU oracle: every s-th matrix
    (global index), s chosen so the oracle needs about `target_seconds` on `cores` cores
    (rate estimate 1.5 GFLOP/s per core for the plain Crout loop)."""
    n_all = vbgen.sizes(cfg)
    total = vbgen.expected_flops(n_all)
    budget = target_seconds * cores * 1.5e9
    stride = max(1, int(np.ceil(total / budget)))
    idx = np.arange(0, len(n_all), stride)
    n = n_all[idx]
    ld = vbgen.ldda_for(n)
    off, tot = vbgen.arena_layout(n, ld)
    arena = np.zeros(tot)
    for j, g in enumerate(idx):
        nn = int(n[j])
        A = vbgen.f1_matrix(cfg.seed, int(g), nn, vbgen.is_nonspd(cfg, int(g)))
        blk = arena[off[j]: off[j] + int(ld[j]) * nn].reshape((int(ld[j]), nn), order="F")
        blk[:nn, :] = A
    flops = vbgen.expected_flops(n)
    desc = (f"every {stride}th matrix of {cfg.name} ({len(idx)} matrices, sum n^3/3 = "
            f"{flops / 1e9:.2f} GFLOP), OpenMP dynamic one matrix per core")
    return arena, off, n, ld, flops, desc


def run_oracle(arena0, off, n, ld, cores):
    import oracle
    arena = arena0.copy()
    t0 = time.perf_counter()
    info = oracle.dpotrf_batch(arena, off, n, ld, nthreads=cores)
    dt = time.perf_counter() - t0
    return dt, info


def lapack_baseline(arena0, off, n, ld, cores, desc):
    """The paper's best CPU competitor, LAPACK dpotrf one core per matrix,
    MKL from libtorch_cpu.so, on the oracle's sample: best of 3 (inputs restored untimed); the
    same with scipy's bundled OpenBLAS as `openblas` (SURVEY §8(d) secondary baseline)."""
    def one(lib_path, kind):
        import cpu_baselines
        best, info = None, None
        for _ in range(3):
            arena = arena0.copy()
            dt, info = cpu_baselines.dpotrf_batch(arena, off, n, ld, cores, lib_path=lib_path)
            best = dt if best is None else min(best, dt)
        return {"value": vbgen.expected_flops(n[info == 0]) / best / 1e9, "unit": "GFLOP/s",
                "cores": cores, "kind": kind, "sample": desc.replace("OpenMP dynamic",
                "pthreads, LPT order,"), "seconds": best}
    try:
        import cpu_baselines
        out = one(None, "MKL dpotrf one core per matrix" if cpu_baselines.is_mkl()
                  else "LAPACK dpotrf one core per matrix")
    except Exception as e:  # a reported baseline, not the product: record why it is missing
        return {"value": None, "unavailable": str(e)[:200]}
    try:
        ob = cpu_baselines.openblas_path()
        out["openblas"] = (one(ob, "OpenBLAS (scipy's bundled, LP64) dpotrf one core per matrix")
                           if ob else {"value": None, "unavailable": "scipy's OpenBLAS not found"})
    except Exception as e:
        out["openblas"] = {"value": None, "unavailable": str(e)[:200]}
    return out


def host_cores():
    return len(os.sched_getaffinity(0))


# ------------------------------------------------------------------------------ reference arm
def reference_arm(args, cfg, rank, world):
    if rank != 0:
        return  # rank 0 alone runs the CPU oracle; the other ranks exit without work
    cores = host_cores()
    per_step = min(15.0, max(2.0, 150.0 / max(1, args.steps + args.warmup)))
    arena0, off, n, ld, flops, desc = oracle_sample(cfg, per_step, cores)
    for _ in range(args.warmup):
        run_oracle(arena0, off, n, ld, cores)
    times = []
    for _ in range(args.steps):
        dt, info = run_oracle(arena0, off, n, ld, cores)
        times.append(dt)
    total = sum(times)
    ok_flops = vbgen.expected_flops(n[info == 0])
    value = ok_flops * args.steps / total / 1e9
    line = {
        "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": total / args.steps * 1e3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "impl": "reference",
        "config": config_dict(cfg, world),
        "cpu_baseline": {"value": value, "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
                         "sample": desc},
        "e2e": {"value": value, "unit": "GFLOP/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def config_dict(cfg, world):
    return {"workload": f"{cfg.name}: {cfg.desc} (BASELINE.json configs[{list(vbgen.CONFIGS).index(cfg.name)}])",
            "batch": cfg.batch, "dist": cfg.dist, "nmax": cfg.nmax, "seed": cfg.seed,
            "ldda": "roundup(n,32)", "values": "F1: a_ij=u in [0,1), a_ii=u+n (hash generator)",
            "l2": "inputs regenerated in place + 256 MB L2 flush before every step (untimed)",
            "parallelism": f"LPT shards over {world} GPU(s), no data-path collective"}


# ------------------------------------------------------------------------------ our arm
def load_fp64_peak():
    try:
        with open(PEAKS_FILE) as f:
            d = json.load(f)
        return float(d["fp64_tflops"]), d.get("source", PEAKS_FILE)
    except Exception:
        return 37.0, "fallback: B200 HGX nominal FP64 (37 TF/s)"


def load_hbm_peak():
    try:
        with open(MEASURED_PEAKS) as f:
            return float(json.load(f)["hbm_gbs"]), "MEASURED_PEAKS.json hbm_gbs (measured)"
    except Exception:
        return 6650.0, "fallback: B200_PROFILING.md 6.65 TB/s"


def load_traffic(cfg_name):
    p = os.path.join(ROOT, "profiles", f"ncu_traffic_{cfg_name}.json")
    try:
        with open(p) as f:
            return json.load(f)
    except Exception:
        return None


def our_arm(args, cfg, rank, world, local_rank):
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_abdelfattahhtd16_b200 as vb
    from harness import DeviceBatch

    dev = torch.device("cuda", local_rank)
    torch.cuda.set_device(dev)
    n_all = vbgen.sizes(cfg)
    if args.batch_limit:
        n_all = n_all[: args.batch_limit]
    from paper_conf_ipps_abdelfattahhtd16_b200 import shard
    mine = shard.shard_indices(n_all, world, rank)  # LPT on n^3/3, identical on every rank
    n_loc = n_all[mine]
    single = args.precision == "s"
    if single:
        args.no_e2e = True
        args.no_cpu_baseline = True
    db = DeviceBatch(n_loc, seed=cfg.seed, gidx=mine, nonspd_mod=cfg.nonspd_mod, device=dev,
                     dtype="f32" if single else "f64")
    ws = torch.empty(vb.vbatched_dpotrf_workspace_size(db.B), dtype=torch.uint8, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream(dev)
    max_n = int(n_all.max())
    launches_per_step = vb.vbatched_dpotrf_kernel_launches(max_n)  # scan + per-range kernels

    def prepare():
        db.fill()
        flush.fill_(1)  # evict the inputs' tail from L2

    def step(ev):
        # the product call: scan and factorisation kernels chained with PDL on one stream
        torch.cuda.nvtx.range_push("vbatched_dpotrf")
        ev[0].record(stream)
        db.dpotrf(max_n=max_n, stream=stream)  # vbatched_dpotrf (or vbatched_spotrf)
        ev[1].record(stream)
        torch.cuda.nvtx.range_pop()

    def step_split(ev):
        # the same kernels through the two-phase API, an event between the scan and the
        # factorisation launches: the factorisation kernels' own duration (roofline)
        ev[0].record(stream)
        if single:  # no two-phase API for FP32: the whole call (scan included) is timed
            ev[1].record(stream)
            db.dpotrf(max_n=max_n, stream=stream)
        else:
            vb.vbatched_dpotrf_scan("L", db.d_n, db.d_ldda, db.d_info, db.B, max_n, ws, stream)
            ev[1].record(stream)
            vb.vbatched_dpotrf_factor("L", db.d_n, db.d_ptrs, db.d_ldda, db.d_info, db.B, max_n,
                                      ws, stream)
        ev[2].record(stream)

    def barrier():
        if world > 1:
            dist.barrier()

    for _ in range(args.warmup):
        prepare()
        step([torch.cuda.Event(enable_timing=True) for _ in range(2)])
    torch.cuda.synchronize()
    if args.graph:
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph):
            db.dpotrf(max_n=max_n)  # captured on the graph's stream (workspace alloc/free nodes too)
        torch.cuda.synchronize()

        def step(ev):  # noqa: F811 — the timed step becomes one graph replay
            ev[0].record(stream)
            graph.replay()
            ev[1].record(stream)

        for _ in range(args.warmup):
            prepare()
            step([torch.cuda.Event(enable_timing=True) for _ in range(2)])
        torch.cuda.synchronize()
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(args.steps)]
    sampler = ClockSampler(local_rank)
    barrier()
    torch.cuda.synchronize()
    sampler.start()
    # clock soak: the same prepare+step sequence, untimed, for >= --clock-soak seconds, so that
    # the sampler (20 ms period) sees the clocks under this load even when the K timed steps
    # last only a few ms (C1-C4); the timed region follows immediately
    t_soak = time.perf_counter()
    soak_steps = 0
    while time.perf_counter() - t_soak < args.clock_soak:
        prepare()
        step([torch.cuda.Event(enable_timing=True) for _ in range(2)])
        soak_steps += 1
        if soak_steps % 8 == 0:
            torch.cuda.synchronize()
    torch.cuda.synchronize()
    barrier()
    torch.cuda.synchronize()
    for k in range(args.steps):
        prepare()
        step(evs[k])
    torch.cuda.synchronize()
    barrier()
    clocks = sampler.stop()
    clocks["window"] = (f"{args.clock_soak:.1f} s soak of the same steps ({soak_steps} untimed) "
                        "immediately before the timed region + the timed region, 20 ms period")
    step_ms = [e[0].elapsed_time(e[1]) for e in evs]
    # roofline pass (after the timed region, same inputs and launch configuration): K steps
    # of the two-phase API, CUDA events around the factorisation launches
    evk = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
    for k in range(args.steps):
        prepare()
        step_split(evk[k])
    torch.cuda.synchronize()
    kern_ms = [e[1].elapsed_time(e[2]) for e in evk]
    scan_ms = [e[0].elapsed_time(e[1]) for e in evk]
    info = db.info()
    ok_local = vbgen.expected_flops(n_loc[info == 0])
    alg_bytes_local = vbgen.algorithmic_bytes(n_loc[info == 0]) * (0.5 if single else 1.0)
    # global info[] from every rank's (index, info) pairs; flops count only info == 0 matrices
    info_all = shard.gather_info(len(n_all), mine, info, device=dev)
    bad_info = int(np.sum(info_all != expected_info(cfg, n_all, np.arange(len(n_all)))))
    max_total_ms = shard.max_over_ranks(sum(step_ms), device=dev)
    flops_total = vbgen.expected_flops(n_all[info_all == 0])
    per_rank_ms = [sum(step_ms) / args.steps]
    if world > 1:
        t = torch.tensor([sum(step_ms) / args.steps], dtype=torch.float64, device=dev)
        allt = [torch.zeros_like(t) for _ in range(world)]
        dist.all_gather(allt, t)
        per_rank_ms = [float(x.item()) for x in allt]
    value = flops_total * args.steps / (max_total_ms / 1e3) / 1e9

    # roofline of the factorisation launches (everything after the scan) on this rank
    kern_avg_s = sum(kern_ms) / args.steps / 1e3
    if cfg.nmax >= 256:
        peak, src = load_fp64_peak()
        achieved = ok_local / kern_avg_s / 1e12
        roof = {"bound": "tensor", "achieved": achieved, "peak": peak, "unit": "TFLOP/s",
                "frac": achieved / peak, "peak_source": src}
    else:
        peak, src = load_hbm_peak()
        achieved = alg_bytes_local / kern_avg_s / 1e9
        roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "peak_source": src}
    tr = load_traffic(cfg.name + ("_s" if single else ""))
    roof["traffic"] = tr.get("bytes_per_launch") if tr else None
    if tr:
        roof["traffic_source"] = ("NOT measured in this run: read from the committed ncu capture "
                                  f"profiles/ncu_traffic_{cfg.name}.json ({tr.get('source')})")
    roof["kernel"] = vb.factor_kernel_names(max_n)
    roof["kernel_ms"] = sum(kern_ms) / args.steps
    roof["scan_ms"] = sum(scan_ms) / args.steps
    roof["timing"] = ("kernel_ms: CUDA events around the factorisation launches in a second pass "
                      "of --steps steps through the two-phase API (vbatched_dpotrf_scan | event | "
                      "vbatched_dpotrf_factor) right after the timed region; value/ms_per_step: "
                      "the single vbatched_dpotrf call (scan and factorisation PDL-chained)")

    # ---------------- e2e through the host-buffer C-ABI entry point
    e2e = None
    if not args.no_e2e:
        e2e = e2e_leg(args, cfg, db, n_loc, max_n, world, dev)

    # ---------------- CPU baseline (rank 0, N=1 only)
    cpu = cpu_lapack = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cores = host_cores()
        arena0, off, n_s, ld_s, fl, desc = oracle_sample(cfg, args.cpu_seconds, cores)
        dt, info_s = run_oracle(arena0, off, n_s, ld_s, cores)
        cpu = {"value": vbgen.expected_flops(n_s[info_s == 0]) / dt / 1e9, "unit": "GFLOP/s",
               "cores": cores, "kind": "oracle", "sample": desc, "seconds": dt}
        cpu_lapack = lapack_baseline(arena0, off, n_s, ld_s, cores, desc)

    if rank == 0:
        line = {
            "metric": METRIC if not single else METRIC.replace("DPOTRF", "SPOTRF"),
            "value": value, "unit": "GFLOP/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": max_total_ms / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "f64" if not single else "f64 (f32 storage)",
            "data": "synthetic", "config": config_dict(cfg, world),
            "roofline": roof, "cpu_baseline": cpu, "cpu_lapack": cpu_lapack, "e2e": e2e,
            "gpu_launches": launches_per_step * args.steps, "clocks": clocks,
            "ms_per_step_median": float(np.median(step_ms)), "ms_per_step_best": float(min(step_ms)),
            "info_mismatches": bad_info,
            "per_rank_ms": per_rank_ms,
            "library": vb.vbatched_version(),
        }
        if args.batch_limit:
            line["config"]["batch_limit"] = args.batch_limit
        if args.graph:
            line["config"]["launch"] = "CUDA graph replay of one vbatched_dpotrf call"
        print(json.dumps(line), flush=True)


def expected_info(cfg, n, gidx):
    out = np.zeros(len(n), dtype=np.int32)
    if cfg.nonspd_mod:
        for j, g in enumerate(gidx):
            if vbgen.is_nonspd(cfg, int(g)):
                out[j] = vbgen.nonspd_k(cfg.seed, int(g), int(n[j]))
    return out


def e2e_leg(args, cfg, db, n_loc, max_n, world, dev):
    """Same metric through vbatched_dpotrf_host: inputs in pinned host memory, H2D + factor +
    D2H of the whole batch inside the timed call (host wall clock around a blocking call,
    synchronised on both sides; max over ranks)."""
    import ctypes

    import psutil
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_abdelfattahhtd16_b200 as vb
    nbytes = int(db.arena.numel()) * 8
    avail = psutil.virtual_memory().available
    if nbytes * world + (24 << 30) > avail:
        return {"value": None, "unit": "GFLOP/s",
                "skipped": f"host memory: need {nbytes * world / 2**30:.1f} GiB pinned, "
                           f"{avail / 2**30:.1f} GiB available"}
    hp = vb.vbatched_host_alloc(nbytes)
    try:
        host = np.ctypeslib.as_array((ctypes.c_double * (nbytes // 8)).from_address(hp))
        host_t = torch.from_numpy(host)
        hptrs = (hp + 8 * db.off).astype(np.int64)
        info = np.zeros(db.B, dtype=np.int32)
        times = []
        for it in range(1 + args.e2e_steps):
            db.fill()
            torch.cuda.synchronize()
            host_t.copy_(db.arena)  # restore the host inputs (untimed)
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            t0 = time.perf_counter()
            vb.vbatched_dpotrf_host("L", db.n, hptrs, db.ldda, info, db.B, max_n)
            torch.cuda.synchronize()
            t1 = time.perf_counter()
            if it > 0:
                times.append(t1 - t0)
        ok = vbgen.expected_flops(n_loc[info == 0])
        loc = torch.tensor([sum(times), ok], dtype=torch.float64, device=dev)
        if world > 1:
            allv = [torch.zeros_like(loc) for _ in range(world)]
            dist.all_gather(allv, loc)
            allv = torch.stack(allv).cpu().numpy()
        else:
            allv = loc.cpu().numpy()[None, :]
        tmax = float(allv[:, 0].max()) / args.e2e_steps
        payload = int(np.sum(db.ldda.astype(np.int64) * np.maximum(n_loc, 0))) * 8
        return {"value": float(allv[:, 1].sum()) / tmax / 1e9, "unit": "GFLOP/s",
                "h2d_bytes_per_step": payload + 16 * db.B, "d2h_bytes_per_step": payload + 4 * db.B,
                "steps": args.e2e_steps, "s_per_step": tmax,
                "api": "vbatched_dpotrf_host (pinned host buffers, 3-slot 6 GiB device staging ring)"}
    finally:
        vb.vbatched_host_free(hp)


def relaunch_under_torchrun(args) -> int:
    """`python bench.py --gpus N` (N > 1) without torchrun: re-launch this command as N ranks
    (one process per GPU) through torch.distributed.run on 127.0.0.1, so that --gpus N always
    measures N ranks. Returns torchrun's exit code."""
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={args.gpus}", "--master-addr=127.0.0.1", f"--master-port={port}",
           os.path.abspath(__file__), *sys.argv[1:]]
    log("bench: --gpus", args.gpus, "without WORLD_SIZE: re-launching as", " ".join(cmd[1:6]))
    return subprocess.call(cmd)


def main():
    args = parse()
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        sys.exit(relaunch_under_torchrun(args))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        log(f"error: WORLD_SIZE={world} but --gpus={args.gpus}: the line would report the wrong "
            "GPU count")
        sys.exit(2)
    cfg = vbgen.CONFIGS[args.config]
    if args.impl == "reference":
        reference_arm(args, cfg, rank, world)
        return
    import torch
    if os.environ.get("VB_BENCH_SHARE_GPU"):
        # test hook: all ranks on cuda:0 with gloo collectives, to exercise the multi-rank
        # path (shards, max-over-ranks time, info gather) on a one-GPU box. Never a bench value.
        local_rank = 0
    if world > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        if os.environ.get("VB_BENCH_SHARE_GPU"):
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    try:
        our_arm(args, cfg, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
