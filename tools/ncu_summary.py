"""Key metrics of one ncu --set full report (first kernel) as JSON:
python tools/ncu_summary.py report.ncu-rep out.json"""
import csv
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__bytes_read.sum.per_second", "lts__t_sector_hit_rate.pct",
        "sm__inst_executed_pipe_tensor_subpipe_dmma.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "launch__occupancy_limit_shared_mem",
        "launch__occupancy_limit_registers"]
raw = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "raw", "--csv"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, u, v = rows[0], rows[1], rows[2]
out = {"kernel": v[h.index("Kernel Name")][:120]}
for k in KEYS:
    if k in h:
        out[k] = {"value": v[h.index(k)], "unit": u[h.index(k)]}
stalls = {}
for i, k in enumerate(h):
    if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued"):
        try:
            stalls[k.replace("smsp__pcsamp_warps_issue_stalled_", "")] = int(v[i].replace(",", ""))
        except ValueError:
            pass
tot = sum(stalls.values()) or 1
out["stall_samples_pct"] = {k: round(100.0 * s / tot, 1) for k, s in
                            sorted(stalls.items(), key=lambda x: -x[1]) if s}
json.dump(out, open(sys.argv[2], "w"), indent=1)
print(json.dumps(out, indent=1))
