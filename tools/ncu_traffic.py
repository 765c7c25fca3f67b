"""Summarise an ncu launch list (--metrics gpu__time_duration.sum,dram__bytes_read.sum,
dram__bytes_write.sum --csv) of one bench step: per-kernel time shares and DRAM bytes of the
factorisation launches, written to profiles/ncu_traffic_<cfg>.json for bench.py's roofline
`traffic` field.  python tools/ncu_traffic.py launches.csv C5 [source-note]"""
import csv
import json
import os
import sys

path, cfg = sys.argv[1], sys.argv[2]
rows = [r for r in csv.reader(open(path)) if len(r) > 10]
hdr = rows[0]
ki, mi, vi, idi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("ID")
per = {}
for r in rows[1:]:
    name = r[ki]
    if "vb::" not in name or "scan_bin" in name:  # factorisation launches only
        continue
    short = name.split("(")[0].replace("void ", "")
    d = per.setdefault(r[idi], {"kernel": short})
    d[r[mi]] = float(r[vi].replace(",", ""))
launches = list(per.values())
# one bench step = the last complete set of factorisation launches
by_kernel = {}
for d in launches:
    k = by_kernel.setdefault(d["kernel"], {"launches": 0, "ns": 0.0, "dram_bytes": 0.0})
    k["launches"] += 1
    k["ns"] += d.get("gpu__time_duration.sum", 0.0)
    k["dram_bytes"] += d.get("dram__bytes_read.sum", 0.0) + d.get("dram__bytes_write.sum", 0.0)
steps = max(v["launches"] for v in by_kernel.values())
tot_ns = sum(v["ns"] for v in by_kernel.values())
out = {
    "config": cfg,
    "bytes_per_launch": sum(v["dram_bytes"] for v in by_kernel.values()) / steps,
    "per_kernel": {k: {"bytes_per_step": v["dram_bytes"] / steps, "ms_per_step": v["ns"] / steps / 1e6,
                       "time_share": v["ns"] / tot_ns} for k, v in by_kernel.items()},
    "steps_in_list": steps,
    "source": (sys.argv[3] if len(sys.argv) > 3 else "") +
              f" ncu launch list {os.path.basename(path)} (dram__bytes_read.sum + dram__bytes_write.sum, "
              "--clock-control none, serialised cold launches); sum over the factorisation launches per step",
}
json.dump(out, open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                 "profiles", f"ncu_traffic_{cfg}.json"), "w"), indent=1)
print(json.dumps(out, indent=1))
