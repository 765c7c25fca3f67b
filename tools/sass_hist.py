"""Per-kernel SASS opcode histogram of libvbatched.so (the evidence that the kernels run on the
FP64 tensor cores and TMA: DMMA.8x8x4, UBLKCP, SYNCS.*), plus local-memory traffic (LDL/STL =
register spills). python tools/sass_hist.py [lib.so] > profiles/r02/sass_histogram.txt"""
import collections
import re
import subprocess
import sys

lib = sys.argv[1] if len(sys.argv) > 1 else "paper_conf_ipps_abdelfattahhtd16_b200/libvbatched.so"
out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
KEYS = ["DMMA", "DFMA", "DMUL", "DADD", "MUFU.RCP64H", "MUFU.RSQ64H", "UBLKCP", "SYNCS", "LDGSTS",
        "LDS", "STS", "LDG", "STG", "LDL", "STL", "SHFL", "BAR"]
cur, hist = None, {}
for line in out.splitlines():
    m = re.search(r"Function : (\S+)", line)
    if m:
        cur = m.group(1)
        hist[cur] = collections.Counter()
        continue
    m = re.match(r"\s+/\*[0-9a-f]+\*/\s+(?:@!?U?P\w+\s+)?([A-Z0-9_.]+)", line)
    if cur and m:
        op = m.group(1)
        for k in KEYS:
            if op == k or op.startswith(k + "."):
                hist[cur][k] += 1
        hist[cur]["total"] += 1
demangle = subprocess.run(["c++filt"], input="\n".join(hist), capture_output=True, text=True).stdout.split("\n")
print(f"# SASS opcode histogram of {lib} (cuobjdump -sass; static instruction counts)")
print("# columns: " + " ".join(KEYS + ["total"]))
for (name, h), dm in zip(hist.items(), demangle):
    if not name.startswith("_ZN2vb"):
        continue
    short = re.sub(r"\(.*", "", dm)[:110]
    print(f"{short}\n    " + " ".join(f"{k}={h[k]}" for k in KEYS + ["total"] if h[k]))
