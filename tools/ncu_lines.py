"""Aggregate an ncu source page (--page source --csv --print-source cuda,sass) per CUDA line:
python tools/ncu_lines.py report.csv [top]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
f = None
hdr = None
out = []
for r in rows:
    if r and r[0] == "File Path":
        f = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < 8 or not r[0]:
        continue
    try:
        o = len(r) - len(hdr)  # embedded quotes in the source text can split it into extra fields
        s = int(r[4 + o])
        ni = int(r[5 + o])
    except ValueError:
        continue
    if r[2 + o] != '-':
        continue
    out.append((s, ni, f, int(r[0]), r[1][:90], int(r[7 + o] or 0)))
tot = sum(o[0] for o in out)
print("total samples", tot)
for s, ni, f, ln, src, ex in sorted(out, reverse=True)[:top]:
    print(f"{s:7d} {100 * s / tot:5.1f}% ni {ni:6d} {f}:{ln:<5d} ex {ex:>11d}  {src.strip()}")
