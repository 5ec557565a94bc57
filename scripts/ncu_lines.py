"""Aggregate an `ncu --page source --print-source cuda,sass --csv` export by source line:
instructions executed and warp-stall samples per (file, line).  Usage: ncu_lines.py export.csv [top]"""
import csv
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
agg = defaultdict(lambda: [0, 0, ""])
fname, line, src = "?", None, ""
hdr = None
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None:
        continue
    if r[0] != "":
        line, src = r[0], r[1]
        continue
    try:
        ie = float(r[hdr.index("Instructions Executed")]) if "Instructions Executed" in hdr else 0.0
        st = float(r[hdr.index("Warp Stall Sampling (All Samples)")])
    except (ValueError, IndexError):
        continue
    a = agg[(fname, line)]
    a[0] += ie
    a[1] += st
    a[2] = src
tot_i = sum(v[0] for v in agg.values()) or 1
tot_s = sum(v[1] for v in agg.values()) or 1
print(f"total instructions {tot_i:.3g}, stall samples {tot_s:.3g}")
for key in ("stall", "inst"):
    print(f"--- top by {key}")
    items = sorted(agg.items(), key=lambda kv: -(kv[1][1] if key == "stall" else kv[1][0]))[:top]
    for (f, l), (ie, st, s) in items:
        print(f"{f}:{l:>5}  inst {100 * ie / tot_i:5.1f}%  stall {100 * st / tot_s:5.1f}%  {s.strip()[:90]}")
