#!/usr/bin/env python
"""Summarise an `ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,... --csv` launch list of
one search (scripts/prof_search.py): per launch (in order) and per kernel (summed), the device time
share, DRAM bytes and tensor-pipe %.  Launches are cold-cache and serialised under ncu: compare
shares, not absolute times.  Usage: ncu_summary.py launches.csv"""
import csv
import io
import sys
from collections import OrderedDict, defaultdict

txt = open(sys.argv[1]).read()
i = txt.find('"ID"')
rows = list(csv.reader(io.StringIO(txt[i:])))
h = rows[0]
ki, mi, ui, vi, idi = (h.index(c) for c in ("Kernel Name", "Metric Name", "Metric Unit", "Metric Value", "ID"))
launch = OrderedDict()
scale = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3,
         "byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1.0, "Gbyte": 1e3, "%": 1.0}
for r in rows[1:]:
    d = launch.setdefault(int(r[idi]), {"name": r[ki].split("(")[0].replace("void ", "").replace("mv::", "")})
    try:
        d[r[mi]] = float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0)
    except ValueError:  # "n/a" (a metric this chip does not expose)
        pass
tot = sum(d.get("gpu__time_duration.sum", 0.0) for d in launch.values())
print(f"{len(launch)} launches, {tot:.1f} us of device time (cold-cache, serialised)")
print(f"{'#':>3} {'kernel':<34} {'us':>9} {'share':>6} {'DRAM rd MB':>11} {'DRAM wr MB':>11} {'tensor %':>9}")
per = defaultdict(lambda: [0.0, 0.0, 0.0, 0])
for n, d in launch.items():
    t = d.get("gpu__time_duration.sum", 0.0)
    print(f"{n:>3} {d['name'][:34]:<34} {t:9.1f} {100 * t / tot:5.1f}% {d.get('dram__bytes_read.sum', 0):11.1f} "
          f"{d.get('dram__bytes_write.sum', 0):11.1f} {d.get('sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed', 0):9.1f}")
    p = per[d["name"]]
    p[0] += t
    p[1] += d.get("dram__bytes_read.sum", 0)
    p[2] += d.get("dram__bytes_write.sum", 0)
    p[3] += 1
print("\nper kernel:")
for name, (t, rd, wr, c) in sorted(per.items(), key=lambda kv: -kv[1][0]):
    print(f"  {name[:40]:<40} {t:9.1f} us {100 * t / tot:5.1f}%  launches {c}  DRAM {rd:.0f}/{wr:.0f} MB")
