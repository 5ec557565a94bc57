"""Per-search kernel time shares from an `ncu --metrics gpu__time_duration.sum --csv` launch list.
Counts the libmv kernels (mv:: namespace) launched per search (k_plan to k_plan) and their mean
cold-cache, serialised durations.  Usage: launch_summary.py launches.csv"""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 14 and r[12] == "gpu__time_duration.sum"]
tot = defaultdict(float)
cnt = defaultdict(int)
# one search = the launches from one k_plan to the next (its scan and selects, then the next
# search's query staging and coarse step); the add path and data preparation precede the first
# k_plan, the tail after the last one is dropped
plans = [i for i, r in enumerate(rows) if "k_plan" in r[4]]
nplan = max(len(plans) - 1, 0)
for r in rows[plans[0]:plans[-1]] if nplan else []:
    name = r[4]
    short = name.split("(")[0].replace("void ", "").replace("mv::", "")
    if not any(t in name for t in ("mv::", "k_scan", "k_final", "k_coarse", "k_probe", "k_plan", "k_hilo",
                                    "k_query_prep", "k_qplanes", "k_final_big", "k_merge")):
        continue
    v = float(r[14].replace(",", ""))
    unit = r[13]
    us = {"nsecond": v / 1000.0, "ns": v / 1000.0, "usecond": v, "us": v, "msecond": v * 1000.0, "ms": v * 1000.0}.get(unit, v)
    tot[short] += us
    cnt[short] += 1
n = max(nplan, 1)
total = sum(tot.values()) / n
print(f"searches (k_plan to k_plan): {nplan}; libmv device time per search {total:.1f} us")
for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
    print(f"  {k:<40} {v / n:9.1f} us  {100 * v / n / total:5.1f}%  launches/search {cnt[k] / n:.2f}")
