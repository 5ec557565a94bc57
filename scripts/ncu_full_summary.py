#!/usr/bin/env python
"""Key metrics of one `ncu --set full` capture exported with `ncu -i X.ncu-rep --page raw --csv`:
time, DRAM bytes, L2 hit rates, tensor pipe, issue and occupancy, the top stall reasons.
Usage: ncu_full_summary.py raw.csv [label]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h, units = rows[0], rows[1]
label = sys.argv[2] if len(sys.argv) > 2 else sys.argv[1]
KEYS = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_op_read_hit_rate.pct",
        "lts__t_sector_op_write_hit_rate.pct", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__inst_executed.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size"]
for v in rows[2:]:
    d, u = dict(zip(h, v)), dict(zip(h, units))
    print(f"== {label}: {d.get('Kernel Name', '?')[:80]}")
    for k in KEYS[1:]:
        if k in d and d[k] != "":
            print(f"  {k:<66} {d[k]:>18} {u.get(k, '')}")
    st = []
    for k in h:
        if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("_per_issue_active.ratio"):
            try:
                st.append((float(d[k].replace(",", "")), k[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
            except ValueError:
                pass
    print("  top stalls (warps per issue): " + ", ".join(f"{n} {x:.2f}" for x, n in sorted(st, reverse=True)[:6]))
