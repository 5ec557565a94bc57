#!/usr/bin/env python
"""Write profiles/scan_traffic.json and profiles/coarse_tensor_pipe.json (read by bench.py for the
roofline's `traffic` and the coarse step's `tensor_pipe_pct_ncu`) from per-search ncu launch lists
(`scripts/gpu_ncu.sh`: gpu__time_duration, dram__bytes_read/write, sm__pipe_tc_cycles_active).
Usage: make_profile_tables.py SOURCE_TAG cN=launches_cN.csv ..."""
import csv
import io
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def launches(path):
    txt = open(path).read()
    rows = list(csv.reader(io.StringIO(txt[txt.find('"ID"'):])))
    h = rows[0]
    ki, mi, ui, vi, idi = (h.index(c) for c in ("Kernel Name", "Metric Name", "Metric Unit", "Metric Value", "ID"))
    out = {}
    scale = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "nsecond": 1e-3, "us": 1.0,
             "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "%": 1.0}
    for r in rows[1:]:
        d = out.setdefault(int(r[idi]), {"name": r[ki]})
        try:
            d[r[mi]] = float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0)
        except ValueError:
            pass
    return [out[i] for i in sorted(out)]


def main():
    tag = sys.argv[1]
    traffic, tpipe = {}, {}
    for arg in sys.argv[2:]:
        c, path = arg.split("=")
        wl = bench.CONFIGS[c]["workload"] + ("_shard0of8" if bench.CONFIGS[c].get("sharded_build") else "")
        L = launches(path)
        scans = [d for d in L if "k_scan_tc" in d["name"]]
        coarse = [d for d in L if "k_coarse" in d["name"]]
        if scans:
            traffic[wl] = {
                "kernel": "k_scan_tc, phase A + phase B launches of one search",
                "traffic_bytes_per_launch": sum(d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
                                                for d in scans),
                "per_launch_MB": [{"read": d.get("dram__bytes_read.sum", 0) / 1e6,
                                   "write": d.get("dram__bytes_write.sum", 0) / 1e6,
                                   "us": d.get("gpu__time_duration.sum", 0)} for d in scans],
                "source": f"ncu launch list ({tag}), cold-cache serialised launches",
                "note": "dram__bytes_read.sum + dram__bytes_write.sum summed over the two scan launches of one search"}
        if coarse:
            t = sum(d.get("gpu__time_duration.sum", 0) for d in coarse)
            pct = sum(d.get("gpu__time_duration.sum", 0) * d.get("sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed", 0)
                      for d in coarse) / max(t, 1e-9)
            tpipe[wl] = {"kernel": "k_coarse_qm (tcgen05 kind::tf32), both passes", "tensor_pipe_pct": pct,
                         "per_launch_pct": [d.get("sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed", 0)
                                            for d in coarse],
                         "source": f"ncu launch list ({tag}): sm__pipe_tc_cycles_active, duration-weighted"}
    json.dump(traffic, open(os.path.join(ROOT, "profiles", "scan_traffic.json"), "w"), indent=1)
    json.dump(tpipe, open(os.path.join(ROOT, "profiles", "coarse_tensor_pipe.json"), "w"), indent=1)
    print(json.dumps({"traffic": {k: v["traffic_bytes_per_launch"] for k, v in traffic.items()},
                      "tensor_pipe": {k: v["tensor_pipe_pct"] for k, v in tpipe.items()}}, indent=1))


if __name__ == "__main__":
    main()
