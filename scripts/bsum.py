#!/usr/bin/env python
"""One line per bench JSON file: workload, qps, ms, e2e, scan roofline fraction, recall, stages."""
import json
import sys

for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:  # noqa: BLE001
        print(f, "unreadable:", e)
        continue
    if "value" not in d:
        print(f, d)
        continue
    st = " ".join(f"{k} {v:.3f}" for k, v in (d.get("stage_ms") or {}).items())
    print(f"{f}: {d['config']['workload']} {d['value'] / 1e6:.3f}M qps {d['ms_per_step']:.3f} ms e2e "
          f"{(d.get('e2e') or {}).get('value', 0) / 1e6:.3f}M frac {d['roofline']['frac']:.3f} "
          f"recall {d['config'].get('recall@10')} | {st}")
