#!/usr/bin/env python
"""SURVEY §8(f) f2 ablation: Milvus reaches k > 1024 by ceil(k / 1024) rounds, each a full search
for the next 1024 results (§3.3).  A round costs at least one k = 1024 search of
the same batch (it re-runs the coarse step, the scan and a 1024-select; the filter of d < d_l only
adds work), so ceil(k/1024) x t(k = 1024) is a lower bound of the rounds procedure on this
hardware.  This times that bound against the single pass (one scan + one select of the exact
top-k) on configs[3] (SIFT10M IVF_FLAT, nprobe 128, 10k queries) for k = 2048 (the
config's k), 4096 and 16384.  Prints one JSON line."""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def timed(ix, Q, k, nprobe, steps=5):
    for _ in range(2):
        ix.search(Q, k, nprobe)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        ix.search(Q, k, nprobe)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / steps


def main():
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index
    cfg = dict(bench.CONFIGS["c4"])
    dev = torch.device("cuda", 0)
    X, Q, C, _ = bench.make_data(cfg, dev)
    ix = Index(cfg["d"], cfg["metric"], cfg["kind"], cfg["nlist"], device=0)
    ix.set_centroids(C)
    ix.add(X, torch.arange(cfg["n"], dtype=torch.int64, device=dev))
    del X
    nprobe = cfg["nprobe"]
    t1024 = timed(ix, Q, 1024, nprobe)
    rows = []
    for k in (2048, 4096, 16384):
        t = timed(ix, Q, k, nprobe)
        rounds = (k + 1023) // 1024
        rows.append({"k": k, "single_pass_ms": t, "rounds": rounds, "rounds_lower_bound_ms": rounds * t1024,
                     "speedup_vs_rounds_bound": rounds * t1024 / t})
    print(json.dumps({"workload": "sift10m_ivfflat_l2_nlist16384_nprobe128 (configs[3]), nq 10000",
                      "t_k1024_ms": t1024, "rows": rows,
                      "note": "rounds bound = ceil(k/1024) x one k=1024 search (PAPER.md:745-761)"}))


if __name__ == "__main__":
    main()
