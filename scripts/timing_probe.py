#!/usr/bin/env python
"""Per-search device time vs host enqueue time under the binding's options (allocator, profiling,
index type) on configs[1]-sized data: finds host-side stalls between back-to-back searches."""
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index  # noqa: E402

cfg = dict(bench.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "c2"])
dev = torch.device("cuda", 0)
X, Q, C, bs = bench.make_data(cfg, dev)
ids = torch.arange(cfg["n"], dtype=torch.int64, device=dev)
for kind in ("flat", "sq8"):
    for alloc in ("torch", None):
        ix = Index(cfg["d"], cfg["metric"], kind, cfg["nlist"], device=0, allocator=alloc)
        ix.set_centroids(C)
        if kind == "sq8":
            ix.set_sq8(*bench.sq8_params(cfg, X))
        ix.add(X, ids)
        for prof in (False, True):
            for ws in (0, 8 << 30):
                ix.profile(prof)
                ix.set_option("workspace_bytes", ws)
                for _ in range(3):
                    ix.search(Q, cfg["k"], cfg["nprobe"])
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                t0 = time.perf_counter()
                e0.record()
                for _ in range(10):
                    ix.search(Q, cfg["k"], cfg["nprobe"])
                th = (time.perf_counter() - t0) / 10 * 1e3
                e1.record()
                torch.cuda.synchronize()
                print(f"{kind} alloc={alloc} prof={prof} ws={ws}: gpu {e0.elapsed_time(e1) / 10:.3f} ms/search, "
                      f"host enqueue {th:.3f} ms/search", flush=True)
                ix.profile(False)
                ix.profile_read(reset=True)
        ix.close()
