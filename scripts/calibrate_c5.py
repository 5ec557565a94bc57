#!/usr/bin/env python
"""configs[4] data calibration: recall@10 of one shard (of 8) of the 1B SIFT-shaped SQ8 index vs the
shard's exact top-10 (first 1000 queries), as a function of nprobe, for a given micro-centre count.

  python scripts/calibrate_c5.py 24 22      # 2^24 and 2^22 micro centres
"""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index  # noqa: E402

cfg = dict(bench.CONFIGS["c5"])
dev = torch.device("cuda", 0)
for ml in [int(a) for a in sys.argv[1:]]:
    ix, Q, C, gt, n = bench.build_sharded(cfg, dev, 0, 8, Index, spec=bench.c5_spec(128, ml))
    out = []
    for nprobe in (64, 128, 256, 512, 1024):
        D, I = ix.search(Q[:1000], 10, nprobe)
        out.append((nprobe, bench.recall_at(gt[1], I, 10)))
    print(f"micro 2^{ml}: " + " ".join(f"np{a}={b:.4f}" for a, b in out), flush=True)
    del ix
    torch.cuda.empty_cache()
