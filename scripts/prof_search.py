#!/usr/bin/env python
"""One search of a bench config between cudaProfilerStart/Stop, for ncu captures:

  ncu --profile-from-start off --set full --clock-control none --import-source on \
      -o gpurun_out/c4 python scripts/prof_search.py --config c4

Builds the index exactly as bench.py does (untimed), runs `--warmup` searches, then profiles
`--searches` searches.  For c5 it builds shard 0 of 8 (the per-GPU workload of the 8-GPU job).
"""
import argparse
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c4")
    ap.add_argument("--nprobe", type=int, default=0)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--searches", type=int, default=1)
    ap.add_argument("--opt", action="append", default=[], help="name=value (mv_index_set_option)")
    a = ap.parse_args()
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index
    cfg = dict(bench.CONFIGS[a.config])
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(0)
    bs = None
    if cfg.get("sharded_build"):
        ix, Q, C, _, n = bench.build_sharded(cfg, dev, 0, 8, Index, ngt=0)
    else:
        X, Q, C, bs = bench.make_data(cfg, dev)
        n = cfg["n"]
        ix = Index(cfg["d"], cfg["metric"], cfg["kind"], cfg["nlist"], device=0)
        ix.set_centroids(C)
        if cfg["kind"] == "sq8":
            ix.set_sq8(*bench.sq8_params(cfg, X))
        if cfg["kind"] == "pq":
            samp = torch.randperm(n, generator=torch.Generator().manual_seed(5))[: min(n, 64 * cfg["nlist"])]
            ix.train_pq(cfg["pq_m"], X[samp.to(dev)].contiguous(), niter=10)
        ix.add(X, torch.arange(n, dtype=torch.int64, device=dev))
        del X
    for o in a.opt:
        k, v = o.split("=")
        ix.set_option(k, int(v))
    nprobe = a.nprobe or cfg["nprobe"]
    nbits = n if bs is not None else 0
    for _ in range(a.warmup):
        ix.search(Q, cfg["k"], nprobe, bitset=bs, nbits=nbits)
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    for _ in range(a.searches):
        ix.search(Q, cfg["k"], nprobe, bitset=bs, nbits=nbits)
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    print(ix.describe())


if __name__ == "__main__":
    main()
