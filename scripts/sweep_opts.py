#!/usr/bin/env python
"""Time one bench config under several mv_index_set_option settings (one index build):

  python scripts/sweep_opts.py --config c4 --sets "need=16384" "need=32768,capa=512"

Each setting: 3 warm-up searches, then `--steps` timed with CUDA events; prints ms/search, qps and
the per-stage breakdown.  Options never change results (tests/test_gpu_parity.py), only speed."""
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
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--nprobe", type=int, default=0)
    ap.add_argument("--sets", nargs="+", default=[""])
    a = ap.parse_args()
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index
    cfg = dict(bench.CONFIGS[a.config])
    dev = torch.device("cuda", 0)
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
    nprobe = a.nprobe or cfg["nprobe"]
    nbits = n if bs is not None else 0
    names = ["seeding", "need", "capa", "sq8_qc", "flat_qc", "coarse_nqb", "coarse_cs", "coarse_epi", "coarse_nacc",
             "large_k_select", "big_ctas", "big_cap"]
    for st in a.sets:
        for nm in names:
            ix.set_option(nm, 1 if nm == "seeding" else 0)
        for kv in filter(None, st.split(",")):
            k, v = kv.split("=")
            ix.set_option(k, int(v))
        for _ in range(3):
            ix.search(Q, cfg["k"], nprobe, bitset=bs, nbits=nbits)
        torch.cuda.synchronize()
        ix.profile_read(reset=True)
        ix.profile(True)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(a.steps):
            ix.search(Q, cfg["k"], nprobe, bitset=bs, nbits=nbits)
        e1.record()
        torch.cuda.synchronize()
        ix.profile(False)
        stg, ns, _ = ix.profile_read(reset=True)
        cnt = ix.profile_counters(reset=True)
        qn = max(cnt["queries"], 1)
        ms = e0.elapsed_time(e1) / a.steps
        print(f"{a.config} [{st or 'default'}] {ms:.3f} ms/search {cfg['nq'] / ms * 1e3 / 1e6:.3f} Mqps | "
              + " ".join(f"{k} {v / max(ns, 1):.3f}" for k, v in stg.items())
              + f" | emitted/query A {cnt['phase_a_emitted'] / qn:.0f} B {cnt['phase_b_emitted'] / qn:.0f}", flush=True)


if __name__ == "__main__":
    main()
