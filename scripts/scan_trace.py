#!/usr/bin/env python
"""Phase-B timeline of scan CTA 0 (development build with -DMV_SCAN_TRACE, see k_scan_tc.cu):

  python scripts/scan_trace.py --config c5 [--lib exp/libT.so]

Rows of clock64 stamps (per stage `it`, tile `t` or item `w` of CTA 0):
  0 producer issued stage it      7 MMA saw stage it full      2 MMA tile t start (accumulator free)
  3 MMA tile t committed           6 epilogue tile t start       4 epilogue tile t done
  1 MMA item w start (queries in)  5 gatherer published item w
"""
import argparse
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def stats(name, v):
    v = np.asarray(v, dtype=np.float64)
    v = v[np.isfinite(v)]
    if v.size == 0:
        print(f"{name:42s} -")
        return
    print(f"{name:42s} n={v.size:5d} median {np.median(v):8.0f}  mean {v.mean():8.0f}  p90 {np.percentile(v, 90):8.0f}")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c5")
    ap.add_argument("--raw", type=int, default=40)
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
    nbits = n if bs is not None else 0
    for _ in range(3):
        ix.search(Q, cfg["k"], cfg["nprobe"], bitset=bs, nbits=nbits)
    buf = torch.zeros(9 * 1024, dtype=torch.int64, device=dev)
    ix.set_option("scan_trace", buf.data_ptr())
    ix.search(Q, cfg["k"], cfg["nprobe"], bitset=bs, nbits=nbits)
    torch.cuda.synchronize()
    ix.set_option("scan_trace", 0)
    t = buf.cpu().numpy().reshape(9, 1024).astype(np.float64)
    t[t == 0] = np.nan
    base = np.nanmin(t[:8])
    r = t[:8] - base
    print(ix.describe().get("last_scan"), "phase B, CTA 0; cycles")
    n0 = int(np.sum(np.isfinite(r[0])))
    nt = int(np.sum(np.isfinite(r[2])))
    print(f"stages {n0}, tiles {nt}, items {int(np.sum(np.isfinite(r[1])))}")
    stats("producer inter-issue (stage)", np.diff(r[0]))
    stats("stage issue -> MMA sees it full", r[7] - r[0])
    stats("MMA tile period", np.diff(r[2]))
    stats("MMA waits accumulator (t start - t-1 commit)", r[2][1:] - r[3][:-1])
    stats("MMA tile issue time (commit - start)", r[3] - r[2])
    stats("commit -> epilogue start", r[6] - r[3])
    stats("epilogue tile duration", r[4] - r[6])
    stats("epilogue gap (t start - t-1 done)", r[6][1:] - r[4][:-1])
    stats("item: MMA start - gather published", r[1] - r[5])
    stats("gather inter-publish", np.diff(r[5]))
    g = t[8][: 148 * 3].reshape(148, 3)
    dur = (g[:, 1] - g[:, 0]) / 1e3
    print(f"CTA durations (us): min {np.nanmin(dur):.1f} median {np.nanmedian(dur):.1f} max {np.nanmax(dur):.1f}; "
          f"tiles/CTA median {np.nanmedian(g[:, 2]):.0f}")
    print("raw (first tiles): t, start, commit, epi start, epi done")
    for i in range(min(a.raw, nt)):
        print(f"  {i:4d} {r[2][i]:10.0f} {r[3][i]:10.0f} {r[6][i]:10.0f} {r[4][i]:10.0f}")


if __name__ == "__main__":
    main()
