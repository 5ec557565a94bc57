"""Seeded Lloyd k-means -- DATA PREPARATION ONLY.

The north star consumes "supplied centroids" (BASELINE.json; §3.1 builds
the coarse codebook with K-means, K=16384).  Which k-means produced them does not matter to
parity: the oracle and the CUDA path both receive the same centroid array as an input.  This
runs in plain torch (CPU or GPU), outside every timed region, and is used by neither the
oracle's arithmetic nor the CUDA path.

Recipe: n_train = min(n, 64*nlist) rows chosen by a seeded hash order;
init = the first nlist of them; `iters` Lloyd iterations; an empty cluster is re-seeded with
the training point farthest from its centroid; `spherical` re-normalises centroids (Deep).
"""
from __future__ import annotations

import torch

from . import SEED_KMEANS, hash64


def _nearest(x: torch.Tensor, c: torch.Tensor, chunk: int = 1 << 16):
    cn = (c * c).sum(1)
    idx = torch.empty(x.shape[0], dtype=torch.int64, device=x.device)
    dmin = torch.empty(x.shape[0], dtype=torch.float32, device=x.device)
    for s in range(0, x.shape[0], chunk):
        xb = x[s:s + chunk]
        sc = cn[None, :] - 2.0 * (xb @ c.T)
        v, i = sc.min(dim=1)
        idx[s:s + chunk] = i
        dmin[s:s + chunk] = v + (xb * xb).sum(1)
    return idx, dmin


def kmeans(x: torch.Tensor, nlist: int, iters: int = 20, seed: int = SEED_KMEANS, spherical: bool = False,
           n_train: int | None = None) -> torch.Tensor:
    n, d = x.shape
    n_train = min(n, 64 * nlist) if n_train is None else min(n, n_train)
    if n_train < nlist:
        raise ValueError("k-means needs at least nlist training rows")
    order = torch.argsort(hash64(seed, 1, torch.arange(n, dtype=torch.int64, device=x.device)))
    xt = x[order[:n_train]].float().contiguous()
    c = xt[:nlist].clone()
    prev = torch.backends.cuda.matmul.allow_tf32
    torch.backends.cuda.matmul.allow_tf32 = False
    try:
        for _ in range(iters):
            a, dmin = _nearest(xt, c)
            sums = torch.zeros_like(c).index_add_(0, a, xt)
            cnt = torch.bincount(a, minlength=nlist).to(torch.float32)
            nz = cnt > 0
            c[nz] = sums[nz] / cnt[nz, None]
            empty = torch.nonzero(~nz).flatten()
            if empty.numel():
                far = torch.argsort(dmin, descending=True)[: empty.numel()]
                c[empty] = xt[far]
            if spherical:
                c = c / c.norm(dim=1, keepdim=True).clamp_min(1e-12)
    finally:
        torch.backends.cuda.matmul.allow_tf32 = prev
    return c.contiguous()
