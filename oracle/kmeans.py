"""Oracle for SURVEY §8(f) row f1's k-means training of the coarse codebook.  TEST INFRASTRUCTURE
ONLY (see oracle/__init__.py).

PAPER.md:503-514 (§3.1): IVF clusters the vectors into buckets with K-means; the centroids are the
coarse codebook.  One Lloyd iteration, literally: every row goes to its closest centroid
(oracle.assign, fp64, ties to the smaller centroid id), then every centroid becomes the mean of
its rows in fp64, rounded to fp32 once; a centroid without rows keeps its position (reading R18,
DESIGN.md §2); `spherical` normalises the fp64 mean before the rounding (unit-norm data).
"""
from __future__ import annotations

import numpy as np

from .ivf import assign


def lloyd_step(X, C, metric: int, spherical: bool = False, lists=None):
    """One Lloyd iteration from centroids C [nlist, d] over rows X [n, d].  `lists`: the assignment
    to use instead of oracle.assign (the conditional-oracle protocol).  Returns (C' fp32, lists)."""
    X = np.asarray(X, dtype=np.float32)
    C = np.asarray(C, dtype=np.float32)
    a = assign(X, C, metric) if lists is None else np.asarray(lists, dtype=np.int64)
    out = C.astype(np.float64).copy()
    for l in range(C.shape[0]):
        rows = X[a == l].astype(np.float64)
        if len(rows) == 0:
            continue
        m = rows.sum(axis=0) / len(rows)
        if spherical:
            nn = np.sqrt((m * m).sum())
            if nn > 0:
                m = m / nn
        out[l] = m
    return out.astype(np.float32), a


def kmeans(X, C0, metric: int, niter: int, spherical: bool = False):
    """niter Lloyd iterations from C0."""
    C = np.asarray(C0, dtype=np.float32)
    for _ in range(niter):
        C, _ = lloyd_step(X, C, metric, spherical)
    return C


def sse(X, C, lists) -> float:
    """Within-cluster sum of squared distances (fp64)."""
    X = np.asarray(X, dtype=np.float64)
    d = X - np.asarray(C, dtype=np.float64)[np.asarray(lists)]
    return float((d * d).sum())
