"""Oracle for IVF_PQ.  TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

PAPER.md:519-521 (§3.1): "IVF_PQ uses product quantization that splits each vector into multiple
sub-vectors and applies k-means for each sub-space".  Reading R19: M sub-spaces of
dsub = d / M consecutive dimensions, 256 sub-centroids each (one byte per sub-code), PQ of the
vectors themselves (not of residuals); a code is, per sub-space, the closest sub-centroid (fp64
squared L2, ties to the smaller index); the fine quantizer keeps the decoded vector x_hat = the
concatenation of the chosen sub-centroids, so the IVF search's step (2) computes the distance from
q to x_hat (the asymmetric distance of PQ) -- in fp64, by definition, here.
"""
from __future__ import annotations

import numpy as np

from .ivf import IvfIndex


def pq_encode(X, codebooks) -> np.ndarray:
    """codes[n, M] uint8: per sub-space the closest of the 256 sub-centroids.  codebooks:
    [M, 256, dsub] float32."""
    X = np.asarray(X, dtype=np.float64)
    cb = np.asarray(codebooks, dtype=np.float64)
    M, K, dsub = cb.shape
    out = np.empty((X.shape[0], M), dtype=np.uint8)
    for m in range(M):
        sub = X[:, m * dsub:(m + 1) * dsub]
        for i in range(X.shape[0]):
            d = ((cb[m] - sub[i][None, :]) ** 2).sum(axis=1)
            out[i, m] = int(np.argmin(d))  # first minimum: the smaller index on ties
    return out


def pq_decode(codes, codebooks) -> np.ndarray:
    """x_hat[n, M * dsub] float32: the concatenation of the chosen sub-centroids."""
    cb = np.asarray(codebooks, dtype=np.float32)
    codes = np.asarray(codes)
    return np.concatenate([cb[m][codes[:, m]] for m in range(cb.shape[0])], axis=1).astype(np.float32)


class IvfPqIndex(IvfIndex):
    """IvfIndex whose fine quantizer is PQ: stored vectors are the decoded PQ codes."""

    def __init__(self, d: int, metric: int, centroids, codebooks):
        super().__init__(d, metric, 0, centroids)
        self.codebooks = np.asarray(codebooks, dtype=np.float32)
        assert self.codebooks.shape[0] * self.codebooks.shape[2] == d

    def stored_vectors(self, order) -> np.ndarray:
        # the encoding is per row: computed once per row set (memoised; the arithmetic is unchanged)
        key = (self.ntotal, tuple(np.asarray(order)[:8].tolist()))
        if getattr(self, "_memo", (None,))[0] != key:
            self._memo = (key, pq_decode(pq_encode(self._vecs[order], self.codebooks), self.codebooks))
        return self._memo[1]

    def codes(self, order) -> np.ndarray:
        return pq_encode(self._vecs[order], self.codebooks)
