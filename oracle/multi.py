"""Oracle for the two workloads SURVEY §8(f) row f4 puts on top of the hot path.  TEST
INFRASTRUCTURE ONLY (see oracle/__init__.py).

* Strategy E, partition-based attribute filtering (§4.1): the dataset is split
  into partitions by the value ranges of one attribute; a query with the constraint
  lo <= attr <= hi searches only the partitions whose range overlaps [lo, hi]; a partition whose
  range is covered by [lo, hi] is searched without checking the attribute; in the others the
  attribute is checked with strategy B's bitmap -- reading R16:
  strategy D's cost model is not modelled, a partly covered partition always takes strategy B.
  The partitions' top-k lists are merged (merge_topk).
* Multi-vector queries (§4.2): an entity has mu vectors v_0..v_{mu-1}; the
  similarity of a query entity q and an entity e is g(f(q.v_0, e.v_0), ..., f(q.v_{mu-1}, e.v_{mu-1}))
  with f = inner product and g = the weighted sum sum_i w_i f_i.  The oracle
  computes that definition directly -- per entity, per vector, in float64 -- not the vector
  fusion the GPU path uses (one IP search over concatenated, weighted vectors), so the fusion
  identity is what the parity tests check.
"""
from __future__ import annotations

import numpy as np

from .ivf import IP, PAD_ID, merge_topk, pad_value, select_topk


# ----------------------------------------------------------------------------------------
# Strategy E (§4.1)
# ----------------------------------------------------------------------------------------
def range_bitset(ids, attr, lo: int, hi: int, nbits: int) -> np.ndarray:
    """Strategy B's bitmap for the constraint lo <= attr <= hi, in the hot path's polarity
    (bit = 1 means excluded, indexed by id, LSB-first; reading R6): the ids whose attribute is
    outside [lo, hi]."""
    ids = np.asarray(ids, dtype=np.int64)
    attr = np.asarray(attr, dtype=np.int64)
    bits = np.zeros(nbits, dtype=np.uint8)
    out = ids[(attr < lo) | (attr > hi)]
    bits[out] = 1
    return np.packbits(bits, bitorder="little")


def partition_plan(ranges, lo: int, hi: int):
    """Per partition p with attribute range [plo, phi]: 'skip' when it does not overlap [lo, hi],
    'covered' when lo <= plo and phi <= hi (no attribute check), else 'check'."""
    plan = []
    for plo, phi in ranges:
        if phi < lo or plo > hi:
            plan.append("skip")
        elif lo <= plo and phi <= hi:
            plan.append("covered")
        else:
            plan.append("check")
    return plan


def partition_search(parts, Q, k: int, nprobe: int, lo: int, hi: int, probes=None):
    """Strategy E over `parts` = [(IvfIndex, (plo, phi), ids, attr), ...]: each partition's own
    IVF search -- without a bitset when covered, with range_bitset when partly covered, not at
    all when outside -- and the merge of the partitions' top-k.  `probes`: the buckets of step 1
    when given (the conditional-oracle protocol; partitions share the centroids).  Returns
    (D[m,k], I[m,k])."""
    Q = np.asarray(Q, dtype=np.float32)
    m = Q.shape[0]
    plan = partition_plan([r for _, r, _, _ in parts], lo, hi)
    metric = parts[0][0].metric
    res = []
    for (ix, _, ids, attr), how in zip(parts, plan):
        if how == "skip":
            continue
        if how == "covered":
            D, I, _ = ix.search(Q, k, nprobe, probes=probes)
        else:
            nbits = int(np.max(ids)) + 1 if len(ids) else 0
            D, I, _ = ix.search(Q, k, nprobe, bitset=range_bitset(ids, attr, lo, hi, nbits), nbits=nbits,
                                probes=probes)
        res.append((D, I))
    if not res:
        return np.full((m, k), pad_value(metric)), np.full((m, k), PAD_ID, dtype=np.int64)
    return merge_topk(res, k, metric)


# ----------------------------------------------------------------------------------------
# multi-vector queries (§4.2)
# ----------------------------------------------------------------------------------------
def multivector_scores(Xs, q_parts, weights) -> np.ndarray:
    """g(e) = sum_i w_i (q.v_i . e.v_i) for every entity e (rows of Xs[i]), float64."""
    s = np.zeros(np.asarray(Xs[0]).shape[0], dtype=np.float64)
    for X, q, w in zip(Xs, q_parts, weights):
        s += float(w) * (np.asarray(X, dtype=np.float64) @ np.asarray(q, dtype=np.float64))
    return s


def multivector_topk(Xs, ids, Qs, weights, k: int):
    """Exact top-k entities by the weighted-sum aggregate of per-vector inner products (larger is
    better; ties by smaller id, then row).  Xs[i]: [n, d_i]; Qs[i]: [m, d_i].  Returns
    (D[m,k] float64, I[m,k] int64)."""
    ids = np.asarray(ids, dtype=np.int64)
    m = np.asarray(Qs[0]).shape[0]
    outD = np.empty((m, k))
    outI = np.empty((m, k), dtype=np.int64)
    rows = np.arange(len(ids))
    for j in range(m):
        s = multivector_scores(Xs, [np.asarray(Q)[j] for Q in Qs], weights)
        outD[j], outI[j], _ = select_topk(s, ids, rows, k, IP)
    return outD, outI
