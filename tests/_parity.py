"""Parity helpers (test infrastructure): compare the CUDA path's top-k with the oracle's.

Rule (BASELINE.json north star): returned ids equal the oracle's except where oracle distances
tie within the tolerance; distances within the stated tolerance.  A GPU id at a mismatching
position must be a genuine candidate whose oracle distance ties with the oracle's distance at
that position.  Tolerance per element: |d_gpu - d_oracle| <= rtol * |d_oracle| + atol, where atol
covers cancellation of the ||q||^2 - 2 q.x + ||x||^2 expansion.
"""
from __future__ import annotations

import numpy as np

import oracle as O


def candidate_map(idx: O.IvfIndex, q, probes_row, bitset=None, nbits=0):
    """{id: oracle float64 distance} over the probed lists' non-excluded members (duplicate ids:
    the best distance)."""
    off, order = idx.storage()
    V = idx.stored_vectors(order)
    ids = idx._ids[order]
    rows = np.concatenate([np.arange(off[l], off[l + 1]) for l in probes_row] + [np.zeros(0, np.int64)])
    rows = rows[~O.bit_is_set(bitset, nbits, ids[rows])]
    D = O.distances(q, V[rows], idx.metric)
    m = {}
    for i, dd in zip(ids[rows].tolist(), D.tolist()):
        if i not in m or (dd < m[i] if idx.metric == O.L2 else dd > m[i]):
            m[i] = dd
    return m


def check_topk(Dg, Ig, Do, Io, cmaps=None, rtol=1e-5, atol=0.0, exact=False):
    """Returns the fraction of positions whose ids match exactly (1.0 expected up to ties)."""
    Dg = np.asarray(Dg, dtype=np.float64)
    Ig = np.asarray(Ig)
    Do = np.asarray(Do, dtype=np.float64)
    Io = np.asarray(Io)
    assert Dg.shape == Do.shape and Ig.shape == Io.shape
    pad_o = Io == -1
    assert np.array_equal(Ig == -1, pad_o), "padding positions differ"
    if exact:
        assert np.array_equal(Ig, Io), "ids differ"
        assert np.array_equal(Dg[~pad_o].astype(np.float32), Do[~pad_o].astype(np.float32)), "distances differ"
        return 1.0
    live = ~pad_o
    tol = rtol * np.abs(Do) + atol
    bad = live & ~(np.abs(Dg - Do) <= tol)
    assert not bad.any(), f"{bad.sum()} distances out of tolerance, e.g. gpu={Dg[bad][:5]} oracle={Do[bad][:5]}"
    for i in range(Ig.shape[0]):
        row = Ig[i][Ig[i] >= 0]
        assert len(set(row.tolist())) == len(row), f"duplicate ids in row {i}"
    mism = live & (Ig != Io)
    if mism.any():
        assert cmaps is not None, f"{mism.sum()} id mismatches and no candidate map to adjudicate ties"
        for i, j in zip(*np.nonzero(mism)):
            m = cmaps[i]
            gid = int(Ig[i, j])
            assert gid in m, f"query {i}: GPU id {gid} is not a candidate"
            assert abs(m[gid] - Do[i, j]) <= tol[i, j] * 2 + 1e-300, \
                f"query {i} pos {j}: GPU id {gid} (oracle d={m[gid]}) does not tie with oracle d={Do[i, j]}"
    return 1.0 - mism.sum() / max(live.sum(), 1)


def oracle_from_gpu_storage(ix, metric, kind, centroids, X, ids, sq8=None):
    """Conditional-oracle protocol step 1: an oracle index holding the GPU's accepted assignment.
    Returns (oracle index, gpu list of every input row)."""
    off, sids, _ = ix.storage()
    lists_of_storage = np.repeat(np.arange(len(off) - 1), np.diff(off))
    # map storage rows back to input rows: ids are unique in these tests
    pos = {int(v): r for r, v in enumerate(np.asarray(ids).tolist())}
    inv = np.array([pos[int(v)] for v in sids.tolist()], dtype=np.int64)
    gl = np.empty(len(ids), dtype=np.int64)
    gl[inv] = lists_of_storage
    oi = O.IvfIndex(X.shape[1], metric, kind, centroids)
    if sq8 is not None:
        oi.set_sq8(*sq8)
    oi.add(X, ids, lists=gl)
    return oi, gl


def check_assignment(gl, X, C, metric, sample=None, rtol=1e-5, seed=0):
    """Assignment parity: GPU list == oracle list, or the two centroid distances tie within rtol."""
    n = len(gl)
    rows = np.arange(n) if sample is None or sample >= n else np.random.default_rng(seed).choice(n, sample, replace=False)
    ol = O.assign(X[rows], C, metric)
    diff = np.nonzero(ol != gl[rows])[0]
    for r in diff:
        x = X[rows[r]]
        s = O.distances(x, C[[ol[r], gl[rows[r]]]], metric)
        assert abs(s[0] - s[1]) <= rtol * max(abs(s[0]), 1e-30), f"row {rows[r]}: oracle {ol[r]} vs gpu {gl[rows[r]]}: {s}"
    return len(diff)


def check_probes(Pg, Q, C, nprobe, metric, rtol=1e-5):
    """Probe-set parity modulo centroids tied (within rtol) with the nprobe-th."""
    Po = O.probe(Q, C, nprobe, metric)
    nd = 0
    for i in range(len(Q)):
        a, b = set(Pg[i].tolist()), set(Po[i].tolist())
        if a == b:
            continue
        nd += 1
        s = O.distances(Q[i], C, metric)
        kth = s[Po[i][-1]]
        for c in a ^ b:
            assert abs(s[c] - kth) <= rtol * max(abs(kth), 1e-30), f"query {i}: probe {c} not tied with the boundary"
    return nd


def sampled_oracle_topk(Qs, Ps, off, sids, rows_of, metric, kind, k, sq8=None, bitset=None, nbits=0):
    """Oracle step O5 for a sample of queries at sizes where building the whole oracle index is
    impractical (configs[2..4] full size): for each query, its candidates are the members of the
    (GPU-accepted, separately checked) probed lists, minus the excluded ids; distances to the
    stored (FLAT) or decoded (SQ8, the oracle codec) vectors in fp64; the exact top-k by the total
    order.  These are exactly the steps of oracle.IvfIndex.search, restricted to the probed lists.
    rows_of(ids) -> the raw fp32 vectors of those ids (regenerated or indexed by the caller).
    Returns (D, I, candidate maps)."""
    m = len(Qs)
    outD = np.empty((m, k))
    outI = np.empty((m, k), dtype=np.int64)
    cmaps = []
    for i in range(m):
        rows = np.concatenate([np.arange(off[l], off[l + 1]) for l in Ps[i]] + [np.zeros(0, np.int64)])
        cid = sids[rows]
        keep = ~O.bit_is_set(bitset, nbits, cid)
        rows, cid = rows[keep], cid[keep]
        V = np.asarray(rows_of(cid), dtype=np.float32)
        if kind == O.SQ8:
            V = O.sq8_decode(O.sq8_encode(V, *sq8), *sq8)
        D = O.distances(Qs[i], V, metric)
        outD[i], outI[i], _ = O.select_topk(D, cid, rows, k, metric)
        cmaps.append(dict(zip(cid.tolist(), D.tolist())))
    return outD, outI, cmaps


def gpu_lists_of(ids_sample, off, pos_of):
    """The GPU's list of each sampled id: its storage position -> the list whose range holds it."""
    pos = pos_of(ids_sample)
    return np.searchsorted(off, pos, side="right") - 1
