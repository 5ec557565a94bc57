"""Pins for oracle/multi.py (``-m "not gpu"``): strategy E checked against the
paper's worked example, against brute force over the rows that satisfy the constraint, and
against strategy B on one index; the multi-vector aggregate checked against a pure-Python
brute force and against the vector-fusion identity of PAPER.md:1023-1034."""
import json
import math
import os

import numpy as np
from hypothesis import given, settings, strategies as st

import oracle as O

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _parts(X, ids, attr, ranges, C, metric=O.L2):
    parts = []
    for lo, hi in ranges:
        sel = (attr >= lo) & (attr <= hi)
        ix = O.IvfIndex(X.shape[1], metric, O.FLAT, C)
        ix.add(X[sel], ids[sel])
        parts.append((ix, (lo, hi), ids[sel], attr[sel]))
    return parts


def test_strategy_e_paper_example():
    g = json.load(open(os.path.join(GOLD, "strategy_e.json")))
    assert O.partition_plan([tuple(r) for r in g["ranges"]], *g["query_range"]) == g["plan"]
    # boundaries: touching ranges overlap, an exact cover is 'covered'
    assert O.partition_plan([(1, 100)], 100, 200) == ["check"]
    assert O.partition_plan([(1, 100)], 1, 100) == ["covered"]
    assert O.partition_plan([(1, 100)], 101, 200) == ["skip"]


def test_range_bitset_semantics():
    ids = np.array([0, 3, 9, 17, 8])
    attr = np.array([5, 50, 500, 49, 51])
    b = O.range_bitset(ids, attr, 40, 60, 18)
    # the bitset excludes exactly the out-of-range ids: 0 (attr 5) and 9 (attr 500)
    assert O.bit_is_set(b, 18, np.arange(18)).nonzero()[0].tolist() == [0, 9]


def _brute_filtered(X, ids, attr, Q, k, lo, hi, metric):
    """pure-Python brute force over the rows with lo <= attr <= hi"""
    outD, outI = [], []
    for q in Q.astype(np.float64):
        cand = []
        for x, i, a in zip(X.astype(np.float64), ids, attr):
            if lo <= a <= hi:
                d = math.fsum((qj - xj) ** 2 for qj, xj in zip(q, x)) if metric == O.L2 else math.fsum(q * x)
                cand.append((d if metric == O.L2 else -d, int(i), d))
        cand.sort()
        cand = cand[:k]
        outD.append([c[2] for c in cand] + [O.pad_value(metric)] * (k - len(cand)))
        outI.append([c[1] for c in cand] + [-1] * (k - len(cand)))
    return np.array(outD), np.array(outI)


@settings(max_examples=12, deadline=None)
@given(st.integers(0, 2**31 - 1), st.integers(0, 300), st.integers(0, 300), st.sampled_from([O.L2, O.IP]))
def test_strategy_e_exact_equals_filtered_brute_force(seed, a, b, metric):
    rng = np.random.default_rng(seed)
    n, d, m, k = 60, 5, 3, 7
    X = rng.integers(-4, 5, size=(n, d)).astype(np.float32)
    Q = rng.integers(-4, 5, size=(m, d)).astype(np.float32)
    ids = rng.permutation(1000)[:n]
    attr = rng.integers(1, 300, size=n)
    C = X[:4] + 0.5
    ranges = [(1, 100), (101, 200), (201, 299)]
    lo, hi = min(a, b), max(a, b)
    D, I = O.partition_search(_parts(X, ids, attr, ranges, C, metric), Q, k, 4, lo, hi)  # nprobe = nlist
    Db, Ib = _brute_filtered(X, ids, attr, Q, k, lo, hi, metric)
    assert np.array_equal(I, Ib)
    assert np.allclose(D, Db, rtol=0, atol=1e-9)


def test_strategy_e_equals_strategy_b_on_one_index():
    # shared centroids: every partition probes the same lists as the whole index, so strategy E
    # returns what strategy B (one index + the range bitmap) returns, at any nprobe
    rng = np.random.default_rng(5)
    n, d = 400, 8
    X = rng.normal(size=(n, d)).astype(np.float32)
    Q = rng.normal(size=(6, d)).astype(np.float32)
    ids = rng.permutation(n)
    attr = rng.integers(1, 500, size=n)
    C = X[rng.choice(n, 16, replace=False)]
    ranges = [(1, 100), (101, 200), (201, 300), (301, 400), (401, 500)]
    whole = O.IvfIndex(d, O.L2, O.FLAT, C)
    whole.add(X, ids)
    for lo, hi in [(50, 250), (1, 500), (120, 180), (401, 500), (600, 700)]:
        D, I = O.partition_search(_parts(X, ids, attr, ranges, C), Q, 10, 3, lo, hi)
        Db, Ib, _ = whole.search(Q, 10, 3, bitset=O.range_bitset(ids, attr, lo, hi, n), nbits=n)
        assert np.array_equal(I, Ib), (lo, hi)
        assert np.allclose(D, Db, rtol=1e-12, atol=0)


@settings(max_examples=15, deadline=None)
@given(st.integers(0, 2**31 - 1), st.integers(1, 3))
def test_multivector_brute_force(seed, mu):
    rng = np.random.default_rng(seed)
    n, m, k = 25, 3, 6
    dims = rng.integers(1, 5, size=mu)
    Xs = [rng.integers(-3, 4, size=(n, dd)).astype(np.float32) for dd in dims]
    Qs = [rng.integers(-3, 4, size=(m, dd)).astype(np.float32) for dd in dims]
    w = rng.integers(1, 4, size=mu).astype(np.float64) / 2.0
    ids = rng.permutation(100)[:n]
    D, I = O.multivector_topk(Xs, ids, Qs, w, k)
    for j in range(m):
        s = [(math.fsum(w[i] * math.fsum(float(a) * float(b) for a, b in zip(Qs[i][j], Xs[i][r])) for i in range(mu)), int(ids[r]))
             for r in range(n)]
        s.sort(key=lambda t: (-t[0], t[1]))
        assert I[j].tolist() == [t[1] for t in s[:k]]
        assert np.allclose(D[j], [t[0] for t in s[:k]], rtol=0, atol=1e-12)


def test_multivector_special_cases_and_fusion_identity():
    rng = np.random.default_rng(11)
    n, m = 80, 5
    Xs = [rng.normal(size=(n, 4)).astype(np.float32), rng.normal(size=(n, 6)).astype(np.float32)]
    Qs = [rng.normal(size=(m, 4)).astype(np.float32), rng.normal(size=(m, 6)).astype(np.float32)]
    ids = np.arange(n)
    # mu = 1 is a plain inner-product k-NN
    D, I = O.multivector_topk(Xs[:1], ids, Qs[:1], [1.0], 9)
    De, Ie = O.exact_knn(Xs[0], ids, Qs[0], 9, O.IP)
    assert np.array_equal(I, Ie) and np.allclose(D, De, rtol=1e-12)
    # a zero weight drops its vector
    D, I = O.multivector_topk(Xs, ids, Qs, [0.0, 2.0], 9)
    De, Ie = O.exact_knn(Xs[1], ids, 2.0 * Qs[1], 9, O.IP)
    assert np.array_equal(I, Ie) and np.allclose(D, De, rtol=1e-12)
    # vector fusion: one IP search of [w0 q0, w1 q1] over [v0, v1]
    w = [0.7, 1.9]
    D, I = O.multivector_topk(Xs, ids, Qs, w, 12)
    Xf = np.concatenate(Xs, axis=1)
    Qf = np.concatenate([w[0] * Qs[0].astype(np.float64), w[1] * Qs[1].astype(np.float64)], axis=1)
    De, Ie = O.exact_knn(Xf, ids, Qf, 12, O.IP)
    assert np.array_equal(I, Ie) and np.allclose(D, De, rtol=1e-12)
    # swapping the weights changes the answer (a weight applied to the wrong vector is caught)
    _, I2 = O.multivector_topk(Xs, ids, Qs, w[::-1], 12)
    assert not np.array_equal(I, I2)
