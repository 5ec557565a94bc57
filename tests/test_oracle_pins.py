"""Pins for the oracle (``-m "not gpu"``): each test checks the oracle against something other
than itself -- a value printed/fixed by the paper, a hand computation, a library routine, brute
force, or an invariant the method guarantees.  DESIGN.md §2 maps every oracle function to the
tests below."""
import itertools
import json
import math
import os

import numpy as np
import pytest
import scipy.spatial.distance as ssd
from hypothesis import given, settings, strategies as st

import oracle as O

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def _rng(seed):
    return np.random.default_rng(seed)


# --------------------------------------------------------------------------- distances
def test_hand_distances():
    g = _gold("hand_distances.json")
    q, X = np.array(g["query"]), np.array(g["vectors"])
    assert O.distances(q, X, O.L2).tolist() == g["l2"]
    assert O.distances(q, X, O.IP).tolist() == g["ip"]
    ids = np.arange(len(X))
    _, I = O.exact_knn(X, ids, q[None], 2, O.L2)
    assert I[0].tolist() == g["top2_l2_ids"]
    _, I = O.exact_knn(X, ids, q[None], 2, O.IP)
    assert I[0].tolist() == g["top2_ip_ids"]


def test_distances_match_scipy():
    r = _rng(1)
    Q = r.standard_normal((7, 33)).astype(np.float32)
    X = r.standard_normal((50, 33)).astype(np.float32)
    ref_l2 = ssd.cdist(Q.astype(np.float64), X.astype(np.float64), "sqeuclidean")
    ref_ip = Q.astype(np.float64) @ X.astype(np.float64).T
    for i in range(len(Q)):
        np.testing.assert_allclose(O.distances(Q[i], X, O.L2), ref_l2[i], rtol=1e-12, atol=1e-12)
        np.testing.assert_allclose(O.distances(Q[i], X, O.IP), ref_ip[i], rtol=1e-12, atol=1e-12)


def test_integer_data_distances_exact():
    """SIFT-shaped integer data: fp64 distances equal exact int64 arithmetic."""
    r = _rng(2)
    Q = r.integers(0, 256, (5, 128))
    X = r.integers(0, 256, (40, 128))
    for i in range(5):
        exact = ((X - Q[i]) ** 2).sum(1)
        assert np.array_equal(O.distances(Q[i].astype(np.float32), X.astype(np.float32), O.L2), exact.astype(np.float64))
        exact_ip = (X * Q[i]).sum(1)
        assert np.array_equal(O.distances(Q[i].astype(np.float32), X.astype(np.float32), O.IP), exact_ip.astype(np.float64))


# --------------------------------------------------------------------------- top-k / exact
def _brute(X, ids, q, k, metric, excl=()):
    """Independent brute force: pure Python, math.fsum, explicit sort tuples."""
    items = []
    for r, (x, i) in enumerate(zip(X.tolist(), ids.tolist())):
        if i in excl:
            continue
        if metric == O.L2:
            d = math.fsum((a - b) ** 2 for a, b in zip(q.tolist(), x))
            items.append((d, i, r))
        else:
            d = math.fsum(a * b for a, b in zip(q.tolist(), x))
            items.append((-d, i, r))
    items.sort()
    out = [(t[0] if metric == O.L2 else -t[0], t[1]) for t in items[:k]]
    pad = math.inf if metric == O.L2 else -math.inf
    out += [(pad, -1)] * (k - len(out))
    return out


@settings(max_examples=60, deadline=None)
@given(n=st.integers(0, 25), d=st.integers(1, 6), k=st.integers(1, 30), metric=st.sampled_from([0, 1]),
       seed=st.integers(0, 10_000), ints=st.booleans())
def test_exact_knn_vs_bruteforce(n, d, k, metric, seed, ints):
    r = _rng(seed)
    X = (r.integers(-3, 4, (n, d)) if ints else r.standard_normal((n, d))).astype(np.float32)
    q = (r.integers(-3, 4, d) if ints else r.standard_normal(d)).astype(np.float32)
    ids = r.permutation(3 * n + 1)[:n].astype(np.int64)
    D, I = O.exact_knn(X, ids, q[None], k, metric)
    ref = _brute(X, ids, q, k, metric)
    assert I[0].tolist() == [t[1] for t in ref]
    np.testing.assert_allclose(D[0], [t[0] for t in ref], rtol=1e-12, atol=1e-12)


def test_ties_broken_by_smaller_id():
    X = np.array([[1.0, 0], [0, 1.0], [-1.0, 0], [0, -1.0]], dtype=np.float32)
    ids = np.array([40, 10, 30, 20])
    D, I = O.exact_knn(X, ids, np.zeros((1, 2), np.float32), 4, O.L2)
    assert I[0].tolist() == [10, 20, 30, 40] and D[0].tolist() == [1.0] * 4


def test_padding_when_fewer_than_k():
    X = np.eye(3, dtype=np.float32)
    D, I = O.exact_knn(X, np.arange(3), np.zeros((1, 3), np.float32), 5, O.L2)
    assert I[0].tolist() == [0, 1, 2, -1, -1] and np.isinf(D[0, 3:]).all() and (D[0, 3:] > 0).all()
    D, I = O.exact_knn(X, np.arange(3), np.ones((1, 3), np.float32), 5, O.IP)
    assert I[0, 3:].tolist() == [-1, -1] and (D[0, 3:] == -np.inf).all()


# --------------------------------------------------------------------------- large k rounds
@settings(max_examples=40, deadline=None)
@given(n=st.integers(1, 300), k=st.integers(1, 320), rk=st.integers(1, 64), metric=st.sampled_from([0, 1]),
       seed=st.integers(0, 1000))
def test_rounds_equal_single_sort(n, k, rk, metric, seed):
    """the round-by-round procedure (filter d < d_l and recorded ties) reaches
    exactly the plain top-k -- here with heavy ties (small integer distances)."""
    r = _rng(seed)
    D = r.integers(0, 12, n).astype(np.float64)
    ids = r.integers(0, 50, n)
    rows = np.arange(n)
    D1, I1, _ = O.select_topk(D, ids, rows, k, metric)
    D2, I2 = O.topk_rounds(D, ids, rows, k, metric, round_k=rk)
    assert I1.tolist() == I2.tolist() and np.array_equal(D1, D2)


# --------------------------------------------------------------------------- coarse
def test_figure2_instance():
    g = _gold("figure2.json")
    C, X, q = (np.array(g[k], dtype=np.float32) for k in ("centroids", "vectors", "query"))
    assert O.assign(X, C, O.L2).tolist() == g["expected_assignment"]
    assert O.probe(q[None], C, g["nprobe"], O.L2)[0].tolist() == g["expected_probes"]
    idx = O.IvfIndex(2, O.L2, O.FLAT, C)
    idx.add(X, np.arange(10))
    _, I, _ = idx.search(q[None], 10, g["nprobe"])
    assert sorted(I[0][I[0] >= 0].tolist()) == g["expected_scanned_ids"]
    assert (I[0][7:] == -1).all()


def test_assign_and_probe_ties_smaller_centroid():
    C = np.array([[1.0, 0.0], [-1.0, 0.0], [0.0, 1.0]], dtype=np.float32)
    x = np.zeros((1, 2), np.float32)
    assert O.assign(x, C, O.L2).tolist() == [0]
    assert O.probe(x, C, 3, O.L2)[0].tolist() == [0, 1, 2]
    assert O.probe(x, C, 10, O.L2).shape == (1, 3)          # nprobe > nlist clamps
    assert O.assign(np.array([[0.0, 1.0]], np.float32), C, O.IP).tolist() == [2]


def test_probe_matches_scipy_argsort():
    r = _rng(5)
    C = r.standard_normal((64, 16)).astype(np.float32)
    Q = r.standard_normal((20, 16)).astype(np.float32)
    ref = np.argsort(ssd.cdist(Q.astype(np.float64), C.astype(np.float64), "sqeuclidean"), axis=1, kind="stable")[:, :9]
    assert np.array_equal(O.probe(Q, C, 9, O.L2), ref)
    refip = np.argsort(-(Q.astype(np.float64) @ C.astype(np.float64).T), axis=1, kind="stable")[:, :9]
    assert np.array_equal(O.probe(Q, C, 9, O.IP), refip)


# --------------------------------------------------------------------------- IVF invariants
def _make(kind, metric, n=400, d=12, nlist=8, seed=0, ints=False):
    r = _rng(seed)
    X = (r.integers(0, 16, (n, d)) if ints else r.standard_normal((n, d))).astype(np.float32)
    C = X[r.choice(n, nlist, replace=False)] + np.float32(0.01)
    ids = r.permutation(10 * n)[:n].astype(np.int64)
    idx = O.IvfIndex(d, metric, kind, C)
    if kind == O.SQ8:
        idx.train_sq8(X)
    idx.add(X, ids)
    Q = (r.integers(0, 16, (30, d)) if ints else r.standard_normal((30, d))).astype(np.float32)
    return idx, X, ids, Q


@pytest.mark.parametrize("metric", [O.L2, O.IP])
def test_flat_nprobe_nlist_equals_exact(metric):
    idx, X, ids, Q = _make(O.FLAT, metric)
    De, Ie = O.exact_knn(X, ids, Q, 17, metric)
    D, I, _ = idx.search(Q, 17, idx.nlist)
    assert np.array_equal(I, Ie) and np.array_equal(D, De)


@pytest.mark.parametrize("metric", [O.L2, O.IP])
def test_nlist1_equals_exact(metric):
    r = _rng(3)
    X = r.standard_normal((200, 8)).astype(np.float32)
    ids = np.arange(200)
    idx = O.IvfIndex(8, metric, O.FLAT, X[:1])
    idx.add(X, ids)
    Q = r.standard_normal((10, 8)).astype(np.float32)
    assert np.array_equal(idx.search(Q, 9, 1)[1], O.exact_knn(X, ids, Q, 9, metric)[1])


@pytest.mark.parametrize("metric", [O.L2, O.IP])
def test_sq8_nprobe_nlist_equals_exact_on_decoded(metric):
    idx, X, ids, Q = _make(O.SQ8, metric)
    Xhat = O.sq8_decode(O.sq8_encode(X, idx.vmin, idx.vdiff), idx.vmin, idx.vdiff)
    De, Ie = O.exact_knn(Xhat, ids, Q, 13, metric)
    D, I, _ = idx.search(Q, 13, idx.nlist)
    assert np.array_equal(I, Ie) and np.array_equal(D, De)


def test_kth_distance_monotone_in_nprobe():
    idx, X, ids, Q = _make(O.FLAT, O.L2)
    prev = None
    for npb in range(1, idx.nlist + 1):
        D, _, _ = idx.search(Q, 10, npb)
        if prev is not None:
            assert (D[:, -1] <= prev + 0).all()
        prev = D[:, -1]


def test_candidates_are_exactly_probed_members():
    idx, X, ids, Q = _make(O.FLAT, O.L2, n=120, nlist=6)
    a = O.assign(X, idx.C, O.L2)
    P = O.probe(Q, idx.C, 2, O.L2)
    _, I, _ = idx.search(Q, 1000, 2)
    for i in range(len(Q)):
        expect = set(ids[np.isin(a, P[i])].tolist())
        assert set(I[i][I[i] >= 0].tolist()) == expect


# --------------------------------------------------------------------------- bitset
def test_bitset_semantics():
    idx, X, ids, Q = _make(O.FLAT, O.L2, n=300)
    nbits = int(ids.max()) + 1
    zero = np.zeros((nbits + 7) // 8, np.uint8)
    assert np.array_equal(idx.search(Q, 10, 3, zero, nbits)[1], idx.search(Q, 10, 3)[1])
    ones = np.full((nbits + 7) // 8, 255, np.uint8)
    assert (idx.search(Q, 10, 8, ones, nbits)[1] == -1).all()
    r = _rng(9)
    bits = r.random(nbits) < 0.5
    packed = np.packbits(bits, bitorder="little")
    _, I, _ = idx.search(Q, 50, 8, packed, nbits)
    got = I[I >= 0]
    assert not bits[got].any()
    # == exact search over the survivors (strategy B is exact w.r.t. the bitmap)
    keep = ~bits[ids]
    Ie = O.exact_knn(X[keep], ids[keep], Q, 50, O.L2)[1]
    assert np.array_equal(I, Ie)
    # ids >= nbits are never excluded
    assert not O.bit_is_set(ones, 8, np.array([8, 9, 100])).any()
    assert O.bit_is_set(np.array([0b00000100], np.uint8), 8, np.array([2]))[0]


# --------------------------------------------------------------------------- SQ8 codec
def test_sq8_hand_values():
    g = _gold("sq8_hand.json")
    vmin, vdiff = np.array(g["vmin"], np.float32), np.array(g["vdiff"], np.float32)
    codes = O.sq8_encode(np.array(g["x"], np.float32), vmin, vdiff)
    assert codes.tolist() == g["codes"]
    dec = O.sq8_decode(codes[:1], vmin, vdiff)[0]
    assert dec.tolist() == np.array(g["decoded_first_row_exact"], np.float32).tolist()


def test_sq8_roundtrip_bound_and_endpoints():
    r = _rng(11)
    X = (r.standard_normal((500, 24)) * r.uniform(0.1, 50, 24)).astype(np.float32)
    vmin, vdiff = O.sq8_train(X)
    assert np.array_equal(vmin, X.min(0)) and np.array_equal(vdiff, X.max(0) - X.min(0))
    codes = O.sq8_encode(X, vmin, vdiff)
    assert (codes[X.argmin(0), np.arange(24)] == 0).all()
    assert (codes[X.argmax(0), np.arange(24)] == 255).all()
    err = np.abs(O.sq8_decode(codes, vmin, vdiff).astype(np.float64) - X)
    # bin width vdiff/255, mid-bin decode -> half a bin, except the top value (255) is a full
    # half bin above/below; allow fp32 rounding slack
    bound = vdiff.astype(np.float64) / 255.0 * 1.0 + 1e-5 * np.abs(X).max(0)
    assert (err <= bound[None, :]).all()
    interior = codes < 255
    bound_half = vdiff.astype(np.float64) / 510.0 + 1e-5 * np.abs(X).max(0)
    assert (err[interior] <= np.broadcast_to(bound_half, err.shape)[interior]).all()
    # one byte per dimension: 1/4 the space of fp32
    assert codes.nbytes * 4 == X.nbytes


# --------------------------------------------------------------------------- shard merge
@pytest.mark.parametrize("G", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("metric", [O.L2, O.IP])
def test_merge_of_shards_equals_global(G, metric):
    """per-thread heaps merged give the global top-k; PAPER.md:773-776 the
    same holds for per-segment results."""
    r = _rng(G)
    X = r.integers(0, 6, (240, 4)).astype(np.float32)          # many exact ties
    ids = r.permutation(240).astype(np.int64)
    Q = r.integers(0, 6, (12, 4)).astype(np.float32)
    k = 25
    parts = []
    for g in range(G):
        sel = (ids % G) == g
        parts.append(O.exact_knn(X[sel], ids[sel], Q, k, metric))
    D, I = O.merge_topk(parts, k, metric)
    De, Ie = O.exact_knn(X, ids, Q, k, metric)
    assert np.array_equal(I, Ie) and np.array_equal(D, De)


# --------------------------------------------------------------------------- recall
def test_recall_definition():
    """recall = |S ∩ S'| / |S|."""
    S = np.array([[1, 2, 3, 4], [5, 6, 7, 8]])
    Sp = np.array([[4, 3, 9, 10], [5, 6, 7, 8]])
    assert O.recall_at_k(S, Sp, 4) == pytest.approx(6 / 8)
    assert O.recall_at_k(S, Sp, 2) == pytest.approx(2 / 4)
