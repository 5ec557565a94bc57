"""Pins for oracle/kmeans.py (``-m "not gpu"``): a hand-computed Lloyd step,
the fixed point of well-separated clusters, Lloyd's monotone SSE, empty clusters, the spherical
variant, and a brute-force (pure Python) step."""
import math

import numpy as np
from hypothesis import given, settings, strategies as st

import oracle as O


def test_hand_step():
    # rows 0, 1, 10, 12 on a line; centroids 0 and 9: {0, 1} -> 0, {10, 12} -> 9; means 0.5 and 11
    X = np.array([[0.0], [1.0], [10.0], [12.0]], dtype=np.float32)
    C, a = O.km.lloyd_step(X, np.array([[0.0], [9.0]], dtype=np.float32), O.L2)
    assert a.tolist() == [0, 0, 1, 1]
    assert C.ravel().tolist() == [0.5, 11.0]


def test_fixed_point_and_empty_cluster():
    rng = np.random.default_rng(0)
    centres = np.array([[0, 0], [100, 0], [0, 100]], dtype=np.float64)
    X = np.concatenate([c + rng.normal(size=(50, 2)) for c in centres]).astype(np.float32)
    C1, a = O.km.lloyd_step(X, centres.astype(np.float32), O.L2)
    C2, a2 = O.km.lloyd_step(X, C1, O.L2)
    assert np.array_equal(a, a2) and np.array_equal(C1, C2)        # means of a stable partition
    far = np.concatenate([C1, [[1e6, 1e6]]]).astype(np.float32)    # a centroid no row is closest to
    C3, _ = O.km.lloyd_step(X, far, O.L2)
    assert C3[3].tolist() == [1e6, 1e6]


@settings(max_examples=20, deadline=None)
@given(st.integers(0, 2**31 - 1))
def test_sse_never_increases(seed):
    rng = np.random.default_rng(seed)
    X = rng.normal(size=(80, 3)).astype(np.float32)
    C = X[:6].copy()
    prev = math.inf
    for _ in range(5):
        a = O.assign(X, C, O.L2)
        cur = O.km.sse(X, C, a)
        assert cur <= prev * (1 + 1e-6)
        prev = cur
        C, _ = O.km.lloyd_step(X, C, O.L2, lists=a)


def test_brute_force_step_and_spherical():
    rng = np.random.default_rng(4)
    X = rng.integers(-5, 6, size=(40, 3)).astype(np.float32)
    C0 = (X[:4] + 0.25).astype(np.float32)
    C, a = O.km.lloyd_step(X, C0, O.L2)
    for l in range(4):  # pure Python: nearest by explicit sums, then the mean
        mine = [r for r in range(40)
                if min(range(4), key=lambda c: (math.fsum((float(X[r, j]) - float(C0[c, j])) ** 2 for j in range(3)), c)) == l]
        assert a[mine].tolist() == [l] * len(mine)
        if mine:
            assert np.allclose(C[l], [math.fsum(float(X[r, j]) for r in mine) / len(mine) for j in range(3)], rtol=1e-6)
    Cs, _ = O.km.lloyd_step(X, C0, O.IP, spherical=True)
    assert np.allclose(np.linalg.norm(Cs.astype(np.float64), axis=1), 1.0, atol=1e-6)
