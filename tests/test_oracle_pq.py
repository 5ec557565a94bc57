"""Pins for oracle/pq.py (``-m "not gpu"``): the encoder against a pure-Python
brute force, M = 1 against the coarse quantizer's assignment (vector quantization), the
asymmetric-distance identity sum_m ||q_m - C_m[c_m]||^2 = ||q - x_hat||^2, and IVF_PQ with
nprobe = nlist against exact search over the decoded vectors."""
import math

import numpy as np
from hypothesis import given, settings, strategies as st

import oracle as O


def _cb(rng, M, dsub, scale=3):
    return rng.integers(-scale, scale + 1, size=(M, 256, dsub)).astype(np.float32)


@settings(max_examples=10, deadline=None)
@given(st.integers(0, 2**31 - 1), st.sampled_from([(1, 4), (2, 2), (4, 1)]))
def test_encode_brute_force(seed, shape):
    M, dsub = shape
    rng = np.random.default_rng(seed)
    cb = _cb(rng, M, dsub)
    X = rng.integers(-4, 5, size=(15, M * dsub)).astype(np.float32)
    codes = O.pq_encode(X, cb)
    for i in range(15):
        for m in range(M):
            best = min(range(256), key=lambda j: (math.fsum((float(X[i, m * dsub + t]) - float(cb[m, j, t])) ** 2
                                                            for t in range(dsub)), j))
            assert codes[i, m] == best
    Xh = O.pq_decode(codes, cb)
    assert np.array_equal(Xh[:, :dsub], cb[0][codes[:, 0]])


def test_single_subspace_is_vector_quantization():
    rng = np.random.default_rng(3)
    cb = rng.normal(size=(1, 256, 6)).astype(np.float32)
    X = rng.normal(size=(200, 6)).astype(np.float32)
    assert np.array_equal(O.pq_encode(X, cb)[:, 0], O.assign(X, cb[0], O.L2))


def test_adc_identity():
    rng = np.random.default_rng(8)
    M, dsub = 8, 4
    cb = rng.normal(size=(M, 256, dsub)).astype(np.float32)
    X = rng.normal(size=(50, M * dsub)).astype(np.float32)
    q = rng.normal(size=M * dsub).astype(np.float64)
    codes = O.pq_encode(X, cb)
    Xh = O.pq_decode(codes, cb).astype(np.float64)
    tables = np.array([[((q[m * dsub:(m + 1) * dsub] - cb[m, j].astype(np.float64)) ** 2).sum() for j in range(256)]
                       for m in range(M)])
    adc = np.array([sum(tables[m, codes[i, m]] for m in range(M)) for i in range(50)])
    assert np.allclose(adc, O.distances(q, Xh, O.L2), rtol=1e-12)
    ip_tables = np.array([[q[m * dsub:(m + 1) * dsub] @ cb[m, j].astype(np.float64) for j in range(256)] for m in range(M)])
    adc_ip = np.array([sum(ip_tables[m, codes[i, m]] for m in range(M)) for i in range(50)])
    assert np.allclose(adc_ip, O.distances(q, Xh, O.IP), rtol=1e-12)


def test_ivfpq_full_probe_equals_exact_on_decoded():
    rng = np.random.default_rng(1)
    d, M = 16, 4
    cb = rng.normal(size=(M, 256, d // M)).astype(np.float32)
    X = rng.normal(size=(300, d)).astype(np.float32)
    Q = rng.normal(size=(5, d)).astype(np.float32)
    ids = rng.permutation(1000)[:300]
    C = X[:8]
    for metric in (O.L2, O.IP):
        ix = O.IvfPqIndex(d, metric, C, cb)
        ix.add(X, ids)
        D, I, _ = ix.search(Q, 10, 8)
        Xh = O.pq_decode(O.pq_encode(X, cb), cb)
        De, Ie = O.exact_knn(Xh, ids, Q, 10, metric)
        assert np.array_equal(I, Ie) and np.allclose(D, De, rtol=1e-12)
