"""GPU parity of SURVEY §8(f) row f3, IVF_PQ (through the C ABI) against oracle/pq.py: the stored
sub-codes equal the oracle's encoding bit for bit, and searches (seeded two-phase, L2 and IP,
bitset, k > 256) return the oracle's asymmetric distances (fp64 distance to the decoded vector;
the GPU sums fp32 table entries: rtol 1e-5) with ids equal up to ties (conditional protocol)."""
import numpy as np
import pytest
import torch

import mvgen as G
import oracle as O

from ._parity import candidate_map, check_assignment, check_probes, check_topk, oracle_from_gpu_storage

pytestmark = pytest.mark.gpu


def _data(n, nq, d=96):
    spec = G.DeepSpec(d=d, n_micro=1024)
    return G.deep_base(n, d=d, spec=spec), G.deep_queries(nq, d=d, spec=spec)


def _oracle_pq(ix, metric, C, X, ids, cb):
    oi, gl = oracle_from_gpu_storage(ix, metric, O.FLAT, C, X, ids)
    op = O.IvfPqIndex(X.shape[1], metric, C, cb)
    op.add(X, ids, lists=gl)
    return op, gl


@pytest.mark.parametrize("metric,k,bits", [("l2", 20, False), ("ip", 20, True), ("l2", 300, True)])
def test_ivfpq_vs_oracle(metric, k, bits):
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index
    n, nq, d, M, nlist, nprobe = 10_000, 24, 96, 16, 32, 6
    X, Q = _data(n, nq, d)
    ids = G.permuted_ids(n, seed=9)
    C = X[:: n // nlist][:nlist].clone()
    rng = np.random.default_rng(2)
    cb = X.numpy()[rng.choice(n, 256, replace=False)].reshape(256, M, d // M).transpose(1, 0, 2).copy()
    ix = Index(d, metric, "pq", nlist)
    ix.set_centroids(C.cuda())
    ix.set_pq(M, torch.from_numpy(cb).cuda())
    assert np.array_equal(ix.get_pq(), cb)
    ix.add(X.cuda(), ids.cuda())
    mo = O.L2 if metric == "l2" else O.IP
    op, gl = _oracle_pq(ix, mo, C.numpy(), X.numpy(), ids.numpy(), cb)
    check_assignment(gl, X.numpy(), C.numpy(), mo)
    # the sub-codes, in storage order, equal the oracle's encoding of the same rows
    off, sids, codes = ix.storage(codes=True)
    pos = {int(v): r for r, v in enumerate(ids.numpy().tolist())}
    rows = np.array([pos[int(v)] for v in sids.tolist()])
    assert np.array_equal(codes, O.pq_encode(X.numpy()[rows], cb))
    bs, nbits = (G.mod_bitset(n, 10), n) if bits else (None, 0)
    P = ix.search_probes(Q.cuda(), nprobe).cpu().numpy()
    check_probes(P, Q.numpy(), C.numpy(), nprobe, mo)
    D, I = ix.search(Q.cuda(), k, nprobe, bitset=None if bs is None else bs.cuda(), nbits=nbits)
    torch.cuda.synchronize()
    assert ix.describe()["last_scan"] == "simt.pq_adc"
    bsn = None if bs is None else bs.numpy()
    Do, Io, _ = op.search(Q.numpy(), k, nprobe, bitset=bsn, nbits=nbits, probes=P)
    cm = [candidate_map(op, Q.numpy()[i], P[i], bsn, nbits) for i in range(nq)]
    check_topk(D.cpu().numpy(), I.cpu().numpy(), Do, Io, cm, rtol=1e-5, atol=1e-5)


def test_ivfpq_train_and_full_probe():
    """train_pq (mv_kmeans per sub-space) then nprobe = nlist: exact search over the decoded codes."""
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index
    n, nq, d, M, nlist = 12_000, 25, 64, 8, 16
    X, Q = _data(n, nq, d)
    ids = torch.arange(n)
    ix = Index(d, "l2", "pq", nlist)
    ix.set_centroids(X[:: n // nlist][:nlist].cuda())
    ix.train_pq(M, X.cuda(), niter=4)
    cb = ix.get_pq()
    ix.add(X.cuda(), ids.cuda())
    D, I = ix.search(Q.cuda(), 10, nlist)
    torch.cuda.synchronize()
    Xh = O.pq_decode(O.pq_encode(X.numpy(), cb), cb)
    De, Ie = O.exact_knn(Xh, ids.numpy(), Q.numpy(), 10, O.L2)
    cm = [dict(zip(ids.tolist(), O.distances(Q.numpy()[i], Xh, O.L2))) for i in range(nq)]
    check_topk(D.cpu().numpy(), I.cpu().numpy(), De, Ie, cm, rtol=1e-5, atol=1e-5)
    # the trained codebooks quantize better than the initial sub-centroids (the first 256 rows)
    init = X.numpy()[:256].reshape(256, M, d // M).transpose(1, 0, 2)
    err = lambda c: float(((O.pq_decode(O.pq_encode(X.numpy()[:2000], c), c) - X.numpy()[:2000]) ** 2).sum())
    assert err(cb) < err(init)
