"""GPU parity of SURVEY §8(f) row f4 (through the C ABI): strategy E partitions
(PartitionedIndex: mv_attr_bitset + the a2-a8 search per partition + mv_merge_topk) against
oracle.partition_search, and multi-vector queries by vector fusion (MultiVectorIndex:
mv_fuse_rows + one IP search) against oracle.multivector_topk -- the paper's weighted-sum
definition computed per vector, not the fusion."""
import numpy as np
import pytest
import torch

import mvgen as G
import oracle as O

from ._parity import candidate_map, check_topk, oracle_from_gpu_storage

pytestmark = pytest.mark.gpu

RANGES = [(1, 100), (101, 200), (201, 300), (301, 400), (401, 500)]


def _data(n, nq, d, seed=7):
    spec = G.SiftSpec(d=d, n_micro=512)
    X, Q = G.sift_base(n, d=d, spec=spec), G.sift_queries(nq, d=d, spec=spec)
    g = torch.Generator().manual_seed(seed)
    ids = torch.randperm(4 * n, generator=g)[:n]
    attr = torch.randint(1, 501, (n,), generator=g)
    return X, Q, ids, attr


@pytest.mark.parametrize("metric", ["l2", "ip"])
def test_strategy_e_vs_oracle(metric):
    from paper_conf_sigmod_wangygjxlwglxyy21_b200.filtering import PartitionedIndex
    n, nq, d, nlist, nprobe, k = 6000, 40, 64, 24, 6, 15
    X, Q, ids, attr = _data(n, nq, d)
    C = X[:: n // nlist][:nlist] + 0.25
    px = PartitionedIndex(d, RANGES, metric, "flat", nlist)
    px.set_centroids(C.cuda())
    px.add(X.cuda(), ids.cuda(), attr.cuda())
    mo = O.L2 if metric == "l2" else O.IP
    # the oracle's partitions hold the GPU's accepted assignment (conditional protocol)
    parts = []
    for (lo, hi), ix in zip(RANGES, px.parts):
        sel = ((attr >= lo) & (attr <= hi)).numpy()
        oi, _ = oracle_from_gpu_storage(ix, mo, O.FLAT, C.numpy(), X.numpy()[sel], ids.numpy()[sel])
        parts.append((oi, (lo, hi), ids.numpy()[sel], attr.numpy()[sel]))
    P = px.parts[0].search_probes(Q.cuda(), nprobe).cpu().numpy()
    for lo, hi in [(50, 250), (1, 500), (120, 180), (401, 500), (600, 700), (100, 101)]:
        D, I = px.search(Q.cuda(), k, nprobe, lo, hi)
        torch.cuda.synchronize()
        assert px.last_plan == O.partition_plan(RANGES, lo, hi)
        Do, Io = O.partition_search(parts, Q.numpy(), k, nprobe, lo, hi, probes=P)
        # integer data: exact distances, (distance, id) order on both sides
        check_topk(D.cpu().numpy(), I.cpu().numpy(), Do, Io, exact=True)


def test_strategy_e_equals_strategy_b_on_one_index():
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index
    from paper_conf_sigmod_wangygjxlwglxyy21_b200.filtering import PartitionedIndex
    n, nq, d, nlist, nprobe, k = 8000, 32, 128, 32, 5, 40
    X, Q, ids, attr = _data(n, nq, d, seed=3)
    C = X[:: n // nlist][:nlist] + 0.5
    px = PartitionedIndex(d, RANGES, "l2", "sq8", nlist)
    px.set_centroids(C.cuda())
    px.train_sq8(X.cuda())
    px.add(X.cuda(), ids.cuda(), attr.cuda())
    whole = Index(d, "l2", "sq8", nlist)
    whole.set_centroids(C.cuda())
    whole.set_sq8(*px.parts[0].get_sq8())
    whole.add(X.cuda(), ids.cuda())
    nbits = int(ids.max()) + 1
    for lo, hi in [(50, 250), (120, 180), (1, 500)]:
        D, I = px.search(Q.cuda(), k, nprobe, lo, hi)
        bs = torch.from_numpy(O.range_bitset(ids.numpy(), attr.numpy(), lo, hi, nbits)).cuda()
        Db, Ib = whole.search(Q.cuda(), k, nprobe, bitset=bs, nbits=nbits)
        torch.cuda.synchronize()
        assert torch.equal(I, Ib) and torch.equal(D, Db)


def test_attr_bitset_kernel_matches_oracle():
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import _lib as L
    import ctypes as C
    g = torch.Generator().manual_seed(1)
    n = 100000
    ids = torch.randperm(3 * n, generator=g)[:n]
    attr = torch.randint(-1000, 1000, (n,), generator=g)
    nbits = 3 * n + 5
    out = torch.full((((nbits + 31) // 32) * 4,), 0xAB, dtype=torch.uint8, device="cuda")
    idc, atc = ids.cuda(), attr.cuda()
    L.check(L.load().mv_attr_bitset(C.c_void_p(idc.data_ptr()), C.c_void_p(atc.data_ptr()), n, -200, 350,
                                    C.c_void_p(out.data_ptr()), nbits, None))
    torch.cuda.synchronize()
    ref = O.range_bitset(ids.numpy(), attr.numpy(), -200, 350, nbits)
    got = out.cpu().numpy()
    assert np.array_equal(got[:len(ref)], ref)
    assert not got[len(ref):].any()


@pytest.mark.parametrize("kind", ["flat", "sq8"])
def test_multivector_fusion_vs_oracle(kind):
    from paper_conf_sigmod_wangygjxlwglxyy21_b200.filtering import MultiVectorIndex
    dims, n, nq, k = [32, 48, 16], 5000, 24, 12
    Xs, Qs = [], []
    for j, dd in enumerate(dims):
        spec = G.DeepSpec(d=dd, n_micro=256, seed=100 + j)
        Xs.append(G.deep_base(n, d=dd, spec=spec))
        Qs.append(G.deep_queries(nq, d=dd, spec=spec))
    w = [0.5, 1.25, 2.0]
    ids = torch.arange(n) * 3 + 1
    mx = MultiVectorIndex(dims, kind, nlist=16)
    Xf = mx.fuse([x.cuda() for x in Xs])
    assert torch.equal(Xf.cpu(), torch.cat(Xs, dim=1))  # weights 1: plain concatenation
    mx.set_centroids(Xf[::n // 16][:16])
    if kind == "sq8":
        mx.train_sq8([x.cuda() for x in Xs])
    mx.add([x.cuda() for x in Xs], ids.cuda())
    D, I = mx.search([q.cuda() for q in Qs], w, k, 16)  # nprobe = nlist: exact over the stored vectors
    torch.cuda.synchronize()
    if kind == "flat":
        Do, Io = O.multivector_topk([x.numpy() for x in Xs], ids.numpy(), [q.numpy() for q in Qs], w, k)
        sc = [dict(zip(ids.tolist(), O.multivector_scores([x.numpy() for x in Xs], [q.numpy()[i] for q in Qs], w)))
              for i in range(nq)]
    else:
        # SQ8 stores the fused rows' codes: the oracle decodes them, splits them back into the mu
        # vectors and aggregates per vector
        vmin, vdiff = mx.index.get_sq8()
        Xh = O.sq8_decode(O.sq8_encode(Xf.cpu().numpy(), vmin, vdiff), vmin, vdiff)
        parts = np.split(Xh, np.cumsum(dims)[:-1], axis=1)
        Do, Io = O.multivector_topk(parts, ids.numpy(), [q.numpy() for q in Qs], w, k)
        sc = [dict(zip(ids.tolist(), O.multivector_scores(parts, [q.numpy()[i] for q in Qs], w))) for i in range(nq)]
    # fp32 rounding of w_i q_ij in the fused query: relative 2^-24 per term of the sum
    check_topk(D.cpu().numpy(), I.cpu().numpy(), Do, Io, sc, rtol=1e-5, atol=1e-6)
