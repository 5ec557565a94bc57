"""GPU parity: the CUDA path (through the C ABI) against the oracle on the same seeded inputs.

Sizes span several tiles and ragged tails while the oracle still finishes in seconds.  The
protocol is the conditional oracle of DESIGN.md §6: assignment checked first (equal or tied),
then the oracle re-runs the scan with the GPU's accepted assignment and probes, and ids must
match except at ties.  Integer-valued (SIFT-shaped) data are exact in fp32 and are compared
bit-for-bit.
"""
import numpy as np
import pytest
import torch

import mvgen as G
import oracle as O
from mvgen.kmeans import kmeans

from ._parity import candidate_map, check_assignment, check_probes, check_topk, oracle_from_gpu_storage

pytestmark = pytest.mark.gpu


def _mv():
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index, merge_topk
    return Index, merge_topk


def _sift(n, nq, d=128, n_micro=4096):
    spec = G.SiftSpec(d=d, n_micro=n_micro)
    return G.sift_base(n, d=d, spec=spec), G.sift_queries(nq, d=d, spec=spec)


def _deep(n, nq, d=96, n_micro=4096):
    spec = G.DeepSpec(d=d, n_micro=n_micro)
    return G.deep_base(n, d=d, spec=spec), G.deep_queries(nq, d=d, spec=spec)


def _build(X, ids, C, metric, kind, sq8_sample=None):
    Index, _ = _mv()
    ix = Index(X.shape[1], metric, kind, C.shape[0])
    ix.set_centroids(C.cuda())
    if kind == "sq8":
        ix.train_sq8((X if sq8_sample is None else sq8_sample).cuda())
    ix.add(X.cuda(), ids.cuda())
    return ix


def _run_conditional(ix, X, ids, C, Q, k, nprobe, metric_o, kind_o, bitset=None, nbits=0, atol=0.0, exact=False,
                     sample_assign=None):
    Xn, Cn, Qn, idn = X.numpy(), C.numpy(), Q.numpy(), ids.numpy()
    sq8 = ix.get_sq8() if kind_o == O.SQ8 else None
    oi, gl = oracle_from_gpu_storage(ix, metric_o, kind_o, Cn, Xn, idn, sq8)
    check_assignment(gl, Xn, Cn, metric_o, sample=sample_assign)
    P = ix.search_probes(Q.cuda(), nprobe).cpu().numpy()
    check_probes(P, Qn, Cn, nprobe, metric_o)
    bs_t = None if bitset is None else bitset.cuda()
    D, I = ix.search(Q.cuda(), k, nprobe, bitset=bs_t, nbits=nbits)
    torch.cuda.synchronize()
    Do, Io, _ = oi.search(Qn, k, nprobe, bitset=None if bitset is None else bitset.numpy(), nbits=nbits, probes=P)
    cm = [candidate_map(oi, Qn[i], P[i], None if bitset is None else bitset.numpy(), nbits) for i in range(len(Qn))]
    frac = check_topk(D.cpu().numpy(), I.cpu().numpy(), Do, Io, cm, atol=atol, exact=exact)
    return frac, D, I


# --------------------------------------------------------------------------------------------
def test_c1_exact_equals_bruteforce():
    """configs[0]: 10k x 128 SIFT-shaped, nlist = nprobe = 64, 100 queries, k = 10: IVF_FLAT with
    nprobe = nlist IS exact k-NN; integer data make fp32 exact -> bit-for-bit equality."""
    X, Q = _sift(10_000, 100)
    ids = torch.arange(10_000, dtype=torch.int64)
    C = kmeans(X, 64, iters=8)
    ix = _build(X, ids, C, "l2", "flat")
    D, I = ix.search(Q.cuda(), 10, 64)
    De, Ie = O.exact_knn(X.numpy(), ids.numpy(), Q.numpy(), 10, O.L2)
    check_topk(D.cpu().numpy(), I.cpu().numpy(), De, Ie, exact=True)


@pytest.mark.parametrize("n,nlist,nprobe,nq,k", [(20_000, 256, 16, 200, 10), (7_777, 97, 5, 61, 37)])
def test_flat_l2_sift_conditional(n, nlist, nprobe, nq, k):
    X, Q = _sift(n, nq)
    ids = G.permuted_ids(n, seed=3)
    C = kmeans(X, nlist, iters=6)
    ix = _build(X, ids, C, "l2", "flat")
    frac, _, _ = _run_conditional(ix, X, ids, C, Q, k, nprobe, O.L2, O.FLAT, exact=False)
    assert frac == 1.0  # integer data: no ties can be broken differently except exact ties by id


@pytest.mark.parametrize("metric", ["l2", "ip"])
@pytest.mark.parametrize("d,flat_qc", [(128, 0), (128, 80), (128, 48), (192, 0), (320, 0), (64, 16)])
def test_flat_tc_fractional_queries(metric, d, flat_qc):
    """Integer (tf32-exact) base data with fractional queries: the tensor-core scan takes the
    two-plane (hi/lo) items and the filter mode (DESIGN.md §5 "FLAT precision"); distances are the
    exact fp64 values (rtol 1e-5, atol 0).  flat_qc / d pick the 80-, 48- and 16-query item shapes
    whose two-plane width 2 roundup16(qc/2) exceeds roundup16(qc) (the operand and the TMEM
    accumulators must be sized for it)."""
    X, Q = _sift(15_000, 130, d=d, n_micro=2048)
    Q = Q * 0.7311 + 0.377  # not tf32-representable
    ids = G.permuted_ids(15_000, seed=5)
    C = kmeans(X, 128, iters=5)
    Index, _ = _mv()
    ix = Index(d, metric, "flat", 128)
    if flat_qc:
        ix.set_option("flat_qc", flat_qc)
    ix.set_centroids(C.cuda())
    ix.add(X.cuda(), ids.cuda())
    mo = O.L2 if metric == "l2" else O.IP
    frac, _, _ = _run_conditional(ix, X, ids, C, Q, 10, 9, mo, O.FLAT)
    desc = ix.describe()
    assert desc["last_scan"] == "tcgen05.tf32" and desc["tf32_exact"]
    assert frac > 0.999


@pytest.mark.parametrize("nprobe,metric", [(7, "l2"), (33, "l2"), (64, "ip"), (100, "l2"), (128, "ip")])
def test_coarse_probe_sets(nprobe, metric):
    """a2+a3 on the tensor cores: the probe sets (best-first order included) equal the oracle's
    fp64 top-nprobe modulo scores tied within 1e-5, across the nprobe <= 32, <= 64 and <= 128
    selection shapes, with fractional (two-plane) queries."""
    X, Q = _sift(20_000, 150)
    Q = Q * 0.93 + 0.21
    C = kmeans(X, 1000, iters=3)
    Index, _ = _mv()
    ix = Index(128, metric, "flat", 1000)
    ix.set_centroids(C.cuda())
    P = ix.search_probes(Q.cuda(), nprobe).cpu().numpy()
    assert ix.describe()["last_coarse"] == "tcgen05.tf32"
    mo = O.L2 if metric == "l2" else O.IP
    check_probes(P, Q.numpy(), C.numpy(), nprobe, mo)
    # best-first: the GPU's own order is non-decreasing in the fp64 score
    sc = np.stack([O.distances(Q.numpy()[i], C.numpy(), mo)[P[i]] for i in range(len(P))])
    if mo == O.IP:
        sc = -sc
    assert (np.diff(sc, axis=1) >= -1e-5 * np.abs(sc[:, 1:])).all()


@pytest.mark.parametrize("metric,k", [("ip", 20), ("l2", 20), ("ip", 300), ("l2", 1)])
def test_flat_deep_conditional(metric, k):
    """Arbitrary fp32 data (unit-norm Deep-shaped, not tf32-representable) on the tensor cores:
    tf32 filter with a rigorous bound + exact fp64 re-scoring; the exact top-k, distances within
    1e-5 relative with atol 0 (IVF_FLAT keeps the original vectors)."""
    X, Q = _deep(20_000, 150)
    ids = torch.arange(20_000, dtype=torch.int64) * 2 + 1
    C = kmeans(X, 128, iters=6, spherical=True)
    ix = _build(X, ids, C, metric, "flat")
    mo = O.IP if metric == "ip" else O.L2
    frac, _, _ = _run_conditional(ix, X, ids, C, Q, k, 8, mo, O.FLAT)
    desc = ix.describe()
    assert desc["last_scan"] == "tcgen05.tf32" and not desc["tf32_exact"]
    assert frac > 0.999


@pytest.mark.parametrize("kind,metric,d", [("flat", "l2", 512), ("flat", "ip", 500), ("sq8", "l2", 320),
                                           ("sq8", "ip", 512)])
def test_large_d_gaussian(kind, metric, d):
    """d up to the 512 limit of mv.h, fp32 Gaussian data (filter mode for FLAT)."""
    X = G.gaussian(6000, d, seed=31)
    Q = G.gaussian(70, d, seed=32)
    ids = G.permuted_ids(6000, seed=33)
    C = kmeans(X, 24, iters=4)
    ix = _build(X, ids, C, metric, kind)
    mo = O.IP if metric == "ip" else O.L2
    frac, _, _ = _run_conditional(ix, X, ids, C, Q, 25, 5, mo, O.FLAT if kind == "flat" else O.SQ8,
                                  atol=0.0 if kind == "flat" else 2e-6 * d)
    assert frac > 0.999


@pytest.mark.parametrize("metric", ["ip", "l2"])
def test_sq8_deep_bitset_conditional(metric):
    """configs[2] shape (downsized): Deep-shaped SQ8 with a 10% deletion bitset, k = 100 (lists
    longer than k -> in-scan selection)."""
    X, Q = _deep(30_000, 120)
    ids = torch.arange(30_000, dtype=torch.int64)
    C = kmeans(X, 48, iters=6, spherical=True)
    ix = _build(X, ids, C, metric, "sq8")
    mo = O.IP if metric == "ip" else O.L2
    # SQ8 params and codes are bit-exact with the oracle's codec
    vmin, vdiff = ix.get_sq8()
    ovmin, ovdiff = O.sq8_train(X.numpy())
    assert np.array_equal(vmin, ovmin) and np.array_equal(vdiff, ovdiff)
    off, sids, codes = ix.storage(codes=True)
    assert np.array_equal(codes, O.sq8_encode(X.numpy()[sids], ovmin, ovdiff))
    nbits = 30_000
    bs = G.mod_bitset(nbits, 10)
    frac, D, I = _run_conditional(ix, X, ids, C, Q, 100, 6, mo, O.SQ8, bitset=bs, nbits=nbits, atol=2e-6)
    assert frac > 0.999
    excl = G.unpack_bits(bs, nbits).numpy().astype(bool)
    got = I.cpu().numpy()
    assert not excl[got[got >= 0]].any()


@pytest.mark.parametrize("k", [10, 64])
def test_sq8_sift_l2_conditional(k):
    """configs[4] shape (downsized): SIFT-shaped IVF_SQ8 L2 -- the regime where the L2 expansion
    cancels hardest (norms ~400x the near-neighbour distances); distances within 1e-5 of fp64."""
    X, Q = _sift(15_000, 100, n_micro=1024)
    ids = G.permuted_ids(15_000, seed=13)
    C = kmeans(X, 32, iters=4)
    ix = _build(X, ids, C, "l2", "sq8")
    frac, D, I = _run_conditional(ix, X, ids, C, Q, k, 5, O.L2, O.SQ8)
    assert ix.describe()["last_scan"] == "tcgen05.i8"
    assert frac > 0.999


@pytest.mark.parametrize("k", [300, 1000, 2048, 3000, 4096, 16384])
def test_large_k(k):
    """k > 1024: single-pass radix select == plain top-k of the oracle."""
    n = 20_000
    X, Q = _sift(n, 12)
    ids = G.permuted_ids(n, seed=5)
    C = kmeans(X, 40, iters=5)
    ix = _build(X, ids, C, "l2", "flat")
    nprobe = 40 if k == 16384 else 12  # 40 = nlist: every bucket
    frac, D, I = _run_conditional(ix, X, ids, C, Q, k, nprobe, O.L2, O.FLAT)
    assert frac == 1.0


def test_large_k_bucket_piles():
    """k = 1000 where 3000 candidates share one distance and ten lie much closer: the winners pile
    into one bucket of k_final_big's bucket sort, which then falls back to the bitonic sort; both
    orders are the oracle's (distance, id) order (§3.3)."""
    d, n = 16, 4000
    r = np.random.default_rng(11)
    X = np.full((n, d), 100.0, np.float32)
    X[:3000] = 5.0                                         # 3000 rows at one distance from q = 0
    X[3000:3010] = r.integers(0, 3, (10, d)).astype(np.float32)  # ten much closer
    Q = np.zeros((3, d), np.float32)
    Q[1, 0] = 1.0
    Q[2] = 60.0                                            # the far rows are its nearest
    ids = G.permuted_ids(n, seed=3)
    Xt, Qt = torch.from_numpy(X), torch.from_numpy(Q)
    C = torch.from_numpy(X[:1].copy())
    ix = _build(Xt, ids, C, "l2", "flat")
    for k in (1000, 300):
        D, I = ix.search(Qt.cuda(), k, 1)
        De, Ie = O.exact_knn(X, ids.numpy(), Q, k, O.L2)
        assert np.array_equal(I.cpu().numpy(), Ie), k
        np.testing.assert_array_equal(D.cpu().numpy(), De.astype(np.float32))


def test_large_k_rounds_crosscheck():
    """The paper's rounds-of-1024 procedure on the oracle candidates gives the GPU answer."""
    n = 6000
    X, Q = _sift(n, 4)
    ids = torch.arange(n, dtype=torch.int64)
    C = kmeans(X, 8, iters=4)
    ix = _build(X, ids, C, "l2", "flat")
    D, I = ix.search(Q.cuda(), 3000, 8)
    for i in range(4):
        Dall = O.distances(Q.numpy()[i], X.numpy(), O.L2)
        Dr, Ir = O.topk_rounds(Dall, ids.numpy(), np.arange(n), 3000, O.L2, round_k=1024)
        assert np.array_equal(I.cpu().numpy()[i], Ir)


def test_edge_cases():
    Index, _ = _mv()
    d = 20  # not a multiple of 32: zero padding
    X = G.gaussian(500, d, seed=1)
    Q = G.gaussian(9, d, seed=2)
    C = X[:7].clone()
    # empty index -> all padding
    ix = Index(d, "l2", "flat", 7)
    ix.set_centroids(C.cuda())
    D, I = ix.search(Q.cuda(), 5, 3)
    assert (I == -1).all() and torch.isinf(D).all()
    # nq = 0
    D0, I0 = ix.search(Q[:0].cuda(), 5, 3)
    assert D0.shape == (0, 5)
    ids = torch.arange(500, dtype=torch.int64)
    ix.add(X.cuda(), ids.cuda())
    # k > candidates -> padding; nprobe > nlist clamps; all-ones bitset -> padding
    D, I = ix.search(Q.cuda(), 600, 100)
    De, Ie = O.exact_knn(X.numpy(), ids.numpy(), Q.numpy(), 600, O.L2)
    check_topk(D.cpu().numpy(), I.cpu().numpy(), De, Ie,
               cmaps=[{i: dd for i, dd in zip(range(500), O.distances(Q.numpy()[j], X.numpy(), O.L2))} for j in range(9)])
    ones = torch.full((63,), 255, dtype=torch.uint8)
    D, I = ix.search(Q.cuda(), 5, 7, bitset=ones.cuda(), nbits=500)
    assert (I == -1).all()
    # ids >= nbits are never excluded
    D, I = ix.search(Q.cuda(), 5, 7, bitset=ones.cuda(), nbits=100)
    assert (I >= 100).all()
    # reserved id -1 rejected; k out of range rejected
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import MvError
    with pytest.raises(MvError):
        ix.add(X[:2].cuda(), torch.tensor([3, -1]).cuda())
    with pytest.raises(MvError):
        ix.search(Q.cuda(), 16385, 3)
    with pytest.raises(MvError):
        ix.search(Q.cuda(), 0, 3)


def test_duplicate_ids_and_incremental_add():
    Index, _ = _mv()
    X, Q = _sift(3000, 20, d=32, n_micro=64)
    ids = torch.arange(3000, dtype=torch.int64) % 1000  # duplicates
    C = kmeans(X, 16, iters=4)
    ix = Index(32, "l2", "flat", 16)
    ix.set_centroids(C.cuda())
    ix.add(X[:1000].cuda(), ids[:1000].cuda())
    ix.add(X[1000:].cuda(), ids[1000:].cuda())   # second add: lists keep insertion order
    assert ix.ntotal == 3000
    oi = O.IvfIndex(32, O.L2, O.FLAT, C.numpy())
    oi.add(X.numpy(), ids.numpy())
    off_o, order = oi.storage()
    off_g, sids, _ = ix.storage()
    assert np.array_equal(off_g, off_o) and np.array_equal(sids, ids.numpy()[order])
    D, I = ix.search(Q.cuda(), 50, 4)
    Do, Io, _ = oi.search(Q.numpy(), 50, 4)
    check_topk(D.cpu().numpy(), I.cpu().numpy(), Do, Io, exact=True)


def test_host_buffers_and_determinism():
    X, Q = _sift(5000, 64, d=64, n_micro=256)
    ids = torch.arange(5000, dtype=torch.int64)
    C = kmeans(X, 32, iters=4)
    ix = _build(X, ids, C, "l2", "flat")
    Dd, Id = ix.search(Q.cuda(), 25, 5)
    Dh = np.empty((64, 25), np.float32)
    Ih = np.empty((64, 25), np.int64)
    ix.search(Q.numpy(), 25, 5, out=(Dh, Ih))
    assert np.array_equal(Dh, Dd.cpu().numpy()) and np.array_equal(Ih, Id.cpu().numpy())
    D2, I2 = ix.search(Q.cuda(), 25, 5)
    assert torch.equal(D2, Dd) and torch.equal(I2, Id)
    # per-query results do not depend on the rest of the batch
    D3, I3 = ix.search(Q[17:40].cuda(), 25, 5)
    assert torch.equal(D3, Dd[17:40]) and torch.equal(I3, Id[17:40])


@pytest.mark.parametrize("metric", ["l2", "ip"])
@pytest.mark.parametrize("nsrc,k", [(2, 10), (3, 7), (8, 64), (4, 2048)])
def test_merge_topk_vs_oracle(metric, nsrc, k):
    _, merge_topk = _mv()
    r = np.random.default_rng(nsrc * 100 + k)
    mo = O.L2 if metric == "l2" else O.IP
    nq = 33
    X = r.integers(0, 5, (nsrc * 400, 3)).astype(np.float32)
    ids = r.permutation(nsrc * 400).astype(np.int64)
    Qn = r.integers(0, 5, (nq, 3)).astype(np.float32)
    parts = [O.exact_knn(X[g::nsrc], ids[g::nsrc], Qn, k, mo) for g in range(nsrc)]
    Ds = torch.tensor(np.stack([p[0] for p in parts]), dtype=torch.float32).cuda()
    Is = torch.tensor(np.stack([p[1] for p in parts])).cuda()
    D, I = merge_topk(Ds, Is, metric)
    Do, Io = O.merge_topk(parts, k, mo)
    check_topk(D.cpu().numpy(), I.cpu().numpy(), Do, Io, exact=True)


@pytest.mark.slow
def test_c2_full_size_sampled():
    """configs[1] at full size (1M x 128, nlist 4096, nprobe 16, 10k queries, k 10) in the bench's
    launch configuration; the oracle checks a seeded sample of assignments and queries."""
    Index, _ = _mv()
    n, nq = 1_000_000, 10_000
    X = G.sift_base(n, device="cuda")
    Q = G.sift_queries(nq, device="cuda")
    ids = torch.arange(n, dtype=torch.int64, device="cuda")
    C = kmeans(X, 4096, iters=10)
    ix = Index(128, "l2", "flat", 4096)
    ix.set_centroids(C)
    ix.add(X, ids)
    D, I = ix.search(Q, 10, 16)
    torch.cuda.synchronize()
    Xn, Cn = X.cpu().numpy(), C.cpu().numpy()
    oi, gl = oracle_from_gpu_storage(ix, O.L2, O.FLAT, Cn, Xn, ids.cpu().numpy())
    check_assignment(gl, Xn, Cn, O.L2, sample=2000)
    sel = np.random.default_rng(7).choice(nq, 64, replace=False)
    Qs = Q.cpu().numpy()[sel]
    P = ix.search_probes(torch.tensor(Qs).cuda(), 16).cpu().numpy()
    check_probes(P, Qs, Cn, 16, O.L2)
    Do, Io, _ = oi.search(Qs, 10, 16, probes=P)
    check_topk(D.cpu().numpy()[sel], I.cpu().numpy()[sel], Do, Io, exact=True)


OPTION_SETS = [{"seeding": 0}, {"need": 1, "capa": 16}, {"flat_qc": 32, "sq8_qc": 16},
               {"coarse_nqb": 64, "coarse_cs": 3, "coarse_epi": 16, "coarse_nacc": 1},
               {"workspace_bytes": 1 << 20}, {"large_k_select": 1}, {"large_k_select": 2}, {"large_k_select": 3}, {"large_k_select": 4},
               {"seeding": 0, "big_cap": 1100}, {"big_ctas": 4, "big_cap": 700}, {"big_ctas": 1}]


@pytest.mark.parametrize("kind,metric,k", [("flat", "l2", 10), ("flat", "l2", 300), ("flat", "ip", 10),
                                           ("sq8", "l2", 10), ("sq8", "ip", 64)])
def test_options_never_change_results(kind, metric, k):
    """mv_index_set_option picks launch shapes, the seeding sample and the workspace budget (the
    tiny budget forces many query chunks): results are bit-identical to the defaults."""
    X, Q = _sift(12_000, 300, n_micro=512)
    ids = G.permuted_ids(12_000, seed=11)
    C = kmeans(X, 64, iters=4)
    Qd = Q.cuda()
    ix = _build(X, ids, C, metric, kind)
    D0, I0 = ix.search(Qd, k, 6)
    assert ix.describe()["last_chunks"] == 1
    for opts in OPTION_SETS:
        jx = _build(X, ids, C, metric, kind)
        for name, v in opts.items():
            jx.set_option(name, v)
        D1, I1 = jx.search(Qd, k, 6)
        torch.cuda.synchronize()
        assert torch.equal(I0, I1) and torch.equal(D0, D1), opts
        if "workspace_bytes" in opts:
            assert jx.describe()["last_chunks"] > 1
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import MvError
    with pytest.raises(MvError):
        ix.set_option("no_such_option", 1)


def test_cuda_pool_allocator_equals_torch_allocator():
    """mv_allocator routed to torch's caching allocator (default) vs the library's own pools."""
    Index, _ = _mv()
    X, Q = _sift(8000, 64)
    ids = G.permuted_ids(8000, seed=2)
    C = kmeans(X, 32, iters=4)
    out = []
    for alloc in ("torch", None):
        ix = Index(128, "l2", "flat", 32, allocator=alloc)
        ix.set_centroids(C.cuda())
        ix.add(X.cuda(), ids.cuda())
        out.append(ix.search(Q.cuda(), 15, 4))
        assert ix.describe()["allocator"] == ("caller" if alloc else "cuda-pool")
    assert torch.equal(out[0][0], out[1][0]) and torch.equal(out[0][1], out[1][1])


@pytest.mark.parametrize("nprobe", [1, 5, 33, 100])
def test_coarse_exact_ties_follow_centroid_ids(nprobe):
    """Duplicated centroids and integer data: exact score ties everywhere.  The two-pass coarse step
    (group bound, then the keys at or below it) must return exactly the oracle's order -- best
    score first, ties by the smaller centroid id (reading R2)."""
    X, Q = _sift(20_000, 96, n_micro=512)
    base = kmeans(X, 160, iters=3).round()
    C = torch.cat([base, base[:96], base[::3]])          # 309 centroids, many exact duplicates
    Index, _ = _mv()
    ix = Index(128, "l2", "flat", C.shape[0])
    ix.set_centroids(C.cuda())
    P = ix.search_probes(Q.cuda(), nprobe).cpu().numpy()
    Po = O.probe(Q.numpy(), C.numpy(), nprobe, O.L2)
    assert np.array_equal(P, Po)


@pytest.mark.parametrize("nprobe", [200, 700, 1024])
def test_coarse_large_nprobe(nprobe):
    """nprobe up to 1024 on the tensor-core coarse step (k_probe_select R = 8, 32)."""
    X, Q = _sift(30_000, 64)
    Q = Q * 0.93 + 0.21
    C = kmeans(X, 2048, iters=2)
    Index, _ = _mv()
    ix = Index(128, "l2", "flat", 2048)
    ix.set_centroids(C.cuda())
    P = ix.search_probes(Q.cuda(), nprobe).cpu().numpy()
    assert ix.describe()["last_coarse"] == "tcgen05.tf32"
    check_probes(P, Q.numpy(), C.numpy(), nprobe, O.L2)


def test_large_k_select_overflow_mix():
    """k = 2048 with nprobe = 1 over lists of 30k and 8k rows: queries of the long list exceed
    k_final_big's shared-memory stage (~26k keys) and take the global-memory radix select, the
    others stay on k_final_big (the `over` routing of k_select.cu)."""
    r = np.random.default_rng(5)
    cA, cB, cC = (np.full(16, v, np.float32) for v in (40.0, 140.0, 240.0))
    X = np.concatenate([cA + r.integers(-12, 13, (30_000, 16)), cB + r.integers(-12, 13, (8000, 16)),
                        cC + r.integers(-12, 13, (8000, 16))]).astype(np.float32)
    Qn = np.concatenate([cA + r.integers(-6, 7, (6, 16)), cB + r.integers(-6, 7, (6, 16))]).astype(np.float32)
    ids = G.permuted_ids(len(X), seed=8)
    C = torch.tensor(np.stack([cA, cB, cC]))
    ix = _build(torch.tensor(X), ids, C, "l2", "flat")
    off, _, _ = ix.storage()
    assert sorted(np.diff(off).tolist()) == [8000, 8000, 30_000]
    frac, _, _ = _run_conditional(ix, torch.tensor(X), ids, C, torch.tensor(Qn), 2048, 1, O.L2, O.FLAT, exact=True)
    assert frac == 1.0


@pytest.mark.parametrize("kind,metric", [("flat", "l2"), ("sq8", "ip")])
def test_search_with_probes_equals_search(kind, metric):
    """mv_search_with_probes (the multi-GPU query-split coarse step's entry point) with the probes
    mv_search_probes returns gives bit-identical results to mv_search; host probes are staged."""
    X, Q = _sift(12_000, 90)
    ids = G.permuted_ids(12_000, seed=4)
    C = kmeans(X, 96, iters=4)
    ix = _build(X, ids, C, metric, kind)
    Qd = Q.cuda()
    D0, I0 = ix.search(Qd, 20, 9)
    P = ix.search_probes(Qd, 9)
    D1, I1 = ix.search(Qd, 20, 9, probes=P)
    D2, I2 = ix.search(Qd, 20, 9, probes=P.cpu())
    torch.cuda.synchronize()
    assert torch.equal(I0, I1) and torch.equal(D0, D1)
    assert torch.equal(I0, I2) and torch.equal(D0, D2)


@pytest.mark.parametrize("kind,metric,k", [("flat", "l2", 10), ("sq8", "ip", 100), ("flat", "l2", 600)])
@pytest.mark.parametrize("need", ["1", "1000000"])
def test_seeding_sample_size_extremes(kind, metric, k, need):
    """The seeding phase's sample size (DESIGN.md §5 `need`) only changes how tight tau_q is, never
    the result: the 2k floor (loosest bound, most phase-B emissions) and a sample larger than every
    query's candidate set (phase A scans all probed lists) both equal the oracle."""
    if kind == "flat":
        X, Q = _sift(12_000, 60)
        mo, ko = O.L2, O.FLAT
    else:
        X, Q = _deep(12_000, 60)
        mo, ko = O.IP, O.SQ8
    ids = G.permuted_ids(12_000, seed=21)
    C = kmeans(X, 48, iters=4)
    ix = _build(X, ids, C, metric, kind)
    ix.set_option("need", int(need))
    bs = G.mod_bitset(12_000, 10) if kind == "sq8" else None
    frac, _, _ = _run_conditional(ix, X, ids, C, Q, k, 9, mo, ko, bitset=bs, nbits=12_000 if bs is not None else 0)
    assert frac > (0.999 if kind == "sq8" else 0.9999)


@pytest.mark.parametrize("qc", ["16", "32", "64"])
@pytest.mark.parametrize("metric", ["l2", "ip"])
def test_sq8_item_width_and_accumulators(qc, metric):
    """SQ8 work items of 16 / 32 / 64 queries (8 / 4 / 2 TMEM accumulators in flight),
    lists probed by more queries than one item holds, a bitset: same answer as the oracle."""
    X, Q = _sift(16_000, 150, n_micro=1024)
    ids = G.permuted_ids(16_000, seed=17)
    C = kmeans(X, 24, iters=4)
    Index, _ = _mv()
    ix = Index(128, metric, "sq8", 24)
    ix.set_option("sq8_qc", int(qc))
    ix.set_centroids(C.cuda())
    ix.train_sq8(X.cuda())
    ix.add(X.cuda(), ids.cuda())
    bs = G.mod_bitset(16_000, 7)
    mo = O.IP if metric == "ip" else O.L2
    frac, _, _ = _run_conditional(ix, X, ids, C, Q, 20, 5, mo, O.SQ8, bitset=bs, nbits=16_000)
    assert ix.describe()["last_scan"] == "tcgen05.i8"
    assert frac > 0.999


@pytest.mark.parametrize("k", [10, 300])
def test_identity_ids_fast_path(k):
    """Ids exactly 0..n-1 (the selects map a rank to its id without the sorted_ids gather) and a
    shifted copy (the gather) both equal the oracle."""
    n = 15_000
    X, Q = _sift(n, 40)
    C = kmeans(X, 48, iters=4)
    for ids in (torch.arange(n), torch.arange(n) + 7):
        ix = _build(X, ids, C, "l2", "flat")
        frac, _, _ = _run_conditional(ix, X, ids, C, Q, k, 6, O.L2, O.FLAT, exact=True)
        assert frac == 1.0
