"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (§8(c) step 5).

The oracle checks seeded samples: assignments of sampled rows (equal, or tied within 1e-5), the
probe sets of sampled queries, and their top-k by oracle step O5 over the GPU-accepted lists.
configs[2] (Deep10M SQ8 IP, 10% bitset, k 100), configs[3] (SIFT10M FLAT, nprobe 128, k 2048:
the k_final_big / k_final_select mix), configs[4] (one shard of the 1B SQ8 index, built on the
device; its rows are regenerated from mvgen's counter hash for the oracle).
"""
import numpy as np
import pytest
import torch

import mvgen as G
import oracle as O
from mvgen.kmeans import kmeans

from ._parity import check_assignment, check_probes, check_topk, gpu_lists_of, sampled_oracle_topk

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


def _mv():
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index
    return Index


def _pos_of_dense(sids):
    inv = np.empty(len(sids), np.int64)
    inv[sids] = np.arange(len(sids))
    return lambda ids: inv[ids]


def test_c3_deep10m_sq8_ip_bitset_full_size():
    Index = _mv()
    n, nq, nlist, nprobe, k = 10_000_000, 10_000, 16384, 32, 100
    X = G.deep_base(n, device="cuda")
    Q = G.deep_queries(nq, device="cuda")
    C = kmeans(X, nlist, iters=10, spherical=True)
    bs = G.mod_bitset(n, 10, device="cuda")
    ids = torch.arange(n, dtype=torch.int64, device="cuda")
    samp = torch.randperm(n, generator=torch.Generator().manual_seed(G.SEED_SQ8))[: 64 * nlist].cuda()
    ix = Index(96, "ip", "sq8", nlist)
    ix.set_centroids(C)
    ix.train_sq8(X[samp])
    ix.add(X, ids)
    D, I = ix.search(Q, k, nprobe, bitset=bs, nbits=n)
    torch.cuda.synchronize()
    Xn, Cn, bsn = X.cpu().numpy(), C.cpu().numpy(), bs.cpu().numpy()
    sq8 = ix.get_sq8()
    off, sids, _ = ix.storage()
    lists = np.repeat(np.arange(nlist), np.diff(off))
    gl = np.empty(n, np.int64)
    gl[sids] = lists
    check_assignment(gl, Xn, Cn, O.IP, sample=2000)
    # SQ8 params of the training sample, codes of sampled rows: bit-exact with the oracle codec
    ov, od = O.sq8_train(Xn[samp.cpu().numpy()])
    assert np.array_equal(sq8[0], ov) and np.array_equal(sq8[1], od)
    sel = np.random.default_rng(7).choice(nq, 64, replace=False)
    Qs = Q.cpu().numpy()[sel]
    P = ix.search_probes(torch.tensor(Qs).cuda(), nprobe).cpu().numpy()
    check_probes(P, Qs, Cn, nprobe, O.IP)
    Do, Io, cm = sampled_oracle_topk(Qs, P, off, sids, lambda c: Xn[c], O.IP, O.SQ8, k, sq8=sq8, bitset=bsn, nbits=n)
    frac = check_topk(D.cpu().numpy()[sel], I.cpu().numpy()[sel], Do, Io, cm, atol=2e-6)
    assert frac > 0.999


def test_c4_sift10m_flat_k2048_full_size():
    Index = _mv()
    n, nq, nlist, nprobe, k = 10_000_000, 10_000, 16384, 128, 2048
    X = G.sift_base(n, device="cuda")
    Q = G.sift_queries(nq, device="cuda")
    C = kmeans(X, nlist, iters=10)
    ix = Index(128, "l2", "flat", nlist)
    ix.set_centroids(C)
    ix.add(X, torch.arange(n, dtype=torch.int64, device="cuda"))
    D, I = ix.search(Q, k, nprobe)
    torch.cuda.synchronize()
    Xn, Cn = X.cpu().numpy(), C.cpu().numpy()
    off, sids, _ = ix.storage()
    lens = np.diff(off)
    # the production select mix: the worst-case candidate bound exceeds k_final_big's stage
    assert np.sort(lens)[::-1][:nprobe].sum() > 26_000
    lists = np.repeat(np.arange(nlist), lens)
    gl = np.empty(n, np.int64)
    gl[sids] = lists
    check_assignment(gl, Xn, Cn, O.L2, sample=2000)
    sel = np.random.default_rng(11).choice(nq, 16, replace=False)
    Qs = Q.cpu().numpy()[sel]
    P = ix.search_probes(torch.tensor(Qs).cuda(), nprobe).cpu().numpy()
    check_probes(P, Qs, Cn, nprobe, O.L2)
    Do, Io, cm = sampled_oracle_topk(Qs, P, off, sids, lambda c: Xn[c], O.L2, O.FLAT, k)
    frac = check_topk(D.cpu().numpy()[sel], I.cpu().numpy()[sel], Do, Io, cm)
    assert frac == 1.0 or frac > 0.9999


def test_c5_shard_sift1b_sq8_sampled_protocol():
    """configs[4]: shard 3 of 8 of the 1B-row SIFT-shaped IVF_SQ8 index (125M rows, nlist 65536),
    built on the device chunk by chunk exactly as bench.py does.  The oracle cannot hold the
    shard: the sampled protocol of SURVEY §8(c) step 5 -- assignments of 1000 sampled rows
    regenerated from the counter hash, probe sets and top-10 of 48 sampled queries over the
    GPU's lists with the rows regenerated (and re-encoded by the oracle codec)."""
    import bench
    Index = _mv()
    cfg = dict(bench.CONFIGS["c5"])
    shard, nshard = 3, 8
    dev = torch.device("cuda", 0)
    ix, Q, C, _, nloc = bench.build_sharded(cfg, dev, shard, nshard, Index, ngt=0)
    k, nprobe = cfg["k"], cfg["nprobe"]
    D, I = ix.search(Q, k, nprobe)
    torch.cuda.synchronize()
    spec = bench.c5_spec(128)
    Cn = C.cpu().numpy()
    off, sids, _ = ix.storage()
    assert len(sids) == nloc and np.all(sids % nshard == shard)
    inv = np.empty(nloc, np.int64)
    inv[(sids - shard) // nshard] = np.arange(nloc)
    pos_of = lambda ids: inv[(ids - shard) // nshard]  # noqa: E731

    def rows_of(ids):
        return spec.rows_at(torch.as_tensor(ids, dtype=torch.int64, device="cuda"), G.SEED_BASE).cpu().numpy()

    r = np.random.default_rng(3)
    samp = r.choice(nloc, 1000, replace=False) * nshard + shard
    gl = gpu_lists_of(samp, off, pos_of)
    ol = O.assign(rows_of(samp), Cn, O.L2)
    for i in np.nonzero(ol != gl)[0]:
        s = O.distances(rows_of(samp[i:i + 1])[0], Cn[[ol[i], gl[i]]], O.L2)
        assert abs(s[0] - s[1]) <= 1e-5 * abs(s[0]), (samp[i], s)
    sq8 = ix.get_sq8()
    sel = r.choice(Q.shape[0], 48, replace=False)
    Qs = Q.cpu().numpy()[sel]
    P = ix.search_probes(torch.tensor(Qs).cuda(), nprobe).cpu().numpy()
    check_probes(P, Qs, Cn, nprobe, O.L2)
    Do, Io, cm = sampled_oracle_topk(Qs, P, off, sids, rows_of, O.L2, O.SQ8, k, sq8=sq8)
    frac = check_topk(D.cpu().numpy()[sel], I.cpu().numpy()[sel], Do, Io, cm)
    assert frac > 0.999
