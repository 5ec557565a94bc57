"""§8 row a8 on CPU: the sharded search's distributed logic (row ownership, one all-gather, merge in
(distance, id, shard, position) order) with world_size 2 over gloo.  The local per-shard search and
the merge are the oracle's (the CUDA library is exercised by tests/test_gpu_sharded.py); what this
pins is that G shards + exchange + merge == one index, including exact distance ties."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as O
from paper_conf_sigmod_wangygjxlwglxyy21_b200.sharded import ShardedIndex, shard_of


class OracleShard:
    """Test double for the local index: exact search over the rows this rank owns."""

    def __init__(self, metric):
        self.metric = metric
        self.X = np.zeros((0, 0), np.float32)
        self.ids = np.zeros(0, np.int64)

    def set_centroids(self, c):
        pass

    def add(self, x, ids):
        x, ids = x.numpy(), ids.numpy()
        self.X = x if self.X.size == 0 else np.concatenate([self.X, x])
        self.ids = np.concatenate([self.ids, ids])

    def search(self, q, k, nprobe, bitset=None, nbits=None):
        D, I = O.exact_knn(self.X, self.ids, q.numpy(), k, self.metric)
        return torch.tensor(D, dtype=torch.float32), torch.tensor(I)


class OracleIvfShard:
    """Test double for an IVF shard: the oracle's two-step IVF search over this rank's rows, with
    probes computed here (search_probes) or supplied (the query-split coarse step)."""

    def __init__(self, metric, C):
        self.metric = metric
        self.ix = O.IvfIndex(C.shape[1], metric, O.FLAT, C)
        self.nlist = C.shape[0]
        self.calls = []

    def set_centroids(self, c):
        pass

    def add(self, x, ids):
        self.ix.add(x.numpy(), ids.numpy())

    def search_probes(self, q, nprobe):
        self.calls.append(("probes", int(q.shape[0])))
        return torch.tensor(O.probe(q.numpy(), self.ix.C, nprobe, self.metric).astype(np.int32))

    def search(self, q, k, nprobe, bitset=None, nbits=None, probes=None):
        self.calls.append(("search", probes is not None))
        D, I, _ = self.ix.search(q.numpy(), k, nprobe, probes=None if probes is None else probes.numpy())
        return torch.tensor(D, dtype=torch.float32), torch.tensor(I)


def _ivf_worker(rank, world, port, out, nq):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        r = np.random.default_rng(11)
        X = r.integers(0, 40, (1200, 6)).astype(np.float32)
        ids = r.permutation(9000)[:1200].astype(np.int64)
        Q = r.integers(0, 40, (nq, 6)).astype(np.float32)
        C = X[r.permutation(1200)[:24]] + 0.5
        sh = ShardedIndex(OracleIvfShard(O.L2, C), merge=oracle_merge, coarse="split")
        sh.add(torch.tensor(X), torch.tensor(ids))
        D, I = sh.search(torch.tensor(Q), 9, 5)
        m = (nq + world - 1) // world
        assert ("probes", max(0, min(nq, (rank + 1) * m) - min(nq, rank * m))) in sh.local.calls or \
            min(nq, (rank + 1) * m) <= min(nq, rank * m)
        assert ("search", True) in sh.local.calls
        if rank == 0:
            out.put((D.numpy(), I.numpy(), X, ids, Q, C))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,nq", [(2, 31), (3, 20)])
def test_gloo_split_coarse_equals_single_ivf(world, nq):
    """Query-split coarse step: each rank computes the probes of its query slice, one
    all-gather of the probe matrix, local scans with the supplied probes, exchange and merge --
    equal to one IVF index over all rows with the same centroids (oracle, nprobe 5 of 24)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ivf_worker, args=(r, world, port, q, nq)) for r in range(world)]
    for p in procs:
        p.start()
    D, I, X, ids, Q, C = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    ref = O.IvfIndex(6, O.L2, O.FLAT, C)
    ref.add(X, ids)
    De, Ie, _ = ref.search(Q, 9, 5)
    assert np.array_equal(I, Ie)
    assert np.array_equal(D, De.astype(np.float32))


def oracle_merge(gd, gi, metric):
    parts = [(gd[s].double().numpy(), gi[s].numpy()) for s in range(gd.shape[0])]
    D, I = O.merge_topk(parts, gd.shape[2], metric)
    return torch.tensor(D, dtype=torch.float32), torch.tensor(I)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, metric, out, exchange="auto", nq=25, k=37, n=900):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        r = np.random.default_rng(7)
        X = r.integers(0, 6, (n, 4)).astype(np.float32)   # small integers: many exact ties
        ids = r.permutation(6 * n)[:n].astype(np.int64)
        Q = r.integers(0, 6, (nq, 4)).astype(np.float32)
        sh = ShardedIndex(OracleShard(metric), merge=oracle_merge, exchange=exchange)
        sh.set_centroids(torch.zeros(1, 4))
        sh.add(torch.tensor(X), torch.tensor(ids))           # each rank keeps only its own rows
        assert (shard_of(torch.tensor(sh.local.ids), world) == rank).all()
        D, I = sh.search(torch.tensor(Q), k, 1)
        if rank == 0:
            out.put((D.numpy(), I.numpy(), X, ids, Q))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("metric", [O.L2, O.IP])
def test_two_rank_gloo_sharded_equals_single_index(metric):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, metric, q)) for r in range(2)]
    for p in procs:
        p.start()
    D, I, X, ids, Q = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    De, Ie = O.exact_knn(X, ids, Q, 37, metric)
    assert np.array_equal(I, Ie)
    assert np.array_equal(D, De.astype(np.float32))


@pytest.mark.parametrize("world,nq,k,metric", [(2, 25, 37, O.L2), (3, 25, 300, O.L2), (2, 7, 300, O.IP)])
def test_gloo_alltoall_exchange_equals_single_index(world, nq, k, metric):
    """The large-k exchange (query-slice all_to_all, merge of the own slice, all-gather of the merged
    slices) equals one index, with nq not a multiple of the world size and k beyond
    the candidates of some shards (padding entries)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, metric, q, "alltoall", nq, k)) for r in range(world)]
    for p in procs:
        p.start()
    D, I, X, ids, Q = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    De, Ie = O.exact_knn(X, ids, Q, k, metric)
    assert np.array_equal(I, Ie)
    assert np.array_equal(D, De.astype(np.float32))


def test_gloo_eight_ranks_k16384_alltoall():
    """k = 16384 at G = 8 through the all-to-all exchange
    equals one index (nq = 9, not a multiple of 8; every shard holds fewer than k rows)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    world, nq, k, n = 8, 9, 16384, 20000
    procs = [ctx.Process(target=_worker, args=(r, world, port, O.L2, q, "alltoall", nq, k, n)) for r in range(world)]
    for p in procs:
        p.start()
    D, I, X, ids, Q = q.get(timeout=400)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    De, Ie = O.exact_knn(X, ids, Q, k, O.L2)
    assert np.array_equal(I, Ie)
    assert np.array_equal(D, De.astype(np.float32))


def test_shard_of_is_a_partition():
    ids = torch.tensor([0, 1, 2, 3, 10, 11, -5, 2**40 + 3])
    own = shard_of(ids, 4)
    assert ((own >= 0) & (own < 4)).all()
    assert own.tolist() == [0, 1, 2, 3, 2, 3, 3, 3]
