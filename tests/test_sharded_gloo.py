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


def _worker(rank, world, port, metric, out, exchange="auto", nq=25, k=37):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        r = np.random.default_rng(7)
        X = r.integers(0, 6, (900, 4)).astype(np.float32)   # small integers: many exact ties
        ids = r.permutation(5000)[:900].astype(np.int64)
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


def test_shard_of_is_a_partition():
    ids = torch.tensor([0, 1, 2, 3, 10, 11, -5, 2**40 + 3])
    own = shard_of(ids, 4)
    assert ((own >= 0) & (own < 4)).all()
    assert own.tolist() == [0, 1, 2, 3, 2, 3, 3, 3]
