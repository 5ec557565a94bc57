"""§8 row a8 on the GPU: G vector shards searched independently and merged on device with
mv_merge_topk give bit-identical ids and distances to one index over all rows (G-invariance),
for FLAT (exact integer data) and SQ8, L2 and IP."""
import pytest
import torch

import mvgen as G
from mvgen.kmeans import kmeans

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("kind,metric", [("flat", "l2"), ("flat", "ip"), ("sq8", "l2")])
@pytest.mark.parametrize("nshard", [2, 3, 8])
def test_g_shards_equal_one_index(kind, metric, nshard):
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index, merge_topk
    from paper_conf_sigmod_wangygjxlwglxyy21_b200.sharded import shard_of
    spec = G.SiftSpec(d=128, n_micro=1024)
    X = G.sift_base(24_000, spec=spec).cuda()
    Q = G.sift_queries(200, spec=spec).cuda()
    ids = G.permuted_ids(24_000, seed=21).cuda()
    C = kmeans(X.cpu(), 64, iters=4).cuda()

    def build(sel):
        ix = Index(128, metric, kind, 64)
        ix.set_centroids(C)
        if kind == "sq8":
            ix.set_sq8(X.min(0).values, X.max(0).values - X.min(0).values)
        ix.add(X[sel], ids[sel])
        return ix

    one = build(torch.ones(24_000, dtype=torch.bool, device="cuda"))
    D1, I1 = one.search(Q, 20, 8)
    parts = [build(shard_of(ids, nshard) == g).search(Q, 20, 8) for g in range(nshard)]
    D, I = merge_topk(torch.stack([p[0] for p in parts]), torch.stack([p[1] for p in parts]), metric)
    torch.cuda.synchronize()
    assert torch.equal(I, I1)
    assert torch.equal(D, D1)


@pytest.mark.parametrize("exchange,coarse,k", [("allgather", "replicated", 20), ("alltoall", "split", 300),
                                               ("alltoall", "replicated", 2048)])
def test_nccl_exchange_paths_on_one_gpu(exchange, coarse, k):
    """The NCCL code of ShardedIndex (all_gather_into_tensor, all_to_all_single, the query-split
    coarse step's probe all-gather) on hardware: a one-rank NCCL group (the box has one GPU) must
    return exactly the local index's result."""
    import os
    import socket
    import torch.distributed as dist
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index
    from paper_conf_sigmod_wangygjxlwglxyy21_b200.sharded import ShardedIndex
    spec = G.SiftSpec(d=128, n_micro=1024)
    X = G.sift_base(20_000, spec=spec).cuda()
    Q = G.sift_queries(150, spec=spec).cuda()
    ids = G.permuted_ids(20_000, seed=3).cuda()
    C = kmeans(X.cpu(), 48, iters=4).cuda()
    ix = Index(128, "l2", "flat", 48)
    ix.set_centroids(C)
    ix.add(X, ids)
    D1, I1 = ix.search(Q, k, 6)
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        sh = ShardedIndex(ix, exchange=exchange, coarse=coarse)
        D, I = sh.search(Q, k, 6)
        torch.cuda.synchronize()
        assert dist.get_backend() == "nccl"
        assert torch.equal(I, I1) and torch.equal(D, D1)
    finally:
        dist.destroy_process_group()
