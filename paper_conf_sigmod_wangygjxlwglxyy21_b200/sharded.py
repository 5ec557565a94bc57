"""Vector (segment) sharding over the ranks of a torch.distributed process group -- §8 row a8.

PAPER.md:773-776 (§3.3): "each segment can only be served by a single GPU device"
(§5.3): data are sharded across readers and results merged.  Here row r lives on rank ``id % G``;
every rank holds all nlist lists over its own rows (list sizes are ~1/G of the global ones, so the
per-list load stays balanced); centroids and SQ8 parameters are replicated.  A search runs the local
hot path on every rank (mv_search), exchanges the per-shard top-k with ONE all-gather over NCCL
(NVLink/NVSwitch), and merges on device with mv_merge_topk -- every rank ends with the same result.

The exchange is the only collective; there is no per-step synchronisation besides it.  Merge order is
(distance, id, shard, position) -- identical to the single-index order whenever ids are unique, so
results are G-invariant (tested).

The local index and the merge are injectable so that the distributed logic can be tested with the
gloo backend on CPU (tests/test_sharded_gloo.py); the product path uses the CUDA library.
"""
from __future__ import annotations

from typing import Callable

import torch
import torch.distributed as dist


def shard_of(ids: torch.Tensor, world: int) -> torch.Tensor:
    """Owner rank of each id (ids are int64, any values)."""
    return torch.remainder(ids, world)


class ShardedIndex:
    def __init__(self, local, group=None, merge: Callable | None = None):
        """local: an object with .search(q, k, nprobe, bitset=None, nbits=None) -> (D[nq,k], I[nq,k])
        and .add(x, ids); group: a torch.distributed process group (None = default);
        merge(D[G,nq,k], I[G,nq,k], metric) -> (D, I) (default: mv_merge_topk on device)."""
        self.local = local
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        if merge is None:
            from .index import merge_topk
            merge = merge_topk
        self.merge = merge
        self.metric = getattr(local, "metric", 0)

    @classmethod
    def create(cls, d: int, metric="l2", kind="flat", nlist: int = 1, group=None, device: int | None = None):
        from .index import Index
        return cls(Index(d, metric, kind, nlist, device=device), group=group)

    # -- build: replicated parameters, sharded rows --------------------------------------------
    def set_centroids(self, c: torch.Tensor):
        """Centroids must be identical on every rank: rank 0's copy is broadcast."""
        c = c.contiguous()
        if self.world > 1:
            dist.broadcast(c, src=0, group=self.group)
        self.local.set_centroids(c)

    def set_sq8(self, vmin: torch.Tensor, vdiff: torch.Tensor):
        vmin, vdiff = vmin.contiguous(), vdiff.contiguous()
        if self.world > 1:
            dist.broadcast(vmin, src=0, group=self.group)
            dist.broadcast(vdiff, src=0, group=self.group)
        self.local.set_sq8(vmin, vdiff)

    def add(self, x: torch.Tensor, ids: torch.Tensor):
        """Add the rows this rank owns (the caller may pass the full batch or only its share)."""
        mine = shard_of(ids, self.world) == self.rank
        if not bool(mine.all()):
            x, ids = x[mine].contiguous(), ids[mine].contiguous()
        if ids.numel():
            self.local.add(x, ids)

    # -- search: local top-k, one all-gather, on-device merge -----------------------------------
    def search(self, q: torch.Tensor, k: int, nprobe: int, bitset=None, nbits: int | None = None):
        D, I = self.local.search(q, k, nprobe, bitset=bitset, nbits=nbits)
        if self.world == 1:
            return D, I
        gd, gi = self._all_gather(D), self._all_gather(I)
        return self.merge(gd, gi, self.metric)

    def _all_gather(self, t: torch.Tensor) -> torch.Tensor:
        out = torch.empty((self.world, *t.shape), dtype=t.dtype, device=t.device)
        if dist.get_backend(self.group) == "nccl":
            dist.all_gather_into_tensor(out, t.contiguous(), group=self.group)
        else:
            dist.all_gather(list(out.unbind(0)), t.contiguous(), group=self.group)
        return out
