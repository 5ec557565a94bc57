"""Vector (segment) sharding over the ranks of a torch.distributed process group -- §8 row a8.

PAPER.md:773-776 (§3.3): "each segment can only be served by a single GPU device"
(§5.3): data are sharded across readers and results merged.  Here row r lives on rank ``id % G``;
every rank holds all nlist lists over its own rows (list sizes are ~1/G of the global ones, so the
per-list load stays balanced); centroids and SQ8 parameters are replicated.  A search runs the local
hot path on every rank (mv_search), exchanges the per-shard top-k with ONE all-gather over NCCL
(NVLink/NVSwitch), and merges on device with mv_merge_topk -- every rank ends with the same result.

The exchange is the only collective step; there is no per-step synchronisation besides it.  Merge
order is (distance, id, shard, position) -- identical to the single-index order whenever ids are
unique, so results are G-invariant (tested).

Two exchanges:
  * "allgather" (small k): every rank receives all G local top-k lists, (G-1) x nq x k x 12 B, and
    merges all nq queries;
  * "alltoall" (large k, e.g. k = 2048, where the all-gather would move (G-1) x 246 MB per rank at
    nq = 10k): rank r owns the query slice [r*m, (r+1)*m), m = ceil(nq / G); one all_to_all sends
    every slice to its owner ((G-1)/G of the local result), the owner merges its m queries from G
    sources, and one all-gather of the merged slices gives every rank the full result -- 2 (G-1)/G
    x nq x k x 12 B per rank instead of (G-1) x nq x k x 12 B, and 1/G of the merge work.
  The default picks "alltoall" when k >= 256.

Coarse step (a2/a3): "replicated" (every rank computes all nq probe lists; cheap for small nlist)
or "split" (rank r computes the probes of its query slice and one all-gather of the int32
[nq, nprobe] probe matrix gives every rank all of them -- 2.56 MB at nq = 10k, nprobe = 64 --
then the local scan takes them through mv_search_with_probes).  The default splits when
nq * nlist >= 2^28 (configs[4]: 10k x 65,536, a 2.6 GB score matrix per rank if replicated).

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
    def __init__(self, local, group=None, merge: Callable | None = None, exchange: str = "auto",
                 coarse: str = "auto"):
        """local: an object with .search(q, k, nprobe, bitset=None, nbits=None) -> (D[nq,k], I[nq,k])
        and .add(x, ids); group: a torch.distributed process group (None = default);
        merge(D[G,nq,k], I[G,nq,k], metric) -> (D, I) (default: mv_merge_topk on device);
        exchange: "allgather", "alltoall" or "auto" (alltoall for k >= 256);
        coarse: "replicated", "split" or "auto" (split when nq * nlist >= 2^28)."""
        if exchange not in ("auto", "allgather", "alltoall"):
            raise ValueError(f"unknown exchange {exchange!r}")
        if coarse not in ("auto", "replicated", "split"):
            raise ValueError(f"unknown coarse mode {coarse!r}")
        self.exchange = exchange
        self.coarse = coarse
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
        nlist = int(getattr(self.local, "nlist", 1))
        # an explicit mode runs its collectives at any world size (world 1 included: the NCCL path
        # on a single GPU, tests/test_gpu_sharded.py); "auto" skips them when there is no peer
        split = dist.is_initialized() and (self.coarse == "split" or (
            self.coarse == "auto" and self.world > 1 and q.shape[0] * nlist >= (1 << 28)))
        if split:
            P = self._split_probes(q, nprobe, nlist)
            D, I = self.local.search(q, k, nprobe, bitset=bitset, nbits=nbits, probes=P)
        else:
            D, I = self.local.search(q, k, nprobe, bitset=bitset, nbits=nbits)
        if self.world == 1 and (self.exchange == "auto" or not dist.is_initialized()):
            return D, I
        mode = self.exchange if self.exchange != "auto" else ("alltoall" if k >= 256 else "allgather")
        if mode == "alltoall":
            return self._exchange_alltoall(D, I)
        gd, gi = self._all_gather(D), self._all_gather(I)
        return self.merge(gd, gi, self.metric)

    def _split_probes(self, q: torch.Tensor, nprobe: int, nlist: int) -> torch.Tensor:
        """Query-split coarse step: probes of the rank's slice [r*m, (r+1)*m), one all-gather."""
        G, nq = self.world, int(q.shape[0])
        m = (nq + G - 1) // G
        lo, hi = min(nq, self.rank * m), min(nq, (self.rank + 1) * m)
        npb = min(int(nprobe), nlist)
        mine = torch.zeros((m, npb), dtype=torch.int32, device=q.device)  # padding rows: bucket 0
        if hi > lo:
            mine[: hi - lo] = self.local.search_probes(q[lo:hi].contiguous(), nprobe)
        return self._all_gather(mine).reshape(G * m, npb)[:nq].contiguous()

    def _pad_value(self):
        # the padding convention of the library (R3): id -1, +inf (L2) / -inf (IP)
        return float("-inf") if self.metric in (1, "ip") else float("inf")

    def _exchange_alltoall(self, D: torch.Tensor, I: torch.Tensor):
        """Query-slice exchange: all_to_all of the local top-k by owner slice, merge of the own
        slice's G lists, all-gather of the merged slices.  Rows past nq are padding."""
        G, nq, k = self.world, D.shape[0], D.shape[1]
        m = (nq + G - 1) // G
        if m * G != nq:
            D = torch.cat([D, torch.full((m * G - nq, k), self._pad_value(), dtype=D.dtype, device=D.device)])
            I = torch.cat([I, torch.full((m * G - nq, k), -1, dtype=I.dtype, device=I.device)])
        # send block g = rows [g*m, (g+1)*m) to rank g; receive block s = rank s's rows of my slice
        rd, ri = torch.empty_like(D), torch.empty_like(I)
        dist.all_to_all_single(rd, D.contiguous(), group=self.group)
        dist.all_to_all_single(ri, I.contiguous(), group=self.group)
        md, mi = self.merge(rd.view(G, m, k), ri.view(G, m, k), self.metric)   # my m queries
        gd, gi = self._all_gather(md.contiguous()), self._all_gather(mi.contiguous())
        return gd.reshape(G * m, k)[:nq], gi.reshape(G * m, k)[:nq]

    def _all_gather(self, t: torch.Tensor) -> torch.Tensor:
        out = torch.empty((self.world, *t.shape), dtype=t.dtype, device=t.device)
        if dist.get_backend(self.group) == "nccl":
            dist.all_gather_into_tensor(out, t.contiguous(), group=self.group)
        else:
            dist.all_gather(list(out.unbind(0)), t.contiguous(), group=self.group)
        return out
