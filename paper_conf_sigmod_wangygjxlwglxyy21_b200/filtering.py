"""the two workloads the paper runs on top of the vector hot path, built on
the unchanged a2-a8 search (Index.search, mv_merge_topk) plus two small kernels of libmv
(mv_attr_bitset, mv_fuse_rows).  The binding only routes tensors: every step that computes runs
in libmv.

* PartitionedIndex -- strategy E, partition-based attribute filtering (§4.1):
  the rows are partitioned by the value range of a frequently searched attribute, one IVF index
  per partition over shared centroids; a query batch with the constraint lo <= attr <= hi
  searches only the partitions whose range overlaps [lo, hi]; a covered partition is searched
  without any attribute check; a partly covered one with strategy B's bitmap,
  built on the device by mv_attr_bitset (reading R16: strategy D's cost model is not modelled);
  the partitions' top-k lists are merged on the device (mv_merge_topk).
* MultiVectorIndex -- multi-vector queries by vector fusion (§4.2): an entity's
  mu vectors are stored concatenated; a query entity's vectors are scaled by the weighted-sum
  aggregation's weights and concatenated (mv_fuse_rows), and one inner-product search returns the
  top-k entities by sum_i w_i (q.v_i . e.v_i) -- "the similarity function of inner product is
  decomposable".
"""
from __future__ import annotations

import ctypes as C

import torch

from . import _lib as L
from .index import Index, _torch_stream, merge_topk


def partition_plan(ranges, lo: int, hi: int) -> list[str]:
    """Per partition [plo, phi]: 'skip' (no overlap with [lo, hi]), 'covered' (lo <= plo and
    phi <= hi: no attribute check) or 'check' (strategy B's bitmap)."""
    plan = []
    for plo, phi in ranges:
        if phi < lo or plo > hi:
            plan.append("skip")
        elif lo <= plo and phi <= hi:
            plan.append("covered")
        else:
            plan.append("check")
    return plan


class PartitionedIndex:
    """Strategy E over disjoint inclusive attribute ranges [(lo_0, hi_0), ...] (int64 attribute)."""

    def __init__(self, d: int, ranges, metric="l2", kind="flat", nlist: int = 1, device: int | None = None):
        self.ranges = [(int(a), int(b)) for a, b in ranges]
        for (a0, b0), (a1, b1) in zip(sorted(self.ranges), sorted(self.ranges)[1:]):
            if a1 <= b0:
                raise ValueError("partition ranges must be disjoint")
        self.metric = metric
        self.parts = [Index(d, metric, kind, nlist, device=device) for _ in self.ranges]
        self.device = self.parts[0].device
        dev = torch.device("cuda", self.device)
        self._ids = [torch.empty(0, dtype=torch.int64, device=dev) for _ in self.ranges]
        self._attr = [torch.empty(0, dtype=torch.int64, device=dev) for _ in self.ranges]
        self.last_plan: list[str] = []

    def set_centroids(self, c):
        for p in self.parts:
            p.set_centroids(c)

    def set_sq8(self, vmin, vdiff):
        for p in self.parts:
            p.set_sq8(vmin, vdiff)

    def train_sq8(self, sample):
        self.parts[0].train_sq8(sample)
        vmin, vdiff = self.parts[0].get_sq8()
        for p in self.parts[1:]:
            p.set_sq8(vmin, vdiff)

    @property
    def ntotal(self) -> int:
        return sum(p.ntotal for p in self.parts)

    def add(self, x: torch.Tensor, ids: torch.Tensor, attr: torch.Tensor):
        """Route each row to the partition whose range holds its attribute (the add path)."""
        dev = torch.device("cuda", self.device)
        x, ids, attr = x.to(dev), ids.to(dev, torch.int64), attr.to(dev, torch.int64)
        placed = torch.zeros(attr.shape[0], dtype=torch.bool, device=dev)
        for j, (lo, hi) in enumerate(self.ranges):
            m = (attr >= lo) & (attr <= hi)
            placed |= m
            if bool(m.any()):
                self.parts[j].add(x[m], ids[m])
                self._ids[j] = torch.cat([self._ids[j], ids[m]])
                self._attr[j] = torch.cat([self._attr[j], attr[m]])
        if not bool(placed.all()):
            raise ValueError("some attribute values lie in no partition range")

    def search(self, q, k: int, nprobe: int, lo: int, hi: int, stream=None):
        """Top-k under lo <= attr <= hi: (D[nq,k] float32, I[nq,k] int64)."""
        lib = L.load()
        s = _torch_stream(self.device, stream)
        plan = partition_plan(self.ranges, int(lo), int(hi))
        self.last_plan = plan
        dev = torch.device("cuda", self.device)
        nq = int(q.shape[0])
        Ds, Is = [], []
        with torch.cuda.stream(s):
            for j, how in enumerate(plan):
                if how == "skip" or self.parts[j].ntotal == 0:
                    continue
                if how == "covered":
                    D, I = self.parts[j].search(q, k, nprobe, stream=s)
                else:
                    ids, attr = self._ids[j], self._attr[j]
                    nbits = int(ids.max().item()) + 1
                    bitset = torch.empty(((nbits + 31) // 32) * 4, dtype=torch.uint8, device=dev)
                    L.check(lib.mv_attr_bitset(C.c_void_p(ids.data_ptr()), C.c_void_p(attr.data_ptr()),
                                               int(ids.shape[0]), int(lo), int(hi), C.c_void_p(bitset.data_ptr()),
                                               nbits, C.c_void_p(s.cuda_stream)))
                    D, I = self.parts[j].search(q, k, nprobe, bitset=bitset, nbits=nbits, stream=s)
                Ds.append(D)
                Is.append(I)
            if not Ds:
                pad = float("inf") if str(self.metric).lower() in ("l2", "0") else float("-inf")
                return (torch.full((nq, k), pad, dtype=torch.float32, device=dev),
                        torch.full((nq, k), -1, dtype=torch.int64, device=dev))
            if len(Ds) == 1:
                return Ds[0], Is[0]
            return merge_topk(torch.stack(Ds), torch.stack(Is), self.metric, stream=s)


def fuse_rows(parts, weights=None, stream=None) -> torch.Tensor:
    """mv_fuse_rows: [w_0 parts[0] | w_1 parts[1] | ...] row by row (device fp32)."""
    lib = L.load()
    parts = [p.contiguous().float() for p in parts]
    n = int(parts[0].shape[0])
    if any(int(p.shape[0]) != n for p in parts):
        raise ValueError("every part needs the same number of rows")
    dev = parts[0].device
    s = _torch_stream(dev.index, stream)
    dims = [int(p.shape[1]) for p in parts]
    out = torch.empty((n, sum(dims)), dtype=torch.float32, device=dev)
    ptrs = (C.c_void_p * len(parts))(*[p.data_ptr() for p in parts])
    dd = (C.c_int32 * len(parts))(*dims)
    ww = (C.c_float * len(parts))(*[float(w) for w in weights]) if weights is not None else None
    L.check(lib.mv_fuse_rows(ptrs, dd, ww, len(parts), n, C.c_void_p(out.data_ptr()), C.c_void_p(s.cuda_stream)))
    return out


class MultiVectorIndex:
    """Vector fusion over entities of mu vectors with dimensions `dims`, aggregated by a weighted
    sum of inner products: one MV_IP IVF index over the concatenated vectors."""

    def __init__(self, dims, kind="flat", nlist: int = 1, device: int | None = None):
        self.dims = [int(x) for x in dims]
        self.index = Index(sum(self.dims), "ip", kind, nlist, device=device)

    def fuse(self, parts, weights=None, stream=None) -> torch.Tensor:
        if [int(p.shape[1]) for p in parts] != self.dims:
            raise ValueError(f"parts must have dimensions {self.dims}")
        return fuse_rows(parts, weights, stream)

    def set_centroids(self, c):
        """Centroids of the fused space ([nlist, sum dims])."""
        self.index.set_centroids(c)

    def train_sq8(self, parts):
        self.index.train_sq8(self.fuse(parts))

    def add(self, parts, ids):
        self.index.add(self.fuse(parts), ids)

    def search(self, q_parts, weights, k: int, nprobe: int, bitset=None, nbits: int | None = None, stream=None):
        """Top-k entities by sum_i w_i (q.v_i . e.v_i) (larger is better)."""
        return self.index.search(self.fuse(q_parts, weights, stream), k, nprobe, bitset=bitset, nbits=nbits,
                                 stream=stream)
