"""Thin Python binding over the C ABI (include/mv.h): argument marshalling only.

Tensors are passed as raw pointers (device tensors stay on the device; CPU tensors / numpy arrays
are staged by the library itself).  Every step of the search runs in libmv's CUDA kernels; torch
only provides device memory (the library's mv_allocator is routed to torch's caching allocator),
the current stream and process groups.
"""
from __future__ import annotations

import atexit
import contextlib
import ctypes as C
import weakref

import numpy as np
import torch

from . import _lib as L


def _ptr(x):
    if x is None:
        return None
    if isinstance(x, torch.Tensor):
        return C.c_void_p(x.data_ptr())
    if isinstance(x, np.ndarray):
        return C.c_void_p(x.ctypes.data)
    raise TypeError(f"unsupported buffer type {type(x)}")


def _as_f32(x):
    if isinstance(x, torch.Tensor):
        x = x.contiguous()
        if x.dtype != torch.float32:
            x = x.float()
        return x
    return np.ascontiguousarray(x, dtype=np.float32)


def _as_i64(x):
    if isinstance(x, torch.Tensor):
        return x.contiguous().to(torch.int64)
    return np.ascontiguousarray(x, dtype=np.int64)


def _torch_stream(device: int, stream=None) -> torch.cuda.Stream:
    if stream is None:
        return torch.cuda.current_stream(device)
    if isinstance(stream, torch.cuda.Stream):
        return stream
    return torch.cuda.ExternalStream(int(stream), device=device)


# ---- mv_allocator -> torch's caching allocator ------------------------------------------------
# Blocks are taken on the library's stream, so torch reuses them only in that stream's order
# (the library frees its scratch stream-ordered at the end of each call).
@L.ALLOC_FN
def _torch_alloc(nbytes, stream, ctx):
    try:
        return torch.cuda.caching_allocator_alloc(int(nbytes), device=int(ctx or 0), stream=int(stream or 0))
    except Exception:  # reported to the caller as MV_ENOMEM
        return None


@L.FREE_FN
def _torch_free(ptr, stream, ctx):
    try:
        torch.cuda.caching_allocator_delete(int(ptr))
    except Exception:
        pass


_LIVE = weakref.WeakSet()


@atexit.register
def _close_all():  # destroy indexes while torch's allocator is still alive
    for ix in list(_LIVE):
        try:
            ix.close()
        except Exception:
            pass


METRICS = {"l2": L.MV_L2, "ip": L.MV_IP, L.MV_L2: L.MV_L2, L.MV_IP: L.MV_IP}
TYPES = {"flat": L.MV_IVF_FLAT, "ivf_flat": L.MV_IVF_FLAT, "sq8": L.MV_IVF_SQ8, "ivf_sq8": L.MV_IVF_SQ8,
         "pq": L.MV_IVF_PQ, "ivf_pq": L.MV_IVF_PQ,
         L.MV_IVF_FLAT: L.MV_IVF_FLAT, L.MV_IVF_SQ8: L.MV_IVF_SQ8, L.MV_IVF_PQ: L.MV_IVF_PQ}


class Index:
    """mv_index_create(d, metric, type, nlist) and friends (§3.2.1).

    allocator: "torch" (default: every device allocation of the library goes through torch's
    caching allocator) or None (the library's own cudaMalloc / stream-ordered pool)."""

    def __init__(self, d: int, metric="l2", kind="flat", nlist: int = 1, device: int | None = None,
                 allocator: str | None = "torch"):
        self._lib = L.load()
        self.d, self.nlist = int(d), int(nlist)
        self.metric = METRICS[metric.lower() if isinstance(metric, str) else metric]
        self.kind = TYPES[kind.lower() if isinstance(kind, str) else kind]
        self.device = torch.cuda.current_device() if device is None else int(device)
        self._alloc = None
        if allocator == "torch":
            self._alloc = L.MvAllocator(_torch_alloc, _torch_free, C.c_void_p(self.device))
        elif allocator is not None:
            raise ValueError(f"unknown allocator {allocator!r}")
        h = C.c_void_p()
        L.check(self._lib.mv_index_create(self.d, self.metric, self.kind, self.nlist, self.device,
                                          C.byref(self._alloc) if self._alloc is not None else None, C.byref(h)))
        self._h = h
        _LIVE.add(self)

    # -- lifecycle -----------------------------------------------------------------------------
    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            self._lib.mv_index_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def ntotal(self) -> int:
        return int(self._lib.mv_index_ntotal(self._h))

    def set_option(self, name: str, value: int):
        """mv_index_set_option: launch-shape / sample / workspace tuning (never changes results)."""
        L.check(self._lib.mv_index_set_option(self._h, name.encode(), int(value)))

    # -- build -------------------------------------------------------------------------------
    def set_centroids(self, c):
        c = _as_f32(c)
        L.check(self._lib.mv_index_set_centroids(self._h, _ptr(c)))

    def train_sq8(self, sample):
        s = _as_f32(sample)
        L.check(self._lib.mv_index_train_sq8(self._h, _ptr(s), int(s.shape[0])))

    def set_sq8(self, vmin, vdiff):
        a, b = _as_f32(vmin), _as_f32(vdiff)
        L.check(self._lib.mv_index_set_sq8(self._h, _ptr(a), _ptr(b)))

    def set_pq(self, M: int, codebooks):
        """IVF_PQ sub-centroids [M, 256, d / M]."""
        cb = _as_f32(codebooks)
        L.check(self._lib.mv_index_set_pq(self._h, int(M), _ptr(cb)))
        self.pq_m = int(M)

    def train_pq(self, M: int, sample, niter: int = 10):
        """Per-sub-space k-means (mv_kmeans) over a device sample [n, d], n >= 256."""
        s = _as_f32(sample)
        L.check(self._lib.mv_index_train_pq(self._h, int(M), _ptr(s), int(s.shape[0]), int(niter)))
        self.pq_m = int(M)

    def get_pq(self):
        m = C.c_int32()
        L.check(self._lib.mv_index_get_pq(self._h, C.byref(m), None))
        cb = np.empty((m.value, 256, self.d // m.value), np.float32)
        L.check(self._lib.mv_index_get_pq(self._h, None, _ptr(cb)))
        return cb

    def get_sq8(self):
        vmin = np.empty(self.d, np.float32)
        vdiff = np.empty(self.d, np.float32)
        L.check(self._lib.mv_index_get_sq8(self._h, _ptr(vmin), _ptr(vdiff)))
        return vmin, vdiff

    def _on(self, stream):
        """(torch stream, context manager making it current): temporaries made by the binding are
        then allocated in the same stream order as the library's work."""
        s = _torch_stream(self.device, stream)
        return s, (torch.cuda.stream(s) if stream is not None else contextlib.nullcontext())

    def add(self, x, ids, stream=None):
        s, ctx = self._on(stream)
        with ctx:
            x = _as_f32(x)
            ids = _as_i64(ids)
            n = int(x.shape[0])
            if int(ids.shape[0]) != n:
                raise ValueError("ids and vectors differ in length")
            L.check(self._lib.mv_index_add(self._h, _ptr(x), _ptr(ids), n, C.c_void_p(s.cuda_stream)))

    # -- search ------------------------------------------------------------------------------
    def search(self, q, k: int, nprobe: int, bitset=None, nbits: int | None = None, out=None, stream=None,
               probes=None):
        """Returns (D[nq,k] float32, I[nq,k] int64) on the index device (or into `out`).
        probes: optional int32 [nq, min(nprobe, nlist)] best-first buckets per query (as
        search_probes returns them); the coarse step is then skipped (mv_search_with_probes)."""
        s, ctx = self._on(stream)
        with ctx:
            q = _as_f32(q)
            nq = int(q.shape[0])
            if out is None:
                dev = torch.device("cuda", self.device)
                D = torch.empty((nq, k), dtype=torch.float32, device=dev)
                I = torch.empty((nq, k), dtype=torch.int64, device=dev)
            else:
                D, I = out
            nb = 0
            if bitset is not None:
                nb = int(nbits) if nbits is not None else int(bitset.shape[0]) * 8
            sp = C.c_void_p(s.cuda_stream)
            if probes is not None:
                npb = min(int(nprobe), self.nlist)
                if probes.dtype != torch.int32 or tuple(probes.shape) != (nq, npb) or not probes.is_contiguous():
                    raise ValueError(f"probes must be a contiguous int32 tensor of shape ({nq}, {npb})")
                L.check(self._lib.mv_search_with_probes(self._h, _ptr(q), nq, int(k), int(nprobe), _ptr(probes),
                                                        _ptr(bitset), nb, _ptr(D), _ptr(I), sp))
                return D, I
            L.check(self._lib.mv_search(self._h, _ptr(q), nq, int(k), int(nprobe), _ptr(bitset), nb, _ptr(D), _ptr(I),
                                        sp))
            return D, I

    def search_probes(self, q, nprobe: int, stream=None):
        s, ctx = self._on(stream)
        with ctx:
            q = _as_f32(q)
            nq = int(q.shape[0])
            npb = min(int(nprobe), self.nlist)
            P = torch.empty((nq, npb), dtype=torch.int32, device=torch.device("cuda", self.device))
            L.check(self._lib.mv_search_probes(self._h, _ptr(q), nq, int(nprobe), _ptr(P), C.c_void_p(s.cuda_stream)))
            return P

    # -- measurement ---------------------------------------------------------------------------
    STAGES = ("coarse", "bucket", "scan_a", "seed", "scan", "select")

    def profile(self, on: bool = True):
        L.check(self._lib.mv_profile_enable(self._h, int(bool(on))))

    def profile_read(self, reset: bool = True):
        """Summed CUDA-event milliseconds per stage since the last reset, the number of profiled
        searches and the number of libmv kernel launches."""
        ms = (C.c_double * len(self.STAGES))()
        ns, nl = C.c_int64(), C.c_int64()
        L.check(self._lib.mv_profile_read(self._h, ms, C.byref(ns), C.byref(nl), int(reset)))
        return dict(zip(self.STAGES, list(ms))), int(ns.value), int(nl.value)

    def profile_counters(self, reset: bool = True) -> dict:
        """Emission counters of the profiled searches: queries, seeding-phase and main-scan emissions."""
        out = (C.c_int64 * 3)()
        L.check(self._lib.mv_profile_counters(self._h, out, int(reset)))
        return {"queries": int(out[0]), "phase_a_emitted": int(out[1]), "phase_b_emitted": int(out[2])}

    def describe(self) -> dict:
        import json
        buf = C.create_string_buffer(2048)
        L.check(self._lib.mv_index_describe(self._h, buf, 2048))
        return json.loads(buf.value.decode())

    # -- parity hooks --------------------------------------------------------------------------
    def storage(self, codes: bool = False):
        off = np.empty(self.nlist + 1, np.int64)
        ids = np.empty(self.ntotal, np.int64)
        cw = getattr(self, "pq_m", 0) if self.kind == L.MV_IVF_PQ else self.d
        cd = np.empty((self.ntotal, cw), np.uint8) if codes else None
        L.check(self._lib.mv_index_storage(self._h, _ptr(off), _ptr(ids), _ptr(cd)))
        return off, ids, cd


def merge_topk(dists, ids, metric="l2", stream=None):
    """mv_merge_topk: dists/ids [nsrc, nq, k] device tensors -> merged [nq, k]."""
    lib = L.load()
    m = METRICS[metric.lower() if isinstance(metric, str) else metric]
    dev = dists.device.index if dists.is_cuda else torch.cuda.current_device()
    s = _torch_stream(dev, stream)
    with (torch.cuda.stream(s) if stream is not None else contextlib.nullcontext()):
        dists = dists.contiguous().float()
        ids = ids.contiguous().to(torch.int64)
        nsrc, nq, k = dists.shape
        D = torch.empty((nq, k), dtype=torch.float32, device=dists.device)
        I = torch.empty((nq, k), dtype=torch.int64, device=dists.device)
        L.check(lib.mv_merge_topk(m, _ptr(dists), _ptr(ids), int(nsrc), int(nq), int(k), _ptr(D), _ptr(I),
                                  C.c_void_p(s.cuda_stream) if dists.is_cuda else None))
    return D, I


def kmeans(x, nlist: int, niter: int = 10, metric="l2", spherical: bool = False, init=None, stream=None):
    """mv_kmeans: niter Lloyd iterations of the coarse codebook on the device.
    x: device [n, d] fp32 training rows; init: [nlist, d] initial centroids (default: the first
    nlist rows -- pass a seeded sample).  Returns the [nlist, d] fp32 centroids."""
    lib = L.load()
    x = x.contiguous().float()
    n, d = x.shape
    c = (x[:nlist] if init is None else init).contiguous().float().clone()
    m = METRICS[metric.lower() if isinstance(metric, str) else metric]
    s = _torch_stream(x.device.index, stream)
    L.check(lib.mv_kmeans(_ptr(x), int(n), int(d), m, int(nlist), int(niter), int(bool(spherical)), _ptr(c),
                          int(x.device.index), C.c_void_p(s.cuda_stream)))
    return c
