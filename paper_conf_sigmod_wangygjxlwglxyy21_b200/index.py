"""Thin Python binding over the C ABI (include/mv.h): argument marshalling only.

Tensors are passed as raw pointers (device tensors stay on the device; CPU tensors / numpy arrays
are staged by the library itself).  Every step of the search runs in libmv's CUDA kernels; torch
only provides device memory and the current stream.
"""
from __future__ import annotations

import ctypes as C

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


def _as_f32(x, d=None):
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


def _stream(device: int, stream=None):
    if stream is None:
        return C.c_void_p(torch.cuda.current_stream(device).cuda_stream)
    if isinstance(stream, torch.cuda.Stream):
        return C.c_void_p(stream.cuda_stream)
    return C.c_void_p(int(stream))


METRICS = {"l2": L.MV_L2, "ip": L.MV_IP, L.MV_L2: L.MV_L2, L.MV_IP: L.MV_IP}
TYPES = {"flat": L.MV_IVF_FLAT, "ivf_flat": L.MV_IVF_FLAT, "sq8": L.MV_IVF_SQ8, "ivf_sq8": L.MV_IVF_SQ8,
         L.MV_IVF_FLAT: L.MV_IVF_FLAT, L.MV_IVF_SQ8: L.MV_IVF_SQ8}


class Index:
    """mv_index_create(d, metric, type, nlist) and friends (§3.2.1)."""

    def __init__(self, d: int, metric="l2", kind="flat", nlist: int = 1, device: int | None = None):
        self._lib = L.load()
        self.d, self.nlist = int(d), int(nlist)
        self.metric = METRICS[metric.lower() if isinstance(metric, str) else metric]
        self.kind = TYPES[kind.lower() if isinstance(kind, str) else kind]
        self.device = torch.cuda.current_device() if device is None else int(device)
        h = C.c_void_p()
        L.check(self._lib.mv_index_create(self.d, self.metric, self.kind, self.nlist, self.device, C.byref(h)))
        self._h = h

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

    def get_sq8(self):
        vmin = np.empty(self.d, np.float32)
        vdiff = np.empty(self.d, np.float32)
        L.check(self._lib.mv_index_get_sq8(self._h, _ptr(vmin), _ptr(vdiff)))
        return vmin, vdiff

    def add(self, x, ids, stream=None):
        x = _as_f32(x)
        ids = _as_i64(ids)
        n = int(x.shape[0])
        if int(ids.shape[0]) != n:
            raise ValueError("ids and vectors differ in length")
        L.check(self._lib.mv_index_add(self._h, _ptr(x), _ptr(ids), n, _stream(self.device, stream)))

    # -- search ------------------------------------------------------------------------------
    def search(self, q, k: int, nprobe: int, bitset=None, nbits: int | None = None, out=None, stream=None,
               probes=None):
        """Returns (D[nq,k] float32, I[nq,k] int64) on the index device (or into `out`).
        probes: optional int32 [nq, min(nprobe, nlist)] best-first buckets per query (as
        search_probes returns them); the coarse step is then skipped (mv_search_with_probes)."""
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
        if probes is not None:
            npb = min(int(nprobe), self.nlist)
            if probes.dtype != torch.int32 or tuple(probes.shape) != (nq, npb) or not probes.is_contiguous():
                raise ValueError(f"probes must be a contiguous int32 tensor of shape ({nq}, {npb})")
            L.check(self._lib.mv_search_with_probes(self._h, _ptr(q), nq, int(k), int(nprobe), _ptr(probes),
                                                    _ptr(bitset), nb, _ptr(D), _ptr(I), _stream(self.device, stream)))
            return D, I
        L.check(self._lib.mv_search(self._h, _ptr(q), nq, int(k), int(nprobe), _ptr(bitset), nb, _ptr(D), _ptr(I),
                                    _stream(self.device, stream)))
        return D, I

    def search_probes(self, q, nprobe: int, stream=None):
        q = _as_f32(q)
        nq = int(q.shape[0])
        npb = min(int(nprobe), self.nlist)
        P = torch.empty((nq, npb), dtype=torch.int32, device=torch.device("cuda", self.device))
        L.check(self._lib.mv_search_probes(self._h, _ptr(q), nq, int(nprobe), _ptr(P), _stream(self.device, stream)))
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

    def describe(self) -> dict:
        import json
        buf = C.create_string_buffer(1024)
        L.check(self._lib.mv_index_describe(self._h, buf, 1024))
        return json.loads(buf.value.decode())

    # -- parity hooks --------------------------------------------------------------------------
    def storage(self, codes: bool = False):
        off = np.empty(self.nlist + 1, np.int64)
        ids = np.empty(self.ntotal, np.int64)
        cd = np.empty((self.ntotal, self.d), np.uint8) if codes else None
        L.check(self._lib.mv_index_storage(self._h, _ptr(off), _ptr(ids), _ptr(cd)))
        return off, ids, cd


def merge_topk(dists, ids, metric="l2", stream=None):
    """mv_merge_topk: dists/ids [nsrc, nq, k] device tensors -> merged [nq, k]."""
    lib = L.load()
    m = METRICS[metric.lower() if isinstance(metric, str) else metric]
    dists = dists.contiguous().float()
    ids = ids.contiguous().to(torch.int64)
    nsrc, nq, k = dists.shape
    D = torch.empty((nq, k), dtype=torch.float32, device=dists.device)
    I = torch.empty((nq, k), dtype=torch.int64, device=dists.device)
    dev = dists.device.index if dists.is_cuda else 0
    L.check(lib.mv_merge_topk(m, _ptr(dists), _ptr(ids), int(nsrc), int(nq), int(k), _ptr(D), _ptr(I),
                              _stream(dev, stream) if dists.is_cuda else None))
    return D, I
