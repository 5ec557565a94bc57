"""Seeded synthetic inputs shared by the oracle tests, the CUDA-path tests and bench.py.

This module holds NONE of the method's arithmetic (no distances, no quantisation, no
top-k): it only draws the inputs -- base vectors, queries, ids, bitsets -- and prepares
the centroid codebook that BASELINE.json's north star calls "supplied centroids"
(k-means lives in ``mvgen.kmeans``, data preparation only).

Shapes follow the paper's workloads (§7.1):
  * SIFT-shaped: d=128, 4-byte floats holding small non-negative integers (SIFT1B is
    1B x 128 in 512 GB).  Here: integers in [0,255] from an integer counter hash, so
    every row is reproducible bit-for-bit on CPU and GPU from (seed, row).
  * Deep-shaped: d=96, unit-L2-norm fp32 (Deep1B is 1B x 96 in 384 GB).

Both are two-level mixtures (top centres -> micro centres -> points) so that the data
has the low intrinsic dimension that makes IVF recall meaningful.  The recipe and its
calibration are in DESIGN.md §3.
"""
from __future__ import annotations

import math

import numpy as np
import torch

# --------------------------------------------------------------------------------------
# splitmix64 counter hash in wrap-around int64 torch arithmetic (identical on CPU/GPU)
# --------------------------------------------------------------------------------------
_U64 = 1 << 64


def _s64(c: int) -> int:
    return c - _U64 if c >= (1 << 63) else c


_G = _s64(0x9E3779B97F4A7C15)
_M1 = _s64(0xBF58476D1CE4E5B9)
_M2 = _s64(0x94D049BB133111EB)

SEED_BASE = 0x5EED0001
SEED_QUERY = 0x5EED0002
SEED_BITSET = 0x5EED0003
SEED_KMEANS = 0x5EED0004
SEED_SQ8 = 0x5EED0005


def _srl(x: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of an int64 tensor viewed as uint64."""
    return (x >> k) & ((1 << (64 - k)) - 1)


def _mix(z: torch.Tensor) -> torch.Tensor:
    z = (z ^ _srl(z, 30)) * _M1
    z = (z ^ _srl(z, 27)) * _M2
    return z ^ _srl(z, 31)


def hash64(seed: int, stream: int, ctr: torch.Tensor) -> torch.Tensor:
    """splitmix64(splitmix64(seed, stream) + ctr): one 64-bit draw per counter value."""
    s = torch.tensor([_s64((seed * 0x100000001B3 + stream * 0x9E37) % _U64)], dtype=torch.int64)
    key = _mix(s + _G)  # per-(seed, stream) key
    return _mix(ctr.to(torch.int64) + key.to(ctr.device) + _G)


def hash_u31(seed: int, stream: int, ctr: torch.Tensor) -> torch.Tensor:
    """Top 31 bits of hash64 as a non-negative int64."""
    return _srl(hash64(seed, stream, ctr), 33)


def hash_unit(seed: int, stream: int, ctr: torch.Tensor) -> torch.Tensor:
    """Uniform (0,1) float64 from the top 53 bits."""
    return (_srl(hash64(seed, stream, ctr), 11).to(torch.float64) + 0.5) * (1.0 / (1 << 53))


def splitmix64_np(state: int, count: int) -> list[int]:
    """Textbook sequential SplitMix64 (numpy uint64) -- used only to pin ``_mix``."""
    out = []
    with np.errstate(over="ignore"):
        s = np.uint64(state)
        for _ in range(count):
            s = s + np.uint64(0x9E3779B97F4A7C15)
            z = s
            z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
            z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
            out.append(int(z ^ (z >> np.uint64(31))))
    return out


# --------------------------------------------------------------------------------------
# SIFT-shaped: integer-valued fp32 in [0, 255]
# --------------------------------------------------------------------------------------
class SiftSpec:
    """Two-level integer mixture.  top centre component = floor(255 u^2.5) (skewed towards
    0 like SIFT histograms); micro centre = top + tri(w1); point = micro + tri(w2), all
    clipped to [0,255].  tri(w) = (a mod (w+1)) + (b mod (w+1)) - w (integer triangle)."""

    def __init__(self, d: int = 128, n_top: int = 64, n_micro: int = 65536, w1: int = 40, w2: int = 12,
                 seed: int = SEED_BASE):
        self.d, self.n_top, self.n_micro, self.w1, self.w2, self.seed = d, n_top, n_micro, w1, w2, seed
        ctr = torch.arange(n_top * d, dtype=torch.int64)
        u = hash_unit(seed, 11, ctr)
        self.top = torch.floor(255.0 * u.pow(2.5)).to(torch.int64).reshape(n_top, d)

    def _tri(self, stream: int, ctr: torch.Tensor, w: int) -> torch.Tensor:
        a = hash_u31(self.seed, stream, ctr) % (w + 1)
        b = hash_u31(self.seed, stream + 1, ctr) % (w + 1)
        return a + b - w

    def micro_of(self, rows: torch.Tensor, row_seed: int) -> torch.Tensor:
        return hash_u31(row_seed, 21, rows) % self.n_micro

    def rows(self, row0: int, n: int, row_seed: int, device="cpu") -> torch.Tensor:
        return self.rows_at(torch.arange(row0, row0 + n, dtype=torch.int64, device=device), row_seed)

    def rows_at(self, rows: torch.Tensor, row_seed: int) -> torch.Tensor:
        """Rows with the given global indices (int64 tensor): any subset of the base set, e.g. the
        rows one shard of a vector-sharded index owns, regenerated bit-identically anywhere."""
        d, device = self.d, rows.device
        m = self.micro_of(rows, row_seed)                       # micro centre per row
        t = hash_u31(self.seed, 13, m) % self.n_top             # its top centre
        j = torch.arange(d, dtype=torch.int64, device=device)
        top = self.top.to(device)[t]                            # n x d
        mc = (top + self._tri(31, m[:, None] * d + j[None, :], self.w1)).clamp_(0, 255)
        # point noise is keyed by (row_seed, row) so base and query rows differ
        pc = rows[:, None] * d + j[None, :]
        a = hash_u31(row_seed, 41, pc) % (self.w2 + 1)
        b = hash_u31(row_seed, 42, pc) % (self.w2 + 1)
        x = (mc + a + b - self.w2).clamp_(0, 255)
        return x.to(torch.float32)


def sift_base(n: int, d: int = 128, row0: int = 0, device="cpu", spec: SiftSpec | None = None,
              chunk: int = 1 << 18) -> torch.Tensor:
    spec = spec or SiftSpec(d=d)
    out = torch.empty((n, spec.d), dtype=torch.float32, device=device)
    for s in range(0, n, chunk):
        e = min(n, s + chunk)
        out[s:e] = spec.rows(row0 + s, e - s, SEED_BASE, device)
    return out


def sift_queries(nq: int, d: int = 128, device="cpu", spec: SiftSpec | None = None) -> torch.Tensor:
    spec = spec or SiftSpec(d=d)
    return spec.rows(0, nq, SEED_QUERY, device)


# --------------------------------------------------------------------------------------
# Deep-shaped: unit-norm fp32
# --------------------------------------------------------------------------------------
def _gauss(seed: int, stream: int, ctr: torch.Tensor) -> torch.Tensor:
    u1 = hash_unit(seed, stream, ctr)
    u2 = hash_unit(seed, stream + 1, ctr)
    return torch.sqrt(-2.0 * torch.log(u1)) * torch.cos(2.0 * math.pi * u2)


class DeepSpec:
    """mu_t ~ N(0,I) normalised; micro = normalise(mu_t + s1 g/sqrt(d)); x = normalise(micro + s2 g/sqrt(d)).

    s1 and s2 are relative noise norms (g/sqrt(d) has norm ~1), so the cluster structure does not
    dissolve into isotropic noise as d grows."""

    def __init__(self, d: int = 96, n_top: int = 256, n_micro: int = 262144, s1: float = 0.6, s2: float = 0.5,
                 seed: int = SEED_BASE):
        self.d, self.n_top, self.n_micro, self.s1, self.s2, self.seed = d, n_top, n_micro, s1, s2, seed
        g = _gauss(seed, 51, torch.arange(n_top * d, dtype=torch.int64)).reshape(n_top, d)
        self.top = g / g.norm(dim=1, keepdim=True)

    def rows(self, row0: int, n: int, row_seed: int, device="cpu") -> torch.Tensor:
        d = self.d
        rows = torch.arange(row0, row0 + n, dtype=torch.int64, device=device)
        m = hash_u31(row_seed, 61, rows) % self.n_micro
        t = hash_u31(self.seed, 63, m) % self.n_top
        j = torch.arange(d, dtype=torch.int64, device=device)
        mc = self.top.to(device)[t] + (self.s1 / d ** 0.5) * _gauss(self.seed, 71, m[:, None] * d + j[None, :])
        mc = mc / mc.norm(dim=1, keepdim=True)
        x = mc + (self.s2 / d ** 0.5) * _gauss(row_seed, 81, rows[:, None] * d + j[None, :])
        x = x / x.norm(dim=1, keepdim=True)
        return x.to(torch.float32)


def deep_base(n: int, d: int = 96, row0: int = 0, device="cpu", spec: DeepSpec | None = None,
              chunk: int = 1 << 18) -> torch.Tensor:
    spec = spec or DeepSpec(d=d)
    out = torch.empty((n, spec.d), dtype=torch.float32, device=device)
    for s in range(0, n, chunk):
        e = min(n, s + chunk)
        out[s:e] = spec.rows(row0 + s, e - s, SEED_BASE, device)
    return out


def deep_queries(nq: int, d: int = 96, device="cpu", spec: DeepSpec | None = None) -> torch.Tensor:
    spec = spec or DeepSpec(d=d)
    return spec.rows(0, nq, SEED_QUERY, device)


# --------------------------------------------------------------------------------------
# ids, bitsets, generic small inputs
# --------------------------------------------------------------------------------------
def mod_bitset(nbits: int, mod: int = 10, seed: int = SEED_BITSET, device="cpu") -> torch.Tensor:
    """Deletion bitset, bit i = [hash(seed, i) mod `mod` == 0]; 1 = excluded.  Packed LSB-first:
    bit i lives in byte i>>3 at position i&7 (the ABI convention, include/mv.h)."""
    ids = torch.arange(nbits, dtype=torch.int64, device=device)
    bits = (hash_u31(seed, 91, ids) % mod == 0).to(torch.uint8)
    return pack_bits(bits)


def pack_bits(bits: torch.Tensor) -> torch.Tensor:
    n = bits.numel()
    nb = (n + 7) // 8
    padded = torch.zeros(nb * 8, dtype=torch.uint8, device=bits.device)
    padded[:n] = bits.to(torch.uint8)
    w = torch.tensor([1, 2, 4, 8, 16, 32, 64, 128], dtype=torch.uint8, device=bits.device)
    return (padded.reshape(nb, 8) * w).sum(dim=1, dtype=torch.int64).to(torch.uint8)


def unpack_bits(packed: torch.Tensor, nbits: int) -> torch.Tensor:
    p = packed.to(torch.int64)
    sh = torch.arange(8, dtype=torch.int64, device=packed.device)
    return ((p[:, None] >> sh[None, :]) & 1).reshape(-1)[:nbits].to(torch.uint8)


def gaussian(n: int, d: int, seed: int, stream: int = 0, device="cpu") -> torch.Tensor:
    """Plain N(0,1) fp32 matrix from the counter hash (general non-integer data)."""
    ctr = torch.arange(n * d, dtype=torch.int64, device=device)
    return _gauss(seed, 101 + 2 * stream, ctr).reshape(n, d).to(torch.float32)


def uniform_int(n: int, d: int, lo: int, hi: int, seed: int, stream: int = 0, device="cpu") -> torch.Tensor:
    """Integer-valued fp32 in [lo, hi] (inclusive)."""
    ctr = torch.arange(n * d, dtype=torch.int64, device=device)
    v = hash_u31(seed, 201 + stream, ctr) % (hi - lo + 1) + lo
    return v.reshape(n, d).to(torch.float32)


def permuted_ids(n: int, seed: int, device="cpu") -> torch.Tensor:
    """A seeded permutation of 0..n-1 scaled into sparse int64 ids (ids need not be dense)."""
    key = hash64(seed, 301, torch.arange(n, dtype=torch.int64, device=device))
    perm = torch.argsort(key)
    return perm.to(torch.int64) * 3 + 7
