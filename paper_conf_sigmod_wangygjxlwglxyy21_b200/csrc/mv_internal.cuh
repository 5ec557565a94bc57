// mv_internal.cuh -- shared device helpers and host-side launcher declarations for libmv.
// Nothing here is shared with oracle/ (tests/ compare the two).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>
#include <algorithm>

#include "mv.h"

#define MV_FULL 0xffffffffu
#define MV_KEY_PAD 0xffffffffffffffffull

namespace mv {

constexpr int kMaxK = 16384;          // PAPER.md:801-802 (§3.3 fn. 5): k <= 16384
constexpr int kLocalSelectMaxK = 1024;  // per-(query,list) selection in the scan for k <= 1024
constexpr int kNumSMs = 148;
constexpr int kProfStages = 6;   // coarse, bucket, scan A, seed select, scan B, final select (mv.h)

__host__ __device__ __forceinline__ int64_t min64(int64_t a, int64_t b) { return a < b ? a : b; }
__host__ __device__ __forceinline__ int64_t max64(int64_t a, int64_t b) { return a > b ? a : b; }

// ------------------------------------------------------------------------------------------
// Orderable keys.  A candidate is one u64: (distance key << 32) | id-rank.  The distance key
// is the IEEE-754 order-preserving map of the "badness" (L2 distance, or -IP), so ascending
// u64 order is the ABI's best-first order (distance, then id, then storage row) -- the id-rank
// of a stored row is its position in the (id, row) sorted order (computed at add time).
// ------------------------------------------------------------------------------------------
__host__ __device__ __forceinline__ uint32_t f2key(float f) {
#ifdef __CUDA_ARCH__
  f = __fadd_rn(f, 0.0f);  // -0 -> +0: equal distances must give equal keys
  uint32_t b = __float_as_uint(f);
#else
  f = f + 0.0f;
  uint32_t b;
  memcpy(&b, &f, 4);
#endif
  return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}

__host__ __device__ __forceinline__ float key2f(uint32_t k) {
  uint32_t b = (k & 0x80000000u) ? (k ^ 0x80000000u) : ~k;
#ifdef __CUDA_ARCH__
  return __uint_as_float(b);
#else
  float f;
  memcpy(&f, &b, 4);
  return f;
#endif
}

// badness key of a distance under the metric (L2: smaller better; IP: larger better)
__device__ __forceinline__ uint32_t dist_key(float d, int metric) { return f2key(metric == MV_L2 ? d : -d); }
__device__ __forceinline__ float key_dist(uint32_t k, int metric) {
  float b = key2f(k);
  return metric == MV_L2 ? b : -b;
}

__device__ __forceinline__ bool bit_excluded(const uint8_t* __restrict__ bitset, int64_t nbits, int64_t id) {
  if (bitset == nullptr || id < 0 || id >= nbits) return false;
  return (__ldg(bitset + (id >> 3)) >> (id & 7)) & 1;
}

// debug event counters (set by the scan when MV_SCAN_TRACE=1): 0 tiles-with-survivors, 1 warm-ups,
// 2 flushes, 3 bisection fallbacks, 4 survivors appended
__device__ __forceinline__ void dbg_count(unsigned long long* c, int i, unsigned long long v) {
  if (c && (threadIdx.x & 31) == 0) atomicAdd(c + i, v);
}

// ------------------------------------------------------------------------------------------
// Warp-cooperative insertion into a sorted (ascending) smem list of length L.  All 32 lanes
// call it; lanes with `has` offer one candidate each.  Candidates not below the current last
// element are dropped (the list keeps the L smallest keys seen; keys are unique).
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ void warp_list_insert(uint64_t* list, int L, uint64_t cand, bool has) {
  const int lane = threadIdx.x & 31;
  uint32_t mask = __ballot_sync(MV_FULL, has && cand < list[L - 1]);
  while (mask) {
    const int src = __ffs(mask) - 1;
    mask &= mask - 1;
    const uint64_t c = __shfl_sync(MV_FULL, cand, src);
    if (!(c < list[L - 1])) continue;  // uniform: every lane reads the same word
    int pos = 0;
    for (int base = 0; base < L; base += 32) {
      const int i = base + lane;
      pos += __popc(__ballot_sync(MV_FULL, i < L && list[i] < c));
    }
    for (int hi = L - 1; hi > pos; hi -= 32) {
      const int i = hi - lane;
      uint64_t v = 0;
      const bool mv_ = i > pos;
      if (mv_) v = list[i - 1];
      __syncwarp();
      if (mv_) list[i] = v;
      __syncwarp();
    }
    if (lane == 0) list[pos] = c;
    __syncwarp();
  }
}

// ------------------------------------------------------------------------------------------
// Warp-register bitonic networks over 32*R u64 keys; element e = r*32 + lane lives in v[r].
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ uint64_t shfl_xor64(uint64_t v, int m) {
  const uint32_t lo = __shfl_xor_sync(MV_FULL, (uint32_t)v, m);
  const uint32_t hi = __shfl_xor_sync(MV_FULL, (uint32_t)(v >> 32), m);
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ uint64_t shfl64(uint64_t v, int src) {
  const uint32_t lo = __shfl_sync(MV_FULL, (uint32_t)v, src);
  const uint32_t hi = __shfl_sync(MV_FULL, (uint32_t)(v >> 32), src);
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }
__device__ __forceinline__ uint64_t umax64(uint64_t a, uint64_t b) { return a < b ? b : a; }

// one compare-exchange step of a bitonic network: element pairs at distance `stride`, the
// direction of block `size` ascending when (e & size) == 0 (size = 0 -> all ascending)
template <int R>
__device__ __forceinline__ void bitonic_step(uint64_t (&v)[R], int size, int stride) {
  const int lane = threadIdx.x & 31;
  if (stride >= 32) {
    const int rs = stride >> 5;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if ((r & rs) == 0) {
        const int e = r * 32 + lane;
        const bool up = size == 0 || (e & size) == 0;
        const uint64_t a = v[r], b = v[r | rs];
        v[r] = up ? umin64(a, b) : umax64(a, b);
        v[r | rs] = up ? umax64(a, b) : umin64(a, b);
      }
    }
  } else {
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int e = r * 32 + lane;
      const bool up = size == 0 || (e & size) == 0;
      const bool lower = (lane & stride) == 0;
      const uint64_t o = shfl_xor64(v[r], stride);
      v[r] = (lower == up) ? umin64(v[r], o) : umax64(v[r], o);
    }
  }
}

template <int R>
__device__ __forceinline__ void warp_bitonic_sort(uint64_t (&v)[R]) {
#pragma unroll
  for (int size = 2; size <= 32 * R; size <<= 1)
#pragma unroll
    for (int stride = size >> 1; stride > 0; stride >>= 1) bitonic_step<R>(v, size == 32 * R ? 0 : size, stride);
}

// bitonic sequence -> ascending
template <int R>
__device__ __forceinline__ void warp_bitonic_merge(uint64_t (&v)[R]) {
#pragma unroll
  for (int stride = 16 * R; stride > 0; stride >>= 1) bitonic_step<R>(v, 0, stride);
}

// list (sorted ascending, 32R entries) := smallest 32R of list U cand (cand sorted ascending)
template <int R>
__device__ __forceinline__ void warp_merge_smallest(uint64_t (&list)[R], const uint64_t (&cand)[R]) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const uint64_t c = shfl64(cand[R - 1 - r], 31 - lane);  // reversed candidate element
    list[r] = umin64(list[r], c);
  }
  warp_bitonic_merge<R>(list);
}

// k-th smallest (1-indexed) of the 128 u32 values v[0..3] x 32 lanes: MSB-first bisection, one
// ballot per value per bit, no divergence.
__device__ __forceinline__ uint32_t warp_kth_u32(const uint32_t (&v)[4], int k) {
  uint32_t ans = 0;
#pragma unroll 1
  for (int b = 31; b >= 0; --b) {
    const uint32_t trial = ans | (1u << b);
    int cnt = 0;
#pragma unroll
    for (int m = 0; m < 4; ++m) cnt += __popc(__ballot_sync(MV_FULL, v[m] < trial));
    if (cnt < k) ans = trial;
  }
  return ans;
}

// One warp folds a tile's 128 candidates -- distance keys k32[m] of element e = m*32 + lane
// (0xffffffff = invalid), tie-break low word low(e) -- into the ascending list L[0..k) (u64 keys,
// PAD-filled), keeping only keys below `li` (the global per-query threshold).  k <= 32: candidates
// above min(L[k-1], li) are dropped with one compare; many survivors (warm-up) are first narrowed
// to the k smallest by a warp radix select, then compacted, sorted and merged (bitonic); a few
// survivors are inserted one by one.  k <= 128: sort-128 + merge; larger k: insertion.
template <typename Low>
__device__ __forceinline__ void warp_select_tile(uint64_t* L, int k, uint64_t li, const uint32_t (&k32)[4], Low low,
                                                 uint64_t* wscr) {
  const int lane = threadIdx.x & 31;
  const uint64_t thr = L[k - 1] < li ? L[k - 1] : li;
  const uint32_t thr32 = (uint32_t)(thr >> 32);
  bool pass[4];
  int npass = 0;
#pragma unroll
  for (int m = 0; m < 4; ++m) {
    pass[m] = k32[m] != 0xffffffffu && k32[m] <= thr32;
    npass += __popc(__ballot_sync(MV_FULL, pass[m]));
  }
  if (npass == 0) return;
  if (k <= 32 && npass > 32) {
    // warm-up: narrow to the k smallest distance keys of this tile (plus exact ties)
    uint32_t v[4];
#pragma unroll
    for (int m = 0; m < 4; ++m) v[m] = pass[m] ? k32[m] : 0xffffffffu;
    const uint32_t t32 = warp_kth_u32(v, k);
    npass = 0;
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      pass[m] = pass[m] && k32[m] <= t32;
      npass += __popc(__ballot_sync(MV_FULL, pass[m]));
    }
  }
  if (k <= 32 && npass <= 32 && npass > 2) {
    // compact the survivors into one register per lane, sort, merge into the list
    int off = 0;
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      const uint32_t bm = __ballot_sync(MV_FULL, pass[m]);
      if (pass[m]) wscr[off + __popc(bm & ((1u << lane) - 1))] = ((uint64_t)k32[m] << 32) | low(m * 32 + lane);
      off += __popc(bm);
    }
    __syncwarp();
    uint64_t c[1] = {lane < npass ? wscr[lane] : MV_KEY_PAD};
    if (!(c[0] < thr)) c[0] = MV_KEY_PAD;
    warp_bitonic_sort<1>(c);
    uint64_t lv[1] = {lane < k ? L[lane] : MV_KEY_PAD};
    warp_merge_smallest<1>(lv, c);
    __syncwarp();
    if (lane < k) L[lane] = lv[0];
    __syncwarp();
  } else if (npass <= 8 || k > 128) {
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      const uint64_t key = pass[m] ? (((uint64_t)k32[m] << 32) | low(m * 32 + lane)) : MV_KEY_PAD;
      warp_list_insert(L, k, key, pass[m] && key < thr);
    }
  } else {
    uint64_t key[4];
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      key[m] = pass[m] ? (((uint64_t)k32[m] << 32) | low(m * 32 + lane)) : MV_KEY_PAD;
      if (!(key[m] < thr)) key[m] = MV_KEY_PAD;
    }
    warp_bitonic_sort<4>(key);
    if (k <= 32) {
      uint64_t lv[1] = {lane < k ? L[lane] : MV_KEY_PAD}, cv[1] = {key[0]};
      warp_merge_smallest<1>(lv, cv);
      __syncwarp();
      if (lane < k) L[lane] = lv[0];
    } else if (k <= 64) {
      uint64_t lv[2], cv[2] = {key[0], key[1]};
#pragma unroll
      for (int r2 = 0; r2 < 2; ++r2) lv[r2] = r2 * 32 + lane < k ? L[r2 * 32 + lane] : MV_KEY_PAD;
      warp_merge_smallest<2>(lv, cv);
      __syncwarp();
#pragma unroll
      for (int r2 = 0; r2 < 2; ++r2)
        if (r2 * 32 + lane < k) L[r2 * 32 + lane] = lv[r2];
    } else {
      uint64_t lv[4];
#pragma unroll
      for (int r2 = 0; r2 < 4; ++r2) lv[r2] = r2 * 32 + lane < k ? L[r2 * 32 + lane] : MV_KEY_PAD;
      warp_merge_smallest<4>(lv, key);
      __syncwarp();
#pragma unroll
      for (int r2 = 0; r2 < 4; ++r2)
        if (r2 * 32 + lane < k) L[r2 * 32 + lane] = lv[r2];
    }
    __syncwarp();
  }
}

// ------------------------------------------------------------------------------------------
// Buffered selection for k <= 32: survivors of each tile are appended to a per-query 32-entry smem
// buffer B (count *nb) and merged into the sorted list L only when the buffer would overflow (and
// once at the end, warp_flush_buffer), so the ~21-step sort/merge network runs a few times per
// query instead of once per tile.  *bnd is a running upper bound on the k-th best distance key,
// tightened as soon as a crowded tile is narrowed to its k smallest keys (exact: anything with k
// smaller keys in the same tile cannot be in the top-k) and after every flush; publish(t32) lets
// the caller share it (the scan folds it into the global per-query tau).
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ void warp_flush_buffer(uint64_t* L, uint64_t* B, int* nb, uint32_t* bnd, int k,
                                                  uint64_t li) {
  const int lane = threadIdx.x & 31;
  const int n = *nb;
  if (n == 0) return;
  const uint64_t thr = L[k - 1] < li ? L[k - 1] : li;
  uint64_t c[1] = {lane < n ? B[lane] : MV_KEY_PAD};
  if (!(c[0] < thr)) c[0] = MV_KEY_PAD;
  warp_bitonic_sort<1>(c);
  uint64_t lv[1] = {lane < k ? L[lane] : MV_KEY_PAD};
  warp_merge_smallest<1>(lv, c);
  __syncwarp();
  if (lane < k) L[lane] = lv[0];
  if (lane == k - 1 && lv[0] != MV_KEY_PAD) *bnd = min(*bnd, (uint32_t)(lv[0] >> 32));
  if (lane == 0) *nb = 0;
  __syncwarp();
}

// Fold one tile into (L, B) after the caller's filter: pass[] marks candidates at or below the
// bound, npass their count (> 0).
template <typename Low, typename Pub>
__device__ __forceinline__ void warp_collect_passed(uint64_t* L, uint64_t* B, int* nb, uint32_t* bnd, int k, uint64_t li,
                                                    const uint32_t (&k32)[4], bool (&pass)[4], int npass, Low low,
                                                    Pub publish, uint64_t* wscr, unsigned long long* dc = nullptr) {
  const int lane = threadIdx.x & 31;
  dbg_count(dc, 0, 1);
  if (npass > 32) dbg_count(dc, 1, 1);
  if (npass > 32) {
    uint32_t v[4];
#pragma unroll
    for (int m = 0; m < 4; ++m) v[m] = pass[m] ? k32[m] : 0xffffffffu;
    const uint32_t t32 = warp_kth_u32(v, k);
    npass = 0;
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      pass[m] = pass[m] && k32[m] <= t32;
      npass += __popc(__ballot_sync(MV_FULL, pass[m]));
    }
    __syncwarp();
    if (lane == 0) {
      *bnd = min(*bnd, t32);
      publish(t32);
    }
    __syncwarp();
    if (npass > 32) {  // pathological exact ties: fold this tile directly
      warp_flush_buffer(L, B, nb, bnd, k, li);
      warp_select_tile(L, k, li, k32, low, wscr);
      return;
    }
  }
  if (*nb + npass > 32) {
    warp_flush_buffer(L, B, nb, bnd, k, li);
    dbg_count(dc, 2, 1);
    // the list's k-th key is an exact upper bound of the query's k-th best: share it
    if (lane == 0 && L[k - 1] != MV_KEY_PAD) publish((uint32_t)(L[k - 1] >> 32));
  }
  dbg_count(dc, 4, npass);
  int off = *nb;
#pragma unroll
  for (int m = 0; m < 4; ++m) {
    const uint32_t bm = __ballot_sync(MV_FULL, pass[m]);
    if (pass[m]) B[off + __popc(bm & ((1u << lane) - 1))] = ((uint64_t)k32[m] << 32) | low(m * 32 + lane);
    off += __popc(bm);
  }
  __syncwarp();
  if (lane == 0) *nb = off;
  __syncwarp();
}

// Filter G query slots per call so their shared-memory loads and ballots overlap (the per-tile
// filter is latency-bound); only slots with survivors enter the (rare, serial) fold.
//   rowk(g, m) -> distance key of element m*32+lane for query g;  st(g) -> per-query state.
template <int G, typename RowK, typename State, typename Low, typename Pub>
__device__ __forceinline__ void warp_filter_group(int nvalid, int k, RowK rowk, State st, Low low, Pub publish,
                                                  uint64_t* wscr, unsigned long long* dc = nullptr, bool fold = true) {
  uint32_t k32[G][4];
  uint32_t thr32[G];
#pragma unroll
  for (int g = 0; g < G; ++g) {
    if (g < nvalid) {
      uint64_t *L, *B;
      int* nb;
      uint32_t* bnd;
      uint64_t li;
      st(g, L, B, nb, bnd, li);
      const uint64_t thr = L[k - 1] < li ? L[k - 1] : li;
      thr32[g] = min((uint32_t)(thr >> 32), *bnd);
#pragma unroll
      for (int m = 0; m < 4; ++m) k32[g][m] = rowk(g, m);
    }
  }
  int npass[G];
  bool pass[G][4];
#pragma unroll
  for (int g = 0; g < G; ++g) {
    npass[g] = 0;
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      pass[g][m] = g < nvalid && k32[g][m] != 0xffffffffu && k32[g][m] <= thr32[g];
      npass[g] += __popc(__ballot_sync(MV_FULL, pass[g][m]));
    }
  }
  if (!fold) return;
#pragma unroll
  for (int g = 0; g < G; ++g) {
    if (npass[g] == 0) continue;
    uint64_t *L, *B;
    int* nb;
    uint32_t* bnd;
    uint64_t li;
    st(g, L, B, nb, bnd, li);
    warp_collect_passed(L, B, nb, bnd, k, li, k32[g], pass[g], npass[g], [&](int v) { return low(g, v); },
                        [&](uint32_t t) { publish(g, t); }, wscr, dc);
  }
}

// Buffered selection for 32 < k <= 32R (R = 2, 4): the sorted list L (k keys in smem) takes
// survivors through a 32-entry buffer B (count *nb), merged by sort-32 + a register bitonic merge
// when full (and by warp_flush_buffer_R at the end); a dense tile (> 32 survivors) is sorted as a
// whole and merged directly.  L[k-1] is always an exact bound of the k-th best seen so far.
template <int R>
__device__ __forceinline__ void warp_merge_into_list(uint64_t* L, int k, const uint64_t (&cand)[R]) {
  const int lane = threadIdx.x & 31;
  uint64_t lv[R];
#pragma unroll
  for (int r = 0; r < R; ++r) lv[r] = r * 32 + lane < k ? L[r * 32 + lane] : MV_KEY_PAD;
  warp_merge_smallest<R>(lv, cand);
  __syncwarp();
#pragma unroll
  for (int r = 0; r < R; ++r)
    if (r * 32 + lane < k) L[r * 32 + lane] = lv[r];
  __syncwarp();
}

template <int R>
__device__ __forceinline__ void warp_flush_buffer_R(uint64_t* L, uint64_t* B, int* nb, int k) {
  const int lane = threadIdx.x & 31;
  const int n = *nb;
  if (n == 0) return;
  uint64_t c[1] = {lane < n ? B[lane] : MV_KEY_PAD};
  if (!(c[0] < L[k - 1])) c[0] = MV_KEY_PAD;
  warp_bitonic_sort<1>(c);
  uint64_t cand[R];
  cand[0] = c[0];
#pragma unroll
  for (int r = 1; r < R; ++r) cand[r] = MV_KEY_PAD;
  warp_merge_into_list<R>(L, k, cand);
  if (lane == 0) *nb = 0;
  __syncwarp();
}

template <int R, typename Low>
__device__ __forceinline__ void warp_collect_R(uint64_t* L, uint64_t* B, int* nb, int k, const uint32_t (&k32)[4],
                                               const bool (&pass)[4], int npass, Low low) {
  const int lane = threadIdx.x & 31;
  if (npass > 32) {
    warp_flush_buffer_R<R>(L, B, nb, k);
    const uint64_t lk = L[k - 1];
    uint64_t key[4];
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      key[m] = pass[m] ? (((uint64_t)k32[m] << 32) | low(m * 32 + lane)) : MV_KEY_PAD;
      if (!(key[m] < lk)) key[m] = MV_KEY_PAD;
    }
    warp_bitonic_sort<4>(key);
    uint64_t cand[R];
#pragma unroll
    for (int r = 0; r < R; ++r) cand[r] = key[r];  // the smallest 32R of the sorted 128
    warp_merge_into_list<R>(L, k, cand);
    return;
  }
  if (*nb + npass > 32) warp_flush_buffer_R<R>(L, B, nb, k);
  int off = *nb;
#pragma unroll
  for (int m = 0; m < 4; ++m) {
    const uint32_t bm = __ballot_sync(MV_FULL, pass[m]);
    if (pass[m]) B[off + __popc(bm & ((1u << lane) - 1))] = ((uint64_t)k32[m] << 32) | low(m * 32 + lane);
    off += __popc(bm);
  }
  __syncwarp();
  if (lane == 0) *nb = off;
  __syncwarp();
}

// Block-wide bitonic sort of n (power of two) u64 keys in shared memory, ascending.
__device__ __forceinline__ void block_bitonic_sort(uint64_t* a, int n) {
  for (int size = 2; size <= n; size <<= 1) {
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      __syncthreads();
      for (int t = threadIdx.x; t < (n >> 1); t += blockDim.x) {
        const int lo = 2 * t - (t & (stride - 1));
        const int hi = lo + stride;
        const bool up = ((lo & size) == 0);
        const uint64_t x = a[lo], y = a[hi];
        if ((x > y) == up) {
          a[lo] = y;
          a[hi] = x;
        }
      }
    }
  }
  __syncthreads();
}

__host__ __device__ __forceinline__ int next_pow2(int x) {
  int p = 1;
  while (p < x) p <<= 1;
  return p;
}

}  // namespace mv

// ------------------------------------------------------------------------------------------
// Host-side launchers (each .cu file owns its kernels).  All enqueue on `st` and return the
// cudaError_t of the launch.
// ------------------------------------------------------------------------------------------
namespace mv {

// k_add.cu
cudaError_t launch_sq8_minmax(const float* x, int64_t n, int d, float* vmin, float* vdiff, cudaStream_t st);
cudaError_t launch_prep_rows(const float* x, int64_t n, int d, int dpad, float* out, cudaStream_t st);
cudaError_t launch_count_lists(const int32_t* lists, int64_t n, int32_t* counts, cudaStream_t st);
cudaError_t launch_store_rows(int type, int metric, const float* xpad, const int64_t* ids, const int32_t* sorted_idx,
                              const int32_t* sorted_list, int64_t n, int dpad, const int64_t* new_off,
                              const int64_t* old_off, const int32_t* add_off, void* payload, double* norms,
                              int64_t* out_ids, const float* vmin, const float* vdiff, const float* sq8_t,
                              cudaStream_t st);
cudaError_t launch_move_old(int type, int dpad, int nlist, const int64_t* old_off, const int64_t* new_off,
                            const void* old_payload, const double* old_norms, const int64_t* old_ids,
                            int64_t old_n, void* payload, double* norms, int64_t* ids, cudaStream_t st);
cudaError_t launch_id_keys(const int64_t* ids, int64_t n, uint64_t* keys, uint32_t* vals, cudaStream_t st);
cudaError_t launch_rank_scatter(const uint64_t* skeys, const uint32_t* svals, int64_t n, uint32_t* rank,
                                int64_t* sorted_ids, cudaStream_t st);
cudaError_t launch_check_ids(const int64_t* ids, int64_t n, int* flag, cudaStream_t st);
cudaError_t launch_new_sizes(const int32_t* add, int nlist, const int64_t* old_off, int64_t* out, cudaStream_t st);
cudaError_t launch_iota_i32(int32_t* out, int64_t n, cudaStream_t st);

// k_coarse.cu
cudaError_t launch_query_prep(const float* q, int64_t nq, int d, int dpad, float* qpad, float* qnorm, cudaStream_t st);
cudaError_t launch_centroid_prep(const float* c, int nlist, int d, int dpad, float* cpad, float* cnorm, cudaStream_t st);
cudaError_t launch_coarse(const float* qpad, int64_t nq, int dpad, const float* cpad, const float* cnorm, int nlist,
                          int metric, int nprobe, int32_t* probes, cudaStream_t st);

// k_bucket.cu
struct Bucketing {
  int32_t* lcount;   // nlist      pairs per list
  int32_t* boff;     // nlist+1    exclusive scan of lcount
  int32_t* bfill;    // nlist      scratch
  int32_t* bq;       // nq*npb (x2 with seeding)  pair ids grouped by list
  int32_t* wcount;   // nlist      work items per list
  int32_t* woff;     // nlist+1
  int2* witems;      // <= nlist + nq*npb   (list, first bucket position), longest first
  int2* witems_unsorted;
  int64_t* qtot;     // nq+1       per-query candidate capacity, then exclusive scan
  int64_t* poff;     // nq*npb (x2 with seeding: phase-A entries at nq*npb + p)  region offset per pair
  int32_t* pcnt;     // nq*npb (x2 with seeding)  candidates written per pair
  int32_t* counter;  // 1          persistent scan work counter
  int32_t* whist;    // kPlanCostBins  work-item cost histogram, then its exclusive scan
  int64_t* bsum;     // 2 x kPlanMaxBlocks  per-block partial sums of the grid-wide scans
};
constexpr int kPlanCostBins = 8192;
constexpr int kPlanMaxBlocks = 1024;
// a4 in one cooperative launch (k_bucket.cu).  With the seeding split the pairs of query q with
// probe rank < ra[q] form a first phase (virtual lists 0..nlist-1, work items first) and the
// others a second (virtual lists nlist..2*nlist-1); arrays are then sized for 2*nlist lists.
struct PlanArgs {
  const int32_t* probes;   // nq x npb, best-first
  int64_t nq;
  int npb, nlist, k, capk;  // capk > 0: SIMT local-selection regions min(capk, |list|); 0: |list|
  int split;               // 1: seeding phase (ra[q] nearest lists) + phase B
  int64_t need;            // seeding: candidates the phase-A lists must hold
  int64_t capA;            // seeding: phase A scans the first min(|l|, capA) rows of each of its lists
  const int64_t* list_off;
  const int* qlo_any;      // FLAT: some query needs its lo plane (nullable)
  int qc_exact, p_exact, qc_split, p_split;
  int32_t* qcfg;           // out: {query chunk, planes}
  int32_t* ra;             // out (split): nq
  Bucketing b;             // out
};
cudaError_t launch_plan(const PlanArgs& a, cudaStream_t st);
// single-CTA exclusive scans (the add path): out[0..n], out[n] = total
cudaError_t launch_scan_i32(const int32_t* in, int n, int32_t* out, cudaStream_t st);   // out[n+1]
cudaError_t launch_scan_i64(const int64_t* in, int64_t n, int64_t* out, cudaStream_t st);  // out[n+1]

// k_scan.cu
struct ScanArgs {
  int type, metric, d, dpad, k, npb, qchunk, nlist;
  const int64_t* list_off;
  const void* payload;
  const double* norms;
  const int64_t* ids;
  const uint32_t* rank;
  const uint8_t* bitset;
  int64_t nbits;
  const float* qpad;
  const float* qnorm;
  const float* vmin;
  const float* vdiff;
  const float* sq8_t;  // 256-entry decode table t_c = (c + 0.5f) / 255.f
  const int32_t* bq;
  const int32_t* boff;
  const int2* witems;
  const int32_t* nwitems;  // device: woff[nlist]
  int32_t* counter;
  const int64_t* poff;
  int32_t* pcnt;
  uint64_t* part;
};
cudaError_t launch_scan(const ScanArgs& a, cudaStream_t st);

// k_scan_tc.cu (tcgen05 path): a filter-and-emit scan run in two phases
struct TcScanParams {
  int type, metric, dpad, k, npb, qchunk, nchunks, nstage, ncol, tmem_cols, nacc, atom;
  int qchunk_split;        // FLAT: queries per work item when the queries need the lo plane (P = 2)
  const int32_t* cfg;      // device {query chunk, planes} of this search (launch_scan_cfg)
  int nlist;               // virtual list v >= nlist is list v - nlist (phase-B pairs)
  int phase;               // 0: seeding phase A (emit every candidate); 1: phase B (emit keys <= tau_q)
  int rowcap;              // rows scanned per list in this launch (phase A: capA; else INT_MAX)
  int64_t nq;              // FLAT query planes are plane-major [2][nq][dpad]
  int off_x, off_q, q_bytes, off_meta, meta_bytes, off_side, off_bar, smem_total;
  const int64_t* list_off;
  const double* norms;     // ||x||^2 (FLAT) or ||x_hat||^2 (SQ8), fp64
  const int64_t* ids;
  const uint32_t* rank;
  const uint8_t* bitset;
  int64_t nbits;
  const uint8_t* qplanes;  // nq x P x dpad (fp32 hi/lo planes or int8 digit planes)
  const double* qnorm;     // ||q||^2 fp64
  const float* qscale;
  const double* qa;        // SQ8: q.a fp64
  const int32_t* bq;
  const int32_t* boff;
  const int2* witems;
  const int32_t* wbeg;     // device: first work item of this launch (nullable = 0)
  const int32_t* nwitems;  // device: one past the last work item of this launch
  const int64_t* poff;     // per pair: output region (capacity = the list length)
  int32_t* pcnt;           // per pair: keys emitted
  uint64_t* part;
  const uint64_t* tau;     // nq: per-query bound for phase B (exact k-th key of phase A)
  int dbg;                 // debug bitmask (MV_SCAN_DEBUG): 1 skip emission, 2 skip epilogue math, 4 skip Q copy
  unsigned long long* prof;  // MV_SCAN_TRACE timeline (CTA 0)
};
bool tc_scan_plan(int type, int dpad, int k, double qpl, TcScanParams& p);  // qpl: expected queries per probed list
// the payload's tensor maps: boxes of 128, 64, 32, 16 rows (one swizzle atom wide)
struct XMaps {
  CUtensorMap m[4];
};
cudaError_t launch_scan_tc(const XMaps& xm, const TcScanParams& p, cudaStream_t st);
// k_scan_qm.cu: FLAT scan with the queries on the MMA's M side (xmap: 128-row boxes, xmap16: 16-row boxes)
bool qm_scan_plan(int dpad, int k, TcScanParams& p);
cudaError_t launch_scan_qm(const CUtensorMap* xmap, const CUtensorMap* xmap16, const TcScanParams& p, cudaStream_t st);
cudaError_t launch_qplanes(int type, const float* qpad, int64_t nq, int dpad, const float* vmin, const float* vdiff,
                           uint8_t* out, float* qscale, double* qa, double* qnorm, cudaStream_t st);
cudaError_t launch_tf32_check(const float* x, int64_t n, int* flag, cudaStream_t st);

// k_coarse_tc.cu (tcgen05 coarse GEMM -> score matrix S, then a warp-per-query top-nprobe)
struct CoarseParams {
  int64_t nq;
  int nlist, nchunks, nstage, nprobe, nqb, csplit, tmem_cols, metric, smem_total;
  int nepi, nacc;          // epilogue warps (multiple of 4, <= 16), TMEM accumulators (<= 4)
  int dbg;                 // MV_COARSE_DEBUG: 2 skip the epilogue, 4 skip the S stores (timing only)
  const float* cnorm;
  float* S;                // nq x lds scores (lds = roundup(nlist, 4))
  int64_t lds;
  uint32_t* G;             // nq x ldg: minimum score key of each 32-centroid group (ldg = ceil(nlist/32))
  int64_t ldg;
  const int* qlo_any;      // device: some query needs its lo plane (nullable = yes)
  int32_t* probes;
};
bool coarse_tc_plan(int dpad, int nprobe, int64_t nq, int nlist, int nsm, CoarseParams& p);
cudaError_t launch_coarse_tc(const CUtensorMap* cmap, const CUtensorMap* qmap, const CoarseParams& p, int64_t nq,
                             cudaStream_t st);
// plane-major tf32 split of n rows; *lo_any (nullable) |= 1 when some lo element is nonzero
cudaError_t launch_hilo(const float* x, int64_t n, int d, int dpad, float* out, int* lo_any, cudaStream_t st);

// k_select.cu
// final select over the pairs of each query; with tau != nullptr instead: tau[q] = the k-th best
// key over the first nuse[q] pairs of query q (left untouched when they hold fewer than k).
// tmax bounds the candidates of one query; over (nq bytes, nullable) is scratch for k > 256.
cudaError_t launch_final_select(const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq, int npb,
                                int k, int metric, const int64_t* sorted_ids, float* out_d, int64_t* out_i,
                                int64_t tmax, uint8_t* over, cudaStream_t st);
cudaError_t launch_tau_select(const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq, int npb,
                              const int32_t* nuse, int k, uint64_t* tau, int64_t tmax, uint8_t* over,
                              cudaStream_t st);
cudaError_t launch_fill_pad(int64_t n, int metric, float* d, int64_t* i, cudaStream_t st);
cudaError_t launch_merge2(int metric, const float* ad, const int64_t* ai, const float* bd, const int64_t* bi,
                          int64_t nq, int k, float* od, int64_t* oi, cudaStream_t st);

}  // namespace mv
