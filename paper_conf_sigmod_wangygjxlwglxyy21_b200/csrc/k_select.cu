// k_select.cu -- §8 rows a7 (per-query final select/merge, k <= 16384, id map, ordering,
// padding) and a8's on-device merge of per-shard results.
//
// PAPER.md:734-761 (§3.3): Faiss' GPU k-selection stops at k = 1024 (shared memory); Milvus
// reaches k <= 16384 by rounds of 1024 that filter out d < d_l and the recorded ties.  Here one
// pass reaches the same set (it is the plain top-k): an MSB radix select over the
// u64 candidate keys (distance key, id rank) finds the k-th key; everything below it is kept,
// the boundary digit bucket is sorted in shared memory, and the k winners are bitonic-sorted.
// Keys are unique (the id rank is a permutation), so ties are impossible at the key level and the
// result is exactly "sort by (distance, id, row), take k".
#include "mv_internal.cuh"

namespace mv {

constexpr int kBoundCap = 4096;   // boundary-bucket capacity (u64) for the radix path
constexpr int kUnroll = 4;        // warp selects: 32-key chunks loaded per round

// the id of a key's rank: sorted_ids[rank], or the rank itself when the index's ids are exactly
// 0..ntotal-1 (the caller passes sorted_ids = nullptr: no random 8-byte gather per result)
__device__ __forceinline__ int64_t rank_to_id(const int64_t* __restrict__ sorted_ids, uint64_t key) {
  const uint32_t r = (uint32_t)(key & 0xffffffffu);
  return sorted_ids ? __ldg(sorted_ids + r) : (int64_t)r;
}

__device__ __forceinline__ bool seg_locate(const int32_t* s_pre, int npb, int idx, int& j) {
  // binary search: largest j with s_pre[j] <= idx
  int lo = 0, hi = npb - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (s_pre[mid] <= idx) lo = mid; else hi = mid - 1;
  }
  j = lo;
  return true;
}

__global__ void __launch_bounds__(256) k_final_select(const int64_t* __restrict__ poff, const int32_t* __restrict__ pcnt,
                                                      const uint64_t* __restrict__ part, int64_t nq, int npb, int k,
                                                      int metric, const int64_t* __restrict__ sorted_ids, float* out_d,
                                                      int64_t* out_i, int selcap, const int32_t* __restrict__ nuse,
                                                      uint64_t* tau_out, const uint8_t* __restrict__ only,
                                                      const int* __restrict__ gate) {
  if (gate && *gate == 0) return;         // approximate-mode work, not needed by this search
  if (only && !only[blockIdx.x]) return;  // handled by k_final_big
  extern __shared__ __align__(16) uint8_t smem[];
  uint64_t* sel = reinterpret_cast<uint64_t*>(smem);       // selcap
  uint64_t* bnd = sel + selcap;                             // kBoundCap
  int32_t* s_pre = reinterpret_cast<int32_t*>(bnd + kBoundCap);  // npb + 1
  uint32_t* hist = reinterpret_cast<uint32_t*>(s_pre + npb + 1);  // 256
  int32_t* s_int = reinterpret_cast<int32_t*>(hist + 256);        // misc
  uint64_t* s_u64 = reinterpret_cast<uint64_t*>(s_int + 8);       // misc (8-aligned below)

  const int64_t q = blockIdx.x;
  const int tid = threadIdx.x;
  const int64_t* po = poff + q * npb;
  const int32_t* pc = pcnt + q * npb;
  if (nuse) npb = nuse[q];  // the first nuse[q] pairs of the query (the seeding phase's), else all
  if (tid == 0) {
    int acc = 0;
    for (int j = 0; j < npb; ++j) {
      s_pre[j] = acc;
      acc += pc[j];
    }
    s_pre[npb] = acc;
  }
  __syncthreads();
  const int T = s_pre[npb];
  int nout = min(T, k);

  if (T <= selcap) {
    const int N = next_pow2(max(T, 2));
    for (int i = tid; i < N; i += 256) {
      uint64_t v = MV_KEY_PAD;
      if (i < T) {
        int j;
        seg_locate(s_pre, npb, i, j);
        v = part[po[j] + (i - s_pre[j])];
      }
      sel[i] = v;
    }
    block_bitonic_sort(sel, N);
  } else {
    // ---- MSB radix select of the k smallest of T keys (T > selcap >= k) ----
    uint64_t pfx = 0;
    int fixed = 0, need = k;
    for (;;) {
      for (int i = tid; i < 256; i += 256) hist[i] = 0;
      __syncthreads();
      const int sh = 64 - fixed - 8;
      for (int i = tid; i < T; i += 256) {
        int j;
        seg_locate(s_pre, npb, i, j);
        const uint64_t x = part[po[j] + (i - s_pre[j])];
        if (fixed == 0 || (x >> (64 - fixed)) == pfx) atomicAdd(hist + ((x >> sh) & 0xff), 1u);
      }
      __syncthreads();
      if (tid == 0) {
        uint32_t cum = 0;
        int b = 0;
        for (; b < 256; ++b) {
          if (cum + hist[b] >= (uint32_t)need) break;
          cum += hist[b];
        }
        s_int[0] = b;
        s_int[1] = need - (int)cum;
        s_int[2] = (int)hist[b];
      }
      __syncthreads();
      const int b = s_int[0];
      need = s_int[1];
      pfx = (pfx << 8) | (uint64_t)b;
      fixed += 8;
      const int inb = s_int[2];
      __syncthreads();
      if (inb <= kBoundCap || fixed == 64) break;
    }
    // gather: below the prefix -> sel (exactly k - need of them); equal -> bnd
    if (tid == 0) { s_int[3] = 0; s_int[4] = 0; }
    __syncthreads();
    const int sh = 64 - fixed;
    for (int i = tid; i < T; i += 256) {
      int j;
      seg_locate(s_pre, npb, i, j);
      const uint64_t x = part[po[j] + (i - s_pre[j])];
      const uint64_t top = sh == 0 ? x : (x >> sh);
      if (top < pfx) sel[atomicAdd(s_int + 3, 1)] = x;
      else if (top == pfx) {
        const int pos = atomicAdd(s_int + 4, 1);
        if (pos < kBoundCap) bnd[pos] = x;
      }
    }
    __syncthreads();
    const int nb = min(s_int[4], kBoundCap);
    const int NB = next_pow2(max(nb, 2));
    for (int i = nb + tid; i < NB; i += 256) bnd[i] = MV_KEY_PAD;
    block_bitonic_sort(bnd, NB);
    const int below = s_int[3];
    for (int i = tid; i < need; i += 256) sel[below + i] = bnd[i];
    const int N = next_pow2(max(k, 2));
    for (int i = k + tid; i < N; i += 256) sel[i] = MV_KEY_PAD;
    block_bitonic_sort(sel, N);
    nout = k;
  }
  (void)s_u64;
  if (tau_out) {  // seeding: the k-th best key of the first nuse pairs bounds the query's top-k
    if (tid == 0 && nout == k) tau_out[q] = sel[k - 1];
    return;
  }
  for (int i = tid; i < k; i += 256) {
    float dv;
    int64_t iv;
    if (i < nout && sel[i] != MV_KEY_PAD) {
      const uint64_t key = sel[i];
      dv = key_dist((uint32_t)(key >> 32), metric);
      iv = rank_to_id(sorted_ids, key);
    } else {
      dv = metric == MV_L2 ? __int_as_float(0x7f800000) : __int_as_float(0xff800000);
      iv = -1;
    }
    out_d[q * k + i] = dv;
    out_i[q * k + i] = iv;
  }
}


// 256 < k: the CTA-per-query select's block size (32 warps: one CTA per SM when the candidate stage
// takes all of shared memory, so the warps are the only latency hiding) and private histograms
constexpr int kBigThreads = 1024;
constexpr int kHistWarps = 8;  // private radix histograms (warps w, w + 8, ... share one)

// Ascending bitonic sort of NK = kBigThreads E keys in shared memory by a kBigThreads block.  Warp w holds
// the contiguous block [32 E w, 32 E (w + 1)) in registers, lane l element 32 j + l in v[j]:
// strides < 32 are shuffles, strides 32 .. 16 E register pairs, larger strides go through shared
// memory (10 of the 66 stages for NK = 2048).  Pair (lo, lo + stride) of a size-`size` stage
// is ascending when (lo & size) == 0: the lower element keeps the minimum.
template <int E, int NT = kBigThreads>
__device__ __forceinline__ void block_sort_regs(uint64_t* win, int NK) {
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int wbase = wid * 32 * E;
  uint64_t v[E > 0 ? E : 1];
  constexpr int SMIN = E > 0 ? 32 * E : 1;  // smallest stride done in shared memory
  __syncthreads();
#pragma unroll
  for (int j = 0; j < E; ++j) v[j] = win[wbase + 32 * j + lane];
  for (int size = 2; size <= NK; size <<= 1) {
    int stride = size >> 1;
    if (stride >= SMIN) {
#pragma unroll
      for (int j = 0; j < E; ++j) win[wbase + 32 * j + lane] = v[j];
      for (; stride >= SMIN; stride >>= 1) {
        __syncthreads();
        for (int t = tid; t < (NK >> 1); t += NT) {
          const int lo = 2 * t - (t & (stride - 1));
          const int hi = lo + stride;
          const bool up = (lo & size) == 0;
          const uint64_t x = win[lo], y = win[hi];
          if ((x > y) == up) {
            win[lo] = y;
            win[hi] = x;
          }
        }
      }
      __syncthreads();
#pragma unroll
      for (int j = 0; j < E; ++j) v[j] = win[wbase + 32 * j + lane];
    }
#pragma unroll
    for (int m = E / 2; m >= 1; m >>= 1) {
      if (stride == 32 * m) {
#pragma unroll
        for (int j = 0; j < E; ++j)
          if ((j & m) == 0) {
            const bool up = ((wbase + 32 * j + lane) & size) == 0;
            const uint64_t x = v[j], y = v[j | m];
            v[j] = up ? umin64(x, y) : umax64(x, y);
            v[j | m] = up ? umax64(x, y) : umin64(x, y);
          }
        stride >>= 1;
      }
    }
    for (; stride > 0; stride >>= 1) {
      const bool lower = (lane & stride) == 0;
#pragma unroll
      for (int j = 0; j < E; ++j) {
        const bool up = ((wbase + 32 * j + lane) & size) == 0;
        const uint64_t o = shfl_xor64(v[j], stride);
        v[j] = (lower == up) ? umin64(v[j], o) : umax64(v[j], o);
      }
    }
  }
#pragma unroll
  for (int j = 0; j < E; ++j) win[wbase + 32 * j + lane] = v[j];
}

// Bucket sort of n unique keys win[0..n), all in [mn, hi], by one NT-thread block: 2048 buckets
// of equal key width, a counting pass, a scan, a scatter into tmp, and each key's rank within its
// bucket (keys are unique: rank = the bucket's keys below it).  cnt: 2048 zeroed u32; misc: 33
// ints.  ~6 barriers and a few dozen instructions per key against a bitonic network's ~60
// compare-exchange stages; false (win untouched) when a bucket holds more than kBucketMax keys
// (piles of keys within a narrow key range), for the caller's bitonic sort.
constexpr int kBucketBins = 2048, kBucketMax = 256;
static_assert(kBucketBins == kHistWarps * 256, "the bucket sort reuses the radix histograms");
// Exclusive scan, in place, of the kBucketBins counts cnt[] by an NT-thread block (misc: >= 32
// ints of scratch; misc[40..43) gets the bucket holding rank r -- its index, start and count --
// when 0 <= r < the total).  Ends with a barrier.
template <int NT>
__device__ void block_scan_bins(uint32_t* cnt, int* misc, int r) {
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  constexpr int PER = kBucketBins / NT;
  uint32_t v[PER], sum = 0;
#pragma unroll
  for (int j = 0; j < PER; ++j) {
    v[j] = cnt[tid * PER + j];
    sum += v[j];
  }
  uint32_t incl = sum;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t u = __shfl_up_sync(MV_FULL, incl, o);
    if (lane >= o) incl += u;
  }
  if (lane == 31) misc[wid] = (int)incl;
  __syncthreads();
  if (wid == 0) {
    uint32_t t = lane < NT / 32 ? (uint32_t)misc[lane] : 0u;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t u = __shfl_up_sync(MV_FULL, t, o);
      if (lane >= o) t += u;
    }
    __syncwarp();
    misc[lane] = (int)t;
  }
  __syncthreads();
  uint32_t run = (wid ? (uint32_t)misc[wid - 1] : 0u) + incl - sum;
#pragma unroll
  for (int j = 0; j < PER; ++j) {
    if (r >= 0 && run <= (uint32_t)r && (uint32_t)r < run + v[j]) {
      misc[40] = tid * PER + j;
      misc[41] = (int)run;
      misc[42] = (int)v[j];
    }
    cnt[tid * PER + j] = run;
    run += v[j];
  }
  __syncthreads();
}

template <int NT>
__device__ bool block_bucket_sort(uint64_t* win, int n, uint64_t mn, uint64_t hi, uint32_t* cnt, uint64_t* tmp,
                                  int* misc) {
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const uint64_t range = hi - mn;
  const int sh = max(0, 64 - __clzll((long long)range) - 11);  // (x - mn) >> sh < 2048
  if (tid == 0) misc[32] = 0;
  __syncthreads();
  int mx = 0;
  for (int i = tid; i < n; i += NT) mx = max(mx, (int)atomicAdd(cnt + ((win[i] - mn) >> sh), 1u) + 1);
  mx = __reduce_max_sync(MV_FULL, mx);
  if (lane == 0) atomicMax(misc + 32, mx);
  __syncthreads();
  if (misc[32] > kBucketMax) {
    for (int i = tid; i < kBucketBins; i += NT) cnt[i] = 0;
    __syncthreads();
    return false;
  }
  block_scan_bins<NT>(cnt, misc, -1);
  for (int i = tid; i < n; i += NT) {
    const uint64_t x = win[i];
    tmp[atomicAdd(cnt + ((x - mn) >> sh), 1u)] = x;
  }
  __syncthreads();
  for (int i = tid; i < n; i += NT) {
    const uint64_t x = tmp[i];
    const int b = (int)((x - mn) >> sh);
    const int s0 = b ? (int)cnt[b - 1] : 0, e0 = (int)cnt[b];
    int r = 0;
    for (int j = s0; j < e0; ++j) r += tmp[j] < x ? 1 : 0;
    win[s0 + r] = x;
  }
  __syncthreads();
  return true;
}

// 256 < k: one CTA (kBigThreads threads) per query stages the query's candidates in shared memory (when
// they fit, else it flags the query for k_final_select's global-memory path), then an MSB radix
// select over the u64 keys -- 8-bit digits, histogram per pass in shared memory, stopping as soon
// as the keys at or below the current prefix are exactly k -- and a bitonic sort of the k winners.

template <int NT>
__global__ void __launch_bounds__(NT, 2048 / NT) k_final_big(const int64_t* __restrict__ poff,
                                                           const int32_t* __restrict__ pcnt,
                                                           const uint64_t* __restrict__ part, int64_t nq, int npb, int k,
                                                           int metric, const int64_t* __restrict__ sorted_ids,
                                                           float* out_d, int64_t* out_i, int cap,
                                                           const int32_t* __restrict__ nuse, uint64_t* tau_out,
                                                           uint8_t* over, const int* __restrict__ gate,
                                                           const uint8_t* only, uint64_t* kmin) {
  if (gate && *gate == 0) return;
  // only: the queries to do (k_final_sample's redo flags, or the flags of a smaller-stage launch --
  // then the same array as over: this CTA reads its flag before rewriting it)
  if (only && !only[blockIdx.x]) {
    if (threadIdx.x == 0) over[blockIdx.x] = 0;
    return;
  }
  extern __shared__ __align__(16) uint8_t smem[];
  const int NK = next_pow2(max(k, 2));
  uint64_t* buf = reinterpret_cast<uint64_t*>(smem);   // cap
  uint64_t* win = buf + cap;                           // NK + kBucketMax
  uint32_t* whist = reinterpret_cast<uint32_t*>(win + NK + kBucketMax);  // kHistWarps x 256
  uint64_t* s_mm = reinterpret_cast<uint64_t*>(whist + kHistWarps * 256);  // min, max
  int32_t* s_pre = reinterpret_cast<int32_t*>(s_mm + 2);  // npb + 1
  int32_t* s_int = s_pre + npb + 1;  // misc (128): [0..3) digit, [8..16) warp totals, [16..59) sort, [64..107) fast path
  const int64_t q = blockIdx.x;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int64_t* po = poff + q * npb;
  const int32_t* pc = pcnt + q * npb;
  const int nu = nuse ? nuse[q] : npb;
  if (wid == 0) {  // prefix of the pair counts, 32 pairs at a time
    int run = 0;
    for (int j0 = 0; j0 < nu; j0 += 32) {
      const int j = j0 + lane;
      const int c = j < nu ? pc[j] : 0;
      int incl = c;
      for (int o = 1; o < 32; o <<= 1) {
        const int v = __shfl_up_sync(MV_FULL, incl, o);
        if (lane >= o) incl += v;
      }
      if (j < nu) s_pre[j] = run + incl - c;
      run += __shfl_sync(MV_FULL, incl, 31);
    }
    if (lane == 0) s_pre[nu] = run;
  }
  for (int i = tid; i < kHistWarps * 256; i += NT) whist[i] = 0;
  if (tid == 0) {
    s_mm[0] = MV_KEY_PAD;
    s_mm[1] = 0;
  }
  __syncthreads();
  const int T = s_pre[nu];
  if (T > cap) {
    if (tid == 0) over[q] = 1;
    return;
  }
  if (tid == 0) over[q] = 0;
  // staging by fire-and-forget 8-B async copies: every lane keeps its loads in flight (a plain
  // load/store loop was latency-bound: one ~1 us global round trip per 32 keys per warp)
  for (int j = wid; j < nu; j += NT / 32) {
    const int c = s_pre[j + 1] - s_pre[j];
    const uint64_t* src = part + po[j];
    const uint32_t dst = (uint32_t)__cvta_generic_to_shared(buf + s_pre[j]);
    for (int i = lane; i < c; i += 32)
      asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(dst + 8 * i), "l"(src + i) : "memory");
  }
  asm volatile("cp.async.wait_all;" ::: "memory");
  __syncthreads();
  int nsel;              // winners to sort, in win[]
  bool sorted = false;   // ... already sorted (the bucket sort)
  uint64_t* res = win;   // the sorted winners
  if (T <= k) {
    for (int i = tid; i < NK; i += NT) win[i] = i < T ? buf[i] : MV_KEY_PAD;
    nsel = T;
  } else {
    // radix select over the bits below the keys' common prefix: the first digit starts at the
    // highest bit where the smallest and largest key differ (near-neighbour distance keys share
    // their top ~10 bits, which a fixed MSB digit would pile into one contended bin).  8-bit
    // digits, private histograms (warps w, w + 8, ... share one), a block-wide scan of the 256
    // bins; it stops as soon as the keys at or below the current prefix are exactly k (keys are
    // unique) -- or, for the seeding bound, at most k + k/64: any bound with >= k candidates at
    // or below it is valid, a looser one only lets phase B emit a few more keys
    uint64_t mn = MV_KEY_PAD, mx = 0;
    for (int i = tid; i < T; i += NT) {
      const uint64_t x = buf[i];
      mn = umin64(mn, x);
      mx = umax64(mx, x);
    }
    for (int o = 16; o > 0; o >>= 1) {
      mn = umin64(mn, shfl_xor64(mn, o));
      mx = umax64(mx, shfl_xor64(mx, o));
    }
    if (lane == 0) {
      atomicMin(reinterpret_cast<unsigned long long*>(s_mm), (unsigned long long)mn);
      atomicMax(reinterpret_cast<unsigned long long*>(s_mm + 1), (unsigned long long)mx);
    }
    if (tid == 0) s_int[120] = 0;
    __syncthreads();
    mn = s_mm[0];
    mx = s_mm[1];
    if (tau_out && kmin && tid == 0) kmin[q] = mn;  // the streaming final select's lower bin edge
    // Fast path: one counting pass over kBucketBins equal-width buckets of [mn, mx] and a scan
    // locate the bucket b* holding the k-th key.  Seeding: the bound is b*'s upper edge (or, when
    // b* holds more than 64 keys, the upper edge of the sub-bucket of a second counting pass over
    // b*'s keys).  Final select: the keys of buckets <= b* are scattered bucket-wise and each is
    // placed by its rank within its bucket -- the first k places are the sorted top-k; taken when
    // no bucket <= b* holds more than kBucketMax keys, else the radix select below.
    const int shv = max(0, 64 - __clzll((long long)(mx - mn)) - 11);
    for (int i = tid; i < T; i += NT) atomicAdd(whist + ((buf[i] - mn) >> shv), 1u);
    __syncthreads();
    {
      int* misc = s_int + 64;
      block_scan_bins<NT>(whist, misc, k - 1);
      const int bs = misc[40], st = misc[41], nb = misc[42];
      if (tau_out) {
        const uint64_t b0 = mn + ((uint64_t)bs << shv);  // b*'s first key value
        uint64_t edge = b0 + (shv ? (~0ull >> (64 - shv)) : 0ull);
        if (nb > 64 && shv > 0) {
          const int sh2 = max(0, shv - 11);
          for (int i = tid; i < kBucketBins; i += NT) whist[i] = 0;
          __syncthreads();
          for (int i = tid; i < T; i += NT) {
            const uint64_t x = buf[i];
            if ((int)((x - mn) >> shv) == bs) atomicAdd(whist + ((x - b0) >> sh2), 1u);
          }
          __syncthreads();
          block_scan_bins<NT>(whist, misc, k - 1 - st);
          edge = b0 + ((uint64_t)misc[40] << sh2) + (sh2 ? (~0ull >> (64 - sh2)) : 0ull);
        }
        if (tid == 0) tau_out[q] = edge < mn || edge > mx ? mx : edge;
        return;
      }
      // the largest bucket <= b*
      int mxc = 0;
      constexpr int PER = kBucketBins / NT;
#pragma unroll
      for (int j = 0; j < PER; ++j) {
        const int b = tid * PER + j;
        if (b < bs) mxc = max(mxc, (int)(whist[b + 1] - whist[b]));
      }
      if (tid == 0) mxc = max(mxc, nb);
      mxc = __reduce_max_sync(MV_FULL, mxc);
      if (lane == 0) atomicMax(s_int + 120, mxc);
      __syncthreads();
      if (s_int[120] <= kBucketMax) {
        for (int i = tid; i < T; i += NT) {  // bucket-wise scatter into win (st + nb <= k - 1 + kBucketMax)
          const uint64_t x = buf[i];
          const int b = (int)((x - mn) >> shv);
          if (b <= bs) win[atomicAdd(whist + b, 1u)] = x;
        }
        __syncthreads();
        for (int i = tid; i < st + nb; i += NT) {
          const uint64_t x = win[i];
          const int b = (int)((x - mn) >> shv);
          const int s0 = b ? (int)whist[b - 1] : 0, e0 = (int)whist[b];
          int r = 0;
          for (int j = s0; j < e0; ++j) r += win[j] < x ? 1 : 0;
          if (s0 + r < k) buf[s0 + r] = x;
        }
        __syncthreads();
        res = buf;
        nsel = k;
        sorted = true;
        goto output;
      }
    }
    for (int i = tid; i < kBucketBins; i += NT) whist[i] = 0;
    __syncthreads();
    int lo = 64 - __clzll((long long)(mn ^ mx));  // bits [lo, 64) are common to every key
    uint64_t pfx = lo >= 64 ? 0 : (mn >> lo);
    int below = 0;  // keys whose bits above lo are < pfx
    const uint32_t slack = tau_out ? (uint32_t)(k >> 6) : 0u;
    for (;;) {
      const int w = min(8, lo), sh = lo - w;
      const uint32_t dmask = (1u << w) - 1;
      uint32_t* hw = whist + (wid % kHistWarps) * 256;
      for (int i = tid; i < T; i += NT) {
        const uint64_t x = buf[i];
        if (lo >= 64 || (x >> lo) == pfx) atomicAdd(hw + ((uint32_t)(x >> sh) & dmask), 1u);
      }
      __syncthreads();
      // bin tid (< 256): its count over the private histograms (cleared for the next pass), a
      // warp scan, the warp totals, and the bin holding the k-th key
      uint32_t v = 0, incl = 0;
      if (tid < 256) {
#pragma unroll
        for (int h = 0; h < kHistWarps; ++h) {
          v += whist[h * 256 + tid];
          whist[h * 256 + tid] = 0;
        }
        incl = v;
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t u = __shfl_up_sync(MV_FULL, incl, o);
          if (lane >= o) incl += u;
        }
        if (lane == 31) s_int[8 + wid] = (int)incl;
      }
      __syncthreads();
      if (tid < 256) {
        uint32_t cum = (uint32_t)below + incl - v;  // keys before bin tid
        for (int w2 = 0; w2 < wid; ++w2) cum += (uint32_t)s_int[8 + w2];
        if (cum < (uint32_t)k && cum + v >= (uint32_t)k) {
          s_int[0] = tid;
          s_int[1] = (int)cum;
          s_int[2] = cum + v - (uint32_t)k <= slack;
        }
      }
      __syncthreads();
      pfx = (pfx << w) | (uint64_t)s_int[0];
      below = s_int[1];
      lo = sh;
      const bool done = s_int[2] || lo == 0;
      __syncthreads();
      if (done) break;
    }
    // winners: keys whose bits above lo are <= pfx (exactly k, or k..k+slack for the seeding bound)
    if (tau_out) {  // seeding: the bound is the winners' upper edge -- no key of the sample lies
                    // between it and the largest winner; no gather, no sort
      if (tid == 0) tau_out[q] = (pfx << lo) | (lo ? (~0ull >> (64 - lo)) : 0ull);
      return;
    }
    if (tid == 0) s_int[3] = 0;
    __syncthreads();
    for (int b0 = 0; b0 < T; b0 += NT) {  // ballot-aggregated appends (one atomic per warp)
      const int i = b0 + tid;
      const uint64_t x = i < T ? buf[i] : MV_KEY_PAD;
      const bool p = i < T && (lo >= 64 ? 0 : (x >> lo)) <= pfx;
      const uint32_t m = __ballot_sync(MV_FULL, p);
      int base = 0;
      if (lane == 0 && m) base = atomicAdd(s_int + 3, __popc(m));
      base = __shfl_sync(MV_FULL, base, 0);
      if (p) {
        win[base + __popc(m & ((1u << lane) - 1))] = x;
        // the output's id gather reads sorted_ids[rank] after the sort: start it now
        if (sorted_ids) asm volatile("prefetch.global.L2 [%0];" ::"l"(sorted_ids + (uint32_t)(x & 0xffffffffu)));
      }
    }
    __syncthreads();
    nsel = k;
    for (int i = k + tid; i < NK; i += NT) win[i] = MV_KEY_PAD;
    // the k winners lie in [mn, the prefix's upper edge]
    sorted = block_bucket_sort<NT>(win, k, mn, (pfx << lo) | (lo ? (~0ull >> (64 - lo)) : 0ull), whist, buf,
                                   s_int + 16);
  }
  __syncthreads();
  if (tau_out) {  // seeding with exactly k candidates: the largest
    if (nsel < k) return;
    uint64_t m = 0;
    for (int i = tid; i < k; i += NT) m = umax64(m, win[i]);
    for (int o = 16; o > 0; o >>= 1) m = umax64(m, shfl_xor64(m, o));
    if (lane == 0) buf[wid] = m;
    __syncthreads();
    if (tid == 0) {
      uint64_t mm = 0;
      for (int w = 0; w < NT / 32; ++w) mm = umax64(mm, buf[w]);
      tau_out[q] = mm;
    }
    return;
  }
  // else a bitonic sort of the NK winners: register-blocked (strides < 32 E by shuffles and in
  // registers, only the larger strides through shared memory)
  if (!sorted) switch (NK / NT) {
    case 1: block_sort_regs<1, NT>(win, NK); break;
    case 2: block_sort_regs<2, NT>(win, NK); break;
    case 4: block_sort_regs<4, NT>(win, NK); break;
    case 8:
      if constexpr (NT <= 512) {
        block_sort_regs<8, NT>(win, NK);
        break;
      }
      [[fallthrough]];
    default: block_sort_regs<0, NT>(win, NK); break;  // NK < 1024 or > 4096: shared memory only
  }
  __syncthreads();
output:
  for (int i = tid; i < k; i += NT) {
    float dv;
    int64_t iv;
    const uint64_t key = res[i];
    if (i < nsel && key != MV_KEY_PAD) {
      dv = key_dist((uint32_t)(key >> 32), metric);
      iv = rank_to_id(sorted_ids, key);
    } else {
      dv = metric == MV_L2 ? __int_as_float(0x7f800000) : __int_as_float(0xff800000);
      iv = -1;
    }
    out_d[q * k + i] = dv;
    out_i[q * k + i] = iv;
  }
}


// 256 < k <= 4096 (the common large-k case, configs[3]'s k = 2048): a sample-threshold select
// that reads each candidate key once and sorts only the k winners.  One CTA per query, no staging
// of the candidates (two CTAs share an SM):
//   1. kSamp keys at a uniform stride; the sample's js-th smallest distance key (js ~ 1.25 k kSamp
//      / T + 12, found by bisection with block counts) is a threshold t expected a little above the
//      k-th key;
//   2. one pass gathers the keys <= t (ballot-aggregated appends) into a window of wcap keys; when
//      k <= count <= wcap the window holds the top-k (else t moves, up to two more passes, and
//      failing that the query is flagged for the staged radix select k_final_big, exact for any
//      input);
//   3. the k-th key of the window by bisection (distance key, then the tied id ranks), the k
//      winners compacted, and a bitonic sort of those k alone (the seeding select stops at the
//      k-th key: no sort at all).
constexpr int kSamp = kBigThreads;
constexpr int kGU = 8;  // gather: keys per lane per step

// number of values in v[0..E) (per thread, masked by cnt) below `trial`, summed over the block
template <int E>
__device__ __forceinline__ int block_count_below(const uint32_t (&v)[E], int nv, uint32_t trial, int* cell) {
  int c = 0;
#pragma unroll
  for (int j = 0; j < E; ++j) c += (j < nv && v[j] < trial) ? 1 : 0;
  c = (int)__reduce_add_sync(MV_FULL, (uint32_t)c);
  __syncthreads();
  if (threadIdx.x == 0) *cell = 0;
  __syncthreads();
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(cell, c);
  __syncthreads();
  return *cell;
}

// the r-th smallest (1-based) of the u32 values held per thread (E each, nv valid): MSB bisection
template <int E>
__device__ __forceinline__ uint32_t block_select_u32(const uint32_t (&v)[E], int nv, int r, int* cell) {
  uint32_t b = 0;
  for (int bit = 31; bit >= 0; --bit) {
    const uint32_t trial = b | (1u << bit);
    if (block_count_below<E>(v, nv, trial, cell) < r) b = trial;
  }
  return b;
}

__global__ void __launch_bounds__(kBigThreads) k_final_sample(const int64_t* __restrict__ poff,
                                                              const int32_t* __restrict__ pcnt,
                                                              const uint64_t* __restrict__ part, int64_t nq, int npb,
                                                              int k, int metric, const int64_t* __restrict__ sorted_ids,
                                                              float* out_d, int64_t* out_i, int wcap,
                                                              const int32_t* __restrict__ nuse, uint64_t* tau_out,
                                                              uint8_t* redo, const int* __restrict__ gate) {
  if (gate && *gate == 0) return;
  extern __shared__ __align__(16) uint8_t smem[];
  const int NK = next_pow2(max(k, 2));
  uint64_t* win = reinterpret_cast<uint64_t*>(smem);  // wcap (<= 4 kBigThreads)
  uint64_t* top = win + wcap;                          // NK: the winners
  int32_t* s_pre = reinterpret_cast<int32_t*>(top + NK);  // npb + 1
  int32_t* s_int = s_pre + npb + 1;                    // misc (4)
  const int64_t q = blockIdx.x;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const uint32_t ltmask = (1u << lane) - 1;
  const int64_t* po = poff + q * npb;
  const int32_t* pc = pcnt + q * npb;
  const int nu = nuse ? nuse[q] : npb;
  if (wid == 0) {
    int run = 0;
    for (int j0 = 0; j0 < nu; j0 += 32) {
      const int j = j0 + lane;
      const int c = j < nu ? pc[j] : 0;
      int incl = c;
      for (int o = 1; o < 32; o <<= 1) {
        const int v = __shfl_up_sync(MV_FULL, incl, o);
        if (lane >= o) incl += v;
      }
      if (j < nu) s_pre[j] = run + incl - c;
      run += __shfl_sync(MV_FULL, incl, 31);
    }
    if (lane == 0) s_pre[nu] = run;
  }
  __syncthreads();
  const int T = s_pre[nu];
  if (tid == 0) redo[q] = 0;
  // gather every key <= t into win (first wcap of them); returns the number of keys <= t
  auto gather = [&](uint64_t t) {
    if (tid == 0) s_int[0] = 0;
    __syncthreads();
    for (int j = wid; j < nu; j += kBigThreads / 32) {
      const int c = s_pre[j + 1] - s_pre[j];
      const uint64_t* src = part + po[j];
      for (int i0 = 0; i0 < c; i0 += 32 * kGU) {  // kGU loads per lane in flight
        uint64_t x[kGU];
#pragma unroll
        for (int u = 0; u < kGU; ++u) {
          const int i = i0 + 32 * u + lane;
          x[u] = i < c ? __ldg(src + i) : MV_KEY_PAD;
        }
#pragma unroll
        for (int u = 0; u < kGU; ++u) {
          const bool p = i0 + 32 * u + lane < c && x[u] <= t;
          const uint32_t m = __ballot_sync(MV_FULL, p);
          if (m) {
            int base = 0;
            if (lane == 0) base = atomicAdd(s_int, __popc(m));
            base = __shfl_sync(MV_FULL, base, 0);
            const int pos = base + __popc(m & ltmask);
            if (p && pos < wcap) win[pos] = x[u];
          }
        }
      }
    }
    __syncthreads();
    return s_int[0];
  };
  int cnt;
  if (T <= wcap) {
    cnt = gather(MV_KEY_PAD);
  } else {
    uint32_t sv[1];
    {  // the uniform-stride sample: thread i takes candidate floor(i T / kSamp) (its distance key)
      const int pos = (int)((int64_t)tid * T / kSamp);
      int lo = 0, hi = nu - 1;
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (s_pre[mid] <= pos) lo = mid; else hi = mid - 1;
      }
      sv[0] = (uint32_t)(part[po[lo] + (pos - s_pre[lo])] >> 32);
    }
    int js = min(kSamp - 1, (int)((double)kSamp * k * 1.25 / T) + 12);
    int lo_ok = -1, hi_bad = kSamp;  // sample ranks known too low (< k keys) / too high (> wcap)
    cnt = -1;
    for (int attempt = 0; attempt < 3; ++attempt) {
      const uint32_t td = block_select_u32<1>(sv, 1, js + 1, s_int + 1);
      const int c = gather(((uint64_t)td << 32) | 0xffffffffull);
      if (c >= k && c <= wcap) {
        cnt = c;
        break;
      }
      if (c < k) lo_ok = js; else hi_bad = js;
      const int nj = c < k ? min(kSamp - 1, js + max(8, (js + 1) / 4)) : (lo_ok + js) / 2;
      if (nj == js || nj <= lo_ok || nj >= hi_bad) break;
      js = nj;
    }
    if (cnt < 0) {  // the staged radix select takes this query
      if (tid == 0) redo[q] = 1;
      return;
    }
  }
  const int n = min(cnt, wcap);
  int nsel = n;
  if (n > k) {
    // the k-th key of the window: its distance key by bisection, then the tied ranks
    constexpr int E = 4;  // wcap <= 4 kBigThreads
    uint32_t dv[E];
#pragma unroll
    for (int j = 0; j < E; ++j) dv[j] = j * kBigThreads + tid < n ? (uint32_t)(win[j * kBigThreads + tid] >> 32) : 0u;
    const int nv = (n - tid + kBigThreads - 1) / kBigThreads;
    const uint32_t dk = block_select_u32<E>(dv, nv, k, s_int + 1);
    const int below = block_count_below<E>(dv, nv, dk, s_int + 1);  // keys with a smaller distance key
    uint32_t rv[E];
#pragma unroll
    for (int j = 0; j < E; ++j)
      rv[j] = (j < nv && dv[j] == dk) ? (uint32_t)win[j * kBigThreads + tid] : 0xffffffffu;
    const uint32_t rk = block_select_u32<E>(rv, nv, k - below, s_int + 1);
    const uint64_t kth = ((uint64_t)dk << 32) | rk;
    if (tau_out) {
      if (tid == 0) tau_out[q] = kth;
      return;
    }
    // compact the k winners (keys are unique: exactly k are <= kth)
    if (tid == 0) s_int[0] = 0;
    __syncthreads();
    for (int j = 0; j < E; ++j) {
      const int i = j * kBigThreads + tid;
      const uint64_t x = i < n ? win[i] : MV_KEY_PAD;
      const bool p = i < n && x <= kth;
      const uint32_t m = __ballot_sync(MV_FULL, p);
      int base = 0;
      if (lane == 0 && m) base = atomicAdd(s_int, __popc(m));
      base = __shfl_sync(MV_FULL, base, 0);
      if (p) top[base + __popc(m & ltmask)] = x;
    }
    nsel = k;
  } else {
    if (tau_out) {  // fewer than k candidates: tau untouched; exactly k: the largest
      if (n == k) {
        uint64_t m = 0;
        for (int i = tid; i < n; i += kBigThreads) m = umax64(m, win[i]);
        for (int o = 16; o > 0; o >>= 1) m = umax64(m, shfl_xor64(m, o));
        if (lane == 0) top[wid] = m;
        __syncthreads();
        if (tid == 0) {
          for (int w = 1; w < kBigThreads / 32; ++w) m = umax64(m, top[w]);
          tau_out[q] = m;
        }
      }
      return;
    }
    for (int i = tid; i < n; i += kBigThreads) top[i] = win[i];
  }
  __syncthreads();
  for (int i = nsel + tid; i < NK; i += kBigThreads) top[i] = MV_KEY_PAD;
  switch (NK / kBigThreads) {
    case 1: block_sort_regs<1>(top, NK); break;
    case 2: block_sort_regs<2>(top, NK); break;
    case 4: block_sort_regs<4>(top, NK); break;
    default: block_sort_regs<0>(top, NK); break;
  }
  __syncthreads();
  for (int i = tid; i < k; i += kBigThreads) {
    float dv;
    int64_t iv;
    const uint64_t key = i < nsel ? top[i] : MV_KEY_PAD;
    if (key != MV_KEY_PAD) {
      dv = key_dist((uint32_t)(key >> 32), metric);
      iv = rank_to_id(sorted_ids, key);
    } else {
      dv = metric == MV_L2 ? __int_as_float(0x7f800000) : __int_as_float(0xff800000);
      iv = -1;
    }
    out_d[q * k + i] = dv;
    out_i[q * k + i] = iv;
  }
}

// 256 < k <= 4096 without staging the candidates: one CTA per query streams the query's keys from
// global memory (every pair's region read by one warp, coalesced) -- a few tens of KB of shared
// memory per CTA, so several CTAs per SM keep their loads in flight (k_final_big stages every
// candidate in shared memory first: one CTA per SM at configs[3]'s sizes, load and compute phases
// in series).  Keys are binned by their distance key into kBucketBins equal-width bins over
// [lo32, hi32] (keys outside go to the end bins):
//   TAU (the seeding select): lo/hi = the keys' min/max distance keys (pass 0); a counting pass and
//     a scan locate the bin b* of the k-th key; the bound is b*'s upper edge (with a second counting
//     pass over b*'s sub-bins when it holds > 64 keys) with every id rank: >= k candidates lie at or
//     below it.  kmin[q] = the smallest key (the final select's lower bin edge).
//   final: lo = kmin[q], hi = khi[q] (the seeding bound: phase B emits nothing above it); a
//     counting pass locates b*; a second pass gathers the keys of bins <= b* (the top-k and b*'s
//     rest, <= cap keys) into shared memory, a bucket sort (bitonic fallback) orders them, the first
//     k are the answer.  A query whose gathered keys exceed cap is flagged in redo[] for the staged
//     select.
template <int NT, bool TAU>
__global__ void __launch_bounds__(NT, TAU ? 1 : 3) k_select_stream(const int64_t* __restrict__ poff, const int32_t* __restrict__ pcnt,
                                                      const uint64_t* __restrict__ part, int64_t nq, int npb, int k,
                                                      int metric, const int64_t* __restrict__ sorted_ids, float* out_d,
                                                      int64_t* out_i, int cap, const int32_t* __restrict__ nuse,
                                                      uint64_t* tau_out, uint64_t* kmin, const uint64_t* __restrict__ khi,
                                                      uint8_t* redo, const int* __restrict__ gate) {
  if (gate && *gate == 0) return;
  extern __shared__ __align__(16) uint8_t smem[];
  uint32_t* hist = reinterpret_cast<uint32_t*>(smem);                 // kBucketBins
  int* misc = reinterpret_cast<int*>(hist + kBucketBins);             // 64
  uint64_t* s_mm = reinterpret_cast<uint64_t*>(misc + 64);            // 2
  int64_t* s_po = reinterpret_cast<int64_t*>(s_mm + 2);               // npb: the non-empty pairs' regions
  int32_t* s_pre = reinterpret_cast<int32_t*>(s_po + npb);            // npb + 33: their key prefix, then padding
  uint64_t* win = reinterpret_cast<uint64_t*>(s_pre + ((npb + 34) & ~1));  // cap (final)
  uint64_t* tmp = win + (TAU ? 0 : cap);                              // cap (final)
  constexpr int NW = NT / 32, U = 4;
  const int64_t q = blockIdx.x;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int64_t* po = poff + q * npb;
  const int32_t* pc = pcnt + q * npb;
  const int nu = nuse ? nuse[q] : npb;
  for (int i = tid; i < kBucketBins; i += NT) hist[i] = 0;
  if (wid == 0) {  // the non-empty pairs, compacted, and the prefix of their key counts
    int run = 0, ne = 0;
    for (int j0 = 0; j0 < nu; j0 += 32) {
      const int j = j0 + lane;
      const int c = j < nu ? pc[j] : 0;
      int incl = c;
      for (int o = 1; o < 32; o <<= 1) {
        const int v = __shfl_up_sync(MV_FULL, incl, o);
        if (lane >= o) incl += v;
      }
      const uint32_t nz = __ballot_sync(MV_FULL, c > 0);
      if (c > 0) {
        const int ci = ne + __popc(nz & ((1u << lane) - 1));
        s_pre[ci] = run + incl - c;
        s_po[ci] = po[j];
      }
      run += __shfl_sync(MV_FULL, incl, 31);
      ne += __popc(nz);
    }
    s_pre[ne + lane] = lane ? 0x7fffffff : run;  // s_pre[ne] = the total, then padding
    if (lane == 0) {
      misc[50] = ne;
      s_mm[0] = MV_KEY_PAD;
      s_mm[1] = 0;
      misc[48] = 0;
      misc[49] = 0;
    }
    s_pre[ne + 32] = 0x7fffffff;
  }
  __syncthreads();
  const int nne = misc[50];
  const int T = s_pre[nne];
  // every key of the query: warp w takes a contiguous slice of the flattened (pair, key) index, U
  // windows of 32 keys per round (independent loads in flight); a window's pair starts are found
  // by one shared load per lane and an OR-reduce (the pair starts strictly increase: empty pairs
  // were dropped).  f(x, valid) is called by all 32 lanes together.
  const int per = ((T + NW - 1) / NW + 31) & ~31;
  auto each = [&](auto&& f) {
    const int b0 = min(T, wid * per), b1 = min(T, b0 + per);
    int c0 = 0;  // pair starts below the window
    {
      int lo = 0, hi = nne;  // the first m with s_pre[m] >= b0
      while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (s_pre[mid] < b0) lo = mid + 1; else hi = mid;
      }
      c0 = lo;
    }
    const uint32_t upto = lane == 31 ? 0xffffffffu : (2u << lane) - 1;
    for (int i0 = b0; i0 < b1; i0 += 32 * U) {
      uint64_t x[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int w0 = i0 + 32 * u;
        const uint32_t off = (uint32_t)(s_pre[min(c0 + lane, nne + 32)] - w0);
        const uint32_t M = __reduce_or_sync(MV_FULL, off < 32u ? 1u << off : 0u);
        const int j = c0 - 1 + __popc(M & upto);
        c0 += __popc(M);
        const int i = w0 + lane;
        x[u] = i < b1 ? __ldg(part + s_po[j] + (i - s_pre[j])) : MV_KEY_PAD;
      }
#pragma unroll
      for (int u = 0; u < U; ++u) f(x[u], x[u] != MV_KEY_PAD);
    }
  };
  uint32_t lo32, hi32;
  if (TAU) {
    uint64_t mn = MV_KEY_PAD, mx = 0;
    each([&](uint64_t x, bool v) {
      if (v) {
        mn = umin64(mn, x);
        mx = umax64(mx, x);
      }
    });
    for (int o = 16; o > 0; o >>= 1) {
      mn = umin64(mn, shfl_xor64(mn, o));
      mx = umax64(mx, shfl_xor64(mx, o));
    }
    if (lane == 0) {
      atomicMin(reinterpret_cast<unsigned long long*>(s_mm), (unsigned long long)mn);
      atomicMax(reinterpret_cast<unsigned long long*>(s_mm + 1), (unsigned long long)mx);
    }
    __syncthreads();
    lo32 = (uint32_t)(s_mm[0] >> 32);
    hi32 = (uint32_t)(s_mm[1] >> 32);
    if (s_mm[0] == MV_KEY_PAD) lo32 = hi32 = 0;
  } else {
    lo32 = (uint32_t)(kmin[q] >> 32);
    hi32 = max(lo32, (uint32_t)(khi[q] >> 32));
  }
  const uint32_t span = hi32 - lo32;
  const int sh = span ? max(0, 32 - __clz((int)span) - 11) : 0;  // (d - lo32) >> sh < 2048
  auto bin = [&](uint64_t x) {
    const uint32_t d = (uint32_t)(x >> 32);
    return d <= lo32 ? 0 : (int)min((uint32_t)(kBucketBins - 1), (d - lo32) >> sh);
  };
  {
    int cnt = 0;
    each([&](uint64_t x, bool v) {
      if (v) {
        atomicAdd(hist + bin(x), 1u);
        ++cnt;
      }
    });
    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(MV_FULL, cnt, o);
    if (lane == 0) atomicAdd(misc + 49, cnt);
  }
  __syncthreads();
  const int ntot = misc[49];
  if (TAU) {
    if (ntot < k) {  // fewer than k candidates: no bound (tau stays at padding), the whole key range
      if (tid == 0 && kmin) kmin[q] = 0;
      return;
    }
    if (tid == 0 && kmin) kmin[q] = s_mm[0];
    block_scan_bins<NT>(hist, misc, k - 1);
    const int bs = misc[40], st = misc[41], nb = misc[42];
    // b*'s upper edge: the bins below b* hold < k keys, so the k-th key's distance is <= the edge
    uint64_t dedge = (uint64_t)lo32 + (((uint64_t)bs + 1) << sh) - 1;
    if (nb > 64 && sh > 0) {  // refine within b*: 2048 sub-bins of width 2^(sh - 11)
      const int sh2 = max(0, sh - 11);
      const uint32_t b0 = lo32 + ((uint32_t)bs << sh);
      for (int i = tid; i < kBucketBins; i += NT) hist[i] = 0;
      __syncthreads();
      each([&](uint64_t x, bool v) {
        if (v && bin(x) == bs) atomicAdd(hist + (int)((((uint32_t)(x >> 32)) - b0) >> sh2), 1u);
      });
      __syncthreads();
      block_scan_bins<NT>(hist, misc, k - 1 - st);
      dedge = (uint64_t)b0 + (((uint64_t)misc[40] + 1) << sh2) - 1;
    }
    if (tid == 0) tau_out[q] = umin64((dedge << 32) | 0xffffffffull, s_mm[1]);
    return;
  } else {
    // winners: the keys of bins <= b* (every key when there are at most k)
    int lim = kBucketBins, n = ntot;
    if (ntot > k) {
      block_scan_bins<NT>(hist, misc, k - 1);
      lim = misc[40];
      n = misc[41] + misc[42];
    }
    if (n > cap) {
      if (tid == 0) redo[q] = 1;
      return;
    }
    if (tid == 0) redo[q] = 0;
    each([&](uint64_t x, bool v) {
      const bool p = v && bin(x) <= lim;
      const uint32_t bal = __ballot_sync(MV_FULL, p);
      int base = 0;
      if (lane == 0 && bal) base = atomicAdd(misc + 48, __popc(bal));
      base = __shfl_sync(MV_FULL, base, 0);
      if (p) win[base + __popc(bal & ((1u << lane) - 1))] = x;
    });
    __syncthreads();
    const int ng = misc[48];
    uint64_t mn = MV_KEY_PAD, mx = 0;
    for (int i = tid; i < ng; i += NT) {
      mn = umin64(mn, win[i]);
      mx = umax64(mx, win[i]);
    }
    for (int o = 16; o > 0; o >>= 1) {
      mn = umin64(mn, shfl_xor64(mn, o));
      mx = umax64(mx, shfl_xor64(mx, o));
    }
    for (int i = tid; i < kBucketBins; i += NT) hist[i] = 0;
    if (tid == 0) {
      s_mm[0] = MV_KEY_PAD;
      s_mm[1] = 0;
    }
    __syncthreads();
    if (lane == 0) {
      atomicMin(reinterpret_cast<unsigned long long*>(s_mm), (unsigned long long)mn);
      atomicMax(reinterpret_cast<unsigned long long*>(s_mm + 1), (unsigned long long)mx);
    }
    __syncthreads();
    if (ng > 1 && !block_bucket_sort<NT>(win, ng, s_mm[0], s_mm[1], hist, tmp, misc)) {
      const int NK = next_pow2(max(ng, 2));
      for (int i = ng + tid; i < NK; i += NT) win[i] = MV_KEY_PAD;
      switch (NK / NT) {
        case 1: block_sort_regs<1, NT>(win, NK); break;
        case 2: block_sort_regs<2, NT>(win, NK); break;
        case 4: block_sort_regs<4, NT>(win, NK); break;
        case 8: block_sort_regs<8, NT>(win, NK); break;
        default: block_sort_regs<0, NT>(win, NK); break;
      }
    }
    __syncthreads();
    for (int i = tid; i < k; i += NT) {
      float dv;
      int64_t iv;
      if (i < ng) {
        const uint64_t key = win[i];
        dv = key_dist((uint32_t)(key >> 32), metric);
        iv = rank_to_id(sorted_ids, key);
      } else {
        dv = metric == MV_L2 ? __int_as_float(0x7f800000) : __int_as_float(0xff800000);
        iv = -1;
      }
      out_d[q * k + i] = dv;
      out_i[q * k + i] = iv;
    }
  }
}

// Seeding bound of a k > 256 search from 4-byte distance keys (phase A with key32): one CTA per
// query stages its sample (the ra nearest lists' keys) in shared memory, bins it into kBucketBins
// equal-width bins over [min, max] (a second counting pass over the k-th key's bin when it holds
// more than 64 keys) and returns that bin's upper edge with every id rank: >= k candidates lie at
// or below it.  kmin[q] = the smallest key (the streaming final select's lower bin edge).  A query
// with fewer than k sample keys, or more than `cap`, keeps tau = padding (phase B then emits every
// candidate of it; the final select's staged fallbacks take any count).
template <int NT>
__global__ void __launch_bounds__(NT) k_tau32(const int64_t* __restrict__ poff, const int32_t* __restrict__ pcnt,
                                             const uint32_t* __restrict__ part32, int64_t nq, int npb,
                                             const int32_t* __restrict__ nuse, int k, uint64_t* tau_out,
                                             uint64_t* kmin, int cap) {
  extern __shared__ __align__(16) uint8_t smem[];
  uint32_t* hist = reinterpret_cast<uint32_t*>(smem);   // kBucketBins
  int* misc = reinterpret_cast<int*>(hist + kBucketBins);  // 64
  int32_t* s_pre = misc + 64;                             // npb + 1
  uint32_t* keys = reinterpret_cast<uint32_t*>(s_pre + ((npb + 4) & ~3));  // cap
  const int64_t q = blockIdx.x;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int64_t* po = poff + q * npb;
  const int32_t* pc = pcnt + q * npb;
  const int nu = nuse ? nuse[q] : npb;
  for (int i = tid; i < kBucketBins; i += NT) hist[i] = 0;
  if (wid == 0) {
    int run = 0;
    for (int j0 = 0; j0 < nu; j0 += 32) {
      const int j = j0 + lane;
      const int c = j < nu ? pc[j] : 0;
      int incl = c;
      for (int o = 1; o < 32; o <<= 1) {
        const int v = __shfl_up_sync(MV_FULL, incl, o);
        if (lane >= o) incl += v;
      }
      if (j < nu) s_pre[j] = run + incl - c;
      run += __shfl_sync(MV_FULL, incl, 31);
    }
    if (lane == 0) {
      s_pre[nu] = run;
      misc[48] = (int)0xffffffff;  // min (as u32 via atomicMin on unsigned)
      misc[49] = 0;                // max
    }
  }
  __syncthreads();
  const int T = s_pre[nu];
  if (T < k || T > cap) {
    if (tid == 0 && kmin) kmin[q] = 0;
    return;
  }
  for (int j = wid; j < nu; j += NT / 32) {
    const int c = s_pre[j + 1] - s_pre[j];
    const uint32_t* src = part32 + po[j];
    const uint32_t dst = (uint32_t)__cvta_generic_to_shared(keys + s_pre[j]);
    for (int i = lane; i < c; i += 32)
      asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(dst + 4 * i), "l"(src + i) : "memory");
  }
  asm volatile("cp.async.wait_all;" ::: "memory");
  __syncthreads();
  uint32_t mn = 0xffffffffu, mx = 0;
  for (int i = tid; i < T; i += NT) {
    mn = min(mn, keys[i]);
    mx = max(mx, keys[i]);
  }
  mn = __reduce_min_sync(MV_FULL, mn);
  mx = __reduce_max_sync(MV_FULL, mx);
  if (lane == 0) {
    atomicMin(reinterpret_cast<unsigned*>(misc + 48), mn);
    atomicMax(reinterpret_cast<unsigned*>(misc + 49), mx);
  }
  __syncthreads();
  mn = (uint32_t)misc[48];
  mx = (uint32_t)misc[49];
  const uint32_t span = mx - mn;
  const int sh = span ? max(0, 32 - __clz((int)span) - 11) : 0;  // (x - mn) >> sh < 2048
  for (int i = tid; i < T; i += NT) atomicAdd(hist + ((keys[i] - mn) >> sh), 1u);
  __syncthreads();
  block_scan_bins<NT>(hist, misc, k - 1);
  const int bs = misc[40], st = misc[41], nb = misc[42];
  uint64_t edge = (uint64_t)mn + (((uint64_t)bs + 1) << sh) - 1;
  if (nb > 64 && sh > 0) {
    const int sh2 = max(0, sh - 11);
    const uint32_t b0 = mn + ((uint32_t)bs << sh);
    for (int i = tid; i < kBucketBins; i += NT) hist[i] = 0;
    __syncthreads();
    for (int i = tid; i < T; i += NT) {
      const uint32_t x = keys[i];
      if ((int)((x - mn) >> sh) == bs) atomicAdd(hist + ((x - b0) >> sh2), 1u);
    }
    __syncthreads();
    block_scan_bins<NT>(hist, misc, k - 1 - st);
    edge = (uint64_t)b0 + (((uint64_t)misc[40] + 1) << sh2) - 1;
  }
  if (tid == 0) {
    edge = min(edge, (uint64_t)mx);
    tau_out[q] = (edge << 32) | 0xffffffffull;
    if (kmin) kmin[q] = (uint64_t)mn << 32;
  }
}

cudaError_t launch_tau32(const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq, int npb,
                         const int32_t* nuse, int k, uint64_t* tau, uint64_t* kmin, int64_t tmax, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  constexpr int NT = 1024;
  const size_t fixed = kBucketBins * 4 + 64 * 4 + (size_t)((npb + 4) & ~3) * 4;
  // two CTAs per SM when the sample fits (configs[3]: need + capA ~ 17k keys), else all of it
  int cap = (int)min64(tmax, (int64_t)((112 * 1024 - fixed) / 4));
  if (cap < tmax) cap = (int)min64(tmax, (int64_t)((226 * 1024 - fixed) / 4));
  const size_t smem = fixed + (size_t)cap * 4;
  cudaError_t e = cudaFuncSetAttribute(k_tau32<NT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k_tau32<NT><<<(unsigned)nq, NT, smem, st>>>(poff, pcnt, reinterpret_cast<const uint32_t*>(part), nq, npb, nuse, k,
                                              tau, kmin, cap);
  return cudaGetLastError();
}

static cudaError_t launch_big_select(const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq,
                                     int npb, int k, int metric, const int64_t* sorted_ids, float* out_d,
                                     int64_t* out_i, const int32_t* nuse, uint64_t* tau, int64_t tmax,
                                     uint8_t* over, const int* gate, BigSel bsel, cudaStream_t st) {
  cudaError_t e;
  // over: 2 nq bytes -- [0, nq) queries past k_final_big's stage, [nq, 2 nq) the redo flags of the
  // first-choice select (streaming or sample-threshold)
  uint8_t* redo = over ? over + nq : nullptr;
  // streaming select: options only -- mode 3 for the seeding bound, mode 4 for the final select.
  // The staged select measured faster for both once the id gather went away (configs[3], ids
  // 0..n-1: final 0.75 ms staged vs 0.88-1.38 ms streaming, the latter with a large run-to-run
  // spread; seeding 0.63 vs 0.72 ms)
  if (k <= 4096 && (tau ? bsel.mode == 3 && bsel.kmin != nullptr : bsel.mode == 4 && bsel.kmin && bsel.khi && redo)) {
    constexpr int NT = 512;
    const size_t base = kBucketBins * 4 + 64 * 4 + 16 + (size_t)npb * 8 + (size_t)((npb + 34) & ~1) * 4;
    if (tau) {
      e = cudaFuncSetAttribute(k_select_stream<NT, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)base);
      if (e != cudaSuccess) return e;
      k_select_stream<NT, true><<<(unsigned)nq, NT, base, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d,
                                                               out_i, 0, nuse, tau, bsel.kmin, nullptr, nullptr, gate);
      return cudaGetLastError();
    }
    // the top-k plus the k-th key's bin (tens of keys); win + tmp also hold the bitonic fallback's
    // next_pow2(gathered) keys.  k = 2048: 52 KB per CTA, four CTAs per SM
    const int cap = k + max(256, k / 4);
    const size_t smem = base + (size_t)cap * 16;
    e = cudaFuncSetAttribute(k_select_stream<NT, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    k_select_stream<NT, false><<<(unsigned)nq, NT, smem, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d,
                                                              out_i, cap, nuse, nullptr, bsel.kmin, bsel.khi, redo, gate);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
  } else if (redo && k <= 3072 && bsel.mode == 1) {
    const int wcap = 4 * kBigThreads;  // >= k + the threshold's slack for k <= 2048; less for larger k
    const size_t smem = (size_t)(wcap + next_pow2(max(k, 2))) * 8 + (size_t)(npb + 1) * 4 + 64;
    if ((e = cudaFuncSetAttribute(k_final_sample, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) != cudaSuccess)
      return e;
    k_final_sample<<<(unsigned)nq, kBigThreads, smem, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d,
                                                            out_i, wcap, nuse, tau, redo, gate);
  } else {
    redo = nullptr;
  }
  const int NK = next_pow2(max(k, 2));
  const int fixed = (NK + kBucketMax) * 8 + kHistWarps * 256 * 4 + 16 + (npb + 1) * 4 + 128 * 4 + 64;
  const int64_t want = max64(tmax, k);  // stage capacity that holds every query
  const int capmax = (227 * 1024 - fixed) / 8;
  // first launch: `ctas` CTAs per SM (228 KB of shared memory per SM, 1 KB reserved per CTA), each
  // staging at most cap1 candidates; the queries past it are flagged and redone by a one-CTA-per-SM
  // launch with all of shared memory (then by k_final_select's global-memory path)
  const int ctas = bsel.ctas > 0 ? min(bsel.ctas, 4) : 2;
  int cap1 = (int)min64((228 * 1024 / ctas - 2048 - fixed) / 8, want);
  if (bsel.cap > 0) cap1 = (int)min64(cap1, max64(bsel.cap, k));
  const uint8_t* only = redo;
  if (over && (ctas > 1 || bsel.cap > 0) && cap1 >= k && cap1 < capmax && bsel.tlo <= cap1) {
    const size_t smem = (size_t)cap1 * 8 + fixed;
    if (ctas <= 2) {
      if ((e = cudaFuncSetAttribute(k_final_big<1024>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) !=
          cudaSuccess)
        return e;
      k_final_big<1024><<<(unsigned)nq, 1024, smem, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d,
                                                          out_i, cap1, nuse, tau, over, gate, only, bsel.kmin);
    } else {
      if ((e = cudaFuncSetAttribute(k_final_big<512>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) !=
          cudaSuccess)
        return e;
      k_final_big<512><<<(unsigned)nq, 512, smem, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d,
                                                        out_i, cap1, nuse, tau, over, gate, only, bsel.kmin);
    }
    if (want <= cap1) return cudaGetLastError();
    only = over;  // the next launch redoes the flagged queries alone
  }
  // all of shared memory, or just the bound tmax when that is smaller
  const int cap = (int)min64(capmax, want);
  if (over && cap >= k) {
    const size_t smem = (size_t)cap * 8 + fixed;
    e = cudaFuncSetAttribute(k_final_big<1024>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    k_final_big<1024><<<(unsigned)nq, 1024, smem, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d,
                                                        out_i, cap, nuse, tau, over, gate, only, bsel.kmin);
    if (want <= cap) return cudaGetLastError();
  } else {
    over = nullptr;
  }
  const int selcap = max(4096, next_pow2(k));
  size_t smem = (size_t)(selcap + kBoundCap) * 8 + (size_t)(npb + 1) * 4 + 256 * 4 + 8 * 4 + 64;
  e = cudaFuncSetAttribute(k_final_select, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k_final_select<<<(unsigned)nq, 256, smem, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d, out_i,
                                                  selcap, nuse, tau, over, gate);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------
// Filter mode's exact re-scoring: the oracle's badness of one stored row for a
// query held in registers by the warp -- fp64 from the fp32 query and the stored row (FLAT: the
// fp32 vector; SQ8: the codes decoded in fp32 in the oracle's order, vmin + ((c + 0.5)/255) vdiff;
// PAPER.md:290-294 §2.1), rounded to fp32.  Warp-cooperative: dims 4 (lane + 32 u) .. +3 per lane
// (dpad <= 512); every lane returns the result.
// ------------------------------------------------------------------------------------------
struct QueryRegs {
  float4 q[4], vm[4], vd[4];
};

template <int TYPE>
__device__ __forceinline__ void load_query_regs(QueryRegs& r, const float* qrow, int dpad, const float* vmin,
                                                const float* vdiff) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const bool in = 4 * (lane + 32 * u) < dpad;
    const float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
    r.q[u] = in ? reinterpret_cast<const float4*>(qrow)[lane + 32 * u] : z;
    if (TYPE == MV_IVF_SQ8) {
      r.vm[u] = in ? reinterpret_cast<const float4*>(vmin)[lane + 32 * u] : z;
      r.vd[u] = in ? reinterpret_cast<const float4*>(vdiff)[lane + 32 * u] : z;
    }
  }
}

template <int TYPE>
__device__ __forceinline__ float exact_badness(const QueryRegs& r, int64_t row, int dpad, bool l2, const void* payload,
                                               const float* __restrict__ sq8_t) {
  const int lane = threadIdx.x & 31;
  double acc = 0.0;
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    if (4 * (lane + 32 * u) < dpad) {
      float4 xv;
      if (TYPE == MV_IVF_FLAT) {
        xv = __ldg(reinterpret_cast<const float4*>(reinterpret_cast<const float*>(payload) + row * dpad) + lane + 32 * u);
      } else {  // the oracle's decode, fp32, one rounding per operation: (t_c * vdiff) + vmin
        const uint32_t cw =
            __ldg(reinterpret_cast<const uint32_t*>(reinterpret_cast<const uint8_t*>(payload) + row * dpad) + lane + 32 * u);
        xv.x = __fadd_rn(__fmul_rn(__ldg(sq8_t + (cw & 0xff)), r.vd[u].x), r.vm[u].x);
        xv.y = __fadd_rn(__fmul_rn(__ldg(sq8_t + ((cw >> 8) & 0xff)), r.vd[u].y), r.vm[u].y);
        xv.z = __fadd_rn(__fmul_rn(__ldg(sq8_t + ((cw >> 16) & 0xff)), r.vd[u].z), r.vm[u].z);
        xv.w = __fadd_rn(__fmul_rn(__ldg(sq8_t + (cw >> 24)), r.vd[u].w), r.vm[u].w);
      }
      if (l2) {
        const double a = (double)r.q[u].x - xv.x, b = (double)r.q[u].y - xv.y;
        const double c = (double)r.q[u].z - xv.z, d = (double)r.q[u].w - xv.w;
        acc = fma(a, a, acc); acc = fma(b, b, acc); acc = fma(c, c, acc); acc = fma(d, d, acc);
      } else {
        acc = fma((double)r.q[u].x, (double)xv.x, acc); acc = fma((double)r.q[u].y, (double)xv.y, acc);
        acc = fma((double)r.q[u].z, (double)xv.z, acc); acc = fma((double)r.q[u].w, (double)xv.w, acc);
      }
    }
  }
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(MV_FULL, acc, o);
  return l2 ? (float)acc : (float)(-acc);
}

// up to 4 rows at once (n <= 4, warp-uniform): their loads are in flight together
template <int TYPE>
__device__ __forceinline__ void exact_badness4(const QueryRegs& r, const int64_t (&row)[4], int n, int dpad, bool l2,
                                               const void* payload, const float* __restrict__ sq8_t, float (&out)[4]) {
  const int lane = threadIdx.x & 31;
  double acc[4] = {0.0, 0.0, 0.0, 0.0};
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    if (4 * (lane + 32 * u) < dpad) {
      float4 xv[4];
#pragma unroll
      for (int m = 0; m < 4; ++m) {
        if (m < n) {
          if (TYPE == MV_IVF_FLAT) {
            xv[m] = __ldg(reinterpret_cast<const float4*>(reinterpret_cast<const float*>(payload) + row[m] * dpad) +
                          lane + 32 * u);
          } else {
            const uint32_t cw = __ldg(
                reinterpret_cast<const uint32_t*>(reinterpret_cast<const uint8_t*>(payload) + row[m] * dpad) + lane + 32 * u);
            xv[m].x = __fadd_rn(__fmul_rn(__ldg(sq8_t + (cw & 0xff)), r.vd[u].x), r.vm[u].x);
            xv[m].y = __fadd_rn(__fmul_rn(__ldg(sq8_t + ((cw >> 8) & 0xff)), r.vd[u].y), r.vm[u].y);
            xv[m].z = __fadd_rn(__fmul_rn(__ldg(sq8_t + ((cw >> 16) & 0xff)), r.vd[u].z), r.vm[u].z);
            xv[m].w = __fadd_rn(__fmul_rn(__ldg(sq8_t + (cw >> 24)), r.vd[u].w), r.vm[u].w);
          }
        }
      }
#pragma unroll
      for (int m = 0; m < 4; ++m) {
        if (m < n) {
          if (l2) {
            const double a = (double)r.q[u].x - xv[m].x, b = (double)r.q[u].y - xv[m].y;
            const double c = (double)r.q[u].z - xv[m].z, d = (double)r.q[u].w - xv[m].w;
            acc[m] = fma(a, a, acc[m]); acc[m] = fma(b, b, acc[m]); acc[m] = fma(c, c, acc[m]); acc[m] = fma(d, d, acc[m]);
          } else {
            acc[m] = fma((double)r.q[u].x, (double)xv[m].x, acc[m]); acc[m] = fma((double)r.q[u].y, (double)xv[m].y, acc[m]);
            acc[m] = fma((double)r.q[u].z, (double)xv[m].z, acc[m]); acc[m] = fma((double)r.q[u].w, (double)xv[m].w, acc[m]);
          }
        }
      }
    }
  }
#pragma unroll
  for (int m = 0; m < 4; ++m) {
    for (int o = 16; o > 0; o >>= 1) acc[m] += __shfl_xor_sync(MV_FULL, acc[m], o);
    out[m] = l2 ? (float)acc[m] : (float)(-acc[m]);
  }
}

// One lane re-scores one stored row (the band members of a 32-key chunk in parallel, one per
// lane); the query row (and SQ8's vmin / vdiff) sit in the warp's shared memory, read as
// broadcasts.  Same arithmetic as exact_badness.
template <int TYPE>
__device__ __forceinline__ float lane_exact_badness(int64_t row, const float* sq, const float* svm, const float* svd,
                                                    int dpad, bool l2, const void* payload,
                                                    const float* __restrict__ sq8_t) {
  double acc = 0.0;
  if (TYPE == MV_IVF_FLAT) {
    const float4* x = reinterpret_cast<const float4*>(reinterpret_cast<const float*>(payload) + row * dpad);
    for (int j4 = 0; j4 < dpad / 4; ++j4) {
      const float4 xv = __ldg(x + j4);
      const float4 qv = reinterpret_cast<const float4*>(sq)[j4];
      if (l2) {
        const double a = (double)qv.x - xv.x, b = (double)qv.y - xv.y, c = (double)qv.z - xv.z, d = (double)qv.w - xv.w;
        acc = fma(a, a, acc); acc = fma(b, b, acc); acc = fma(c, c, acc); acc = fma(d, d, acc);
      } else {
        acc = fma((double)qv.x, (double)xv.x, acc); acc = fma((double)qv.y, (double)xv.y, acc);
        acc = fma((double)qv.z, (double)xv.z, acc); acc = fma((double)qv.w, (double)xv.w, acc);
      }
    }
  } else {
    const uint32_t* x = reinterpret_cast<const uint32_t*>(reinterpret_cast<const uint8_t*>(payload) + row * dpad);
    for (int j4 = 0; j4 < dpad / 4; ++j4) {
      const uint32_t cw = __ldg(x + j4);
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int j = 4 * j4 + u;
        const float xv = __fadd_rn(__fmul_rn(sq8_t[(cw >> (8 * u)) & 0xff], svd[j]), svm[j]);
        if (l2) {
          const double a = (double)sq[j] - xv;
          acc = fma(a, a, acc);
        } else {
          acc = fma((double)sq[j], (double)xv, acc);
        }
      }
    }
  }
  return l2 ? (float)acc : (float)(-acc);
}

// k <= 32 R: one warp per query, two passes over the query's candidates (its pairs' regions,
// walked in 32-key chunks through a flattened index over groups of 32 pairs located by a shuffle
// binary search).  Pass 1 keeps every lane's R smallest keys; the k-th smallest of those 32R keys
// bounds the answer (k distinct keys are at or below it).  Pass 2 streams the keys at or below the
// bound through a 32-entry staging buffer into a sorted register list (sort-32 + bitonic merge).
//
// RT >= 0 (MV_IVF_FLAT / MV_IVF_SQ8): the filter mode's fused refine.  The keys are
// approximate (|b~ - b| <= E_q) unless rf.rgate says the search is exact; pass 1's bound t~ is then
// >= the k-th approximate key, every member of the exact top-k has b~ <= t~ + 2 E_q, and pass 2
// re-scores exactly (exact_badness) only those band keys before staging them -- the sorted list
// keeps the k smallest exact keys.  One kernel instead of a separate k-th select, re-scoring pass
// and final select.
struct RefineArgs {
  const float* qerr;
  const float* qpad;
  int dpad;
  const void* payload;
  const uint32_t* row_of_rank;
  const float *vmin, *vdiff, *sq8_t;
  const int* rgate;  // nullable: filter mode always; else only when *rgate != 0
};

template <int R>
__global__ void __launch_bounds__(256) k_final_warp(const int64_t* __restrict__ poff, const int32_t* __restrict__ pcnt,
                                                    const uint64_t* __restrict__ part, int64_t nq, int npb, int k,
                                                    int metric, const int64_t* __restrict__ sorted_ids, float* out_d,
                                                    int64_t* out_i, const int32_t* __restrict__ nuse,
                                                    uint64_t* tau_out, const int* __restrict__ gate) {
  __shared__ uint64_t stage_all[8][64];
  const int lane = threadIdx.x & 31;
  const int64_t q = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (q >= nq || (gate && *gate == 0)) return;
  uint64_t* stage = stage_all[threadIdx.x >> 5];
  const int stride = npb;
  if (nuse) npb = nuse[q];
  // visit every candidate key of the query, 32 at a time: f(key) with key = PAD past the end
  auto for_each_chunk = [&](auto&& f) {
    for (int g = 0; g < npb; g += 32) {
      const int j = g + lane;
      const int cnt = j < npb ? pcnt[q * stride + j] : 0;
      const int64_t off = j < npb ? poff[q * stride + j] : 0;
      int incl = cnt;
      for (int o = 1; o < 32; o <<= 1) {
        const int v = __shfl_up_sync(MV_FULL, incl, o);
        if (lane >= o) incl += v;
      }
      const int excl = incl - cnt;
      const int T = __shfl_sync(MV_FULL, incl, 31);
      // kUnroll chunks' loads in flight per lane (one dependent global load per chunk was the
      // warp's latency chain: configs[2]'s ~1500 keys per query = ~47 round trips per pass)
      for (int e00 = 0; e00 < T; e00 += 32 * kUnroll) {
        uint64_t kk[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
          const int e = e00 + 32 * u + lane;
          int lo = 0;  // pair holding element e: the largest s with excl[s] <= e
#pragma unroll
          for (int step = 16; step > 0; step >>= 1) {
            const int ex = __shfl_sync(MV_FULL, excl, (lo + step) & 31);
            if (lo + step < 32 && ex <= e) lo += step;
          }
          const int64_t o = __shfl_sync(MV_FULL, off, lo);
          const int ex = __shfl_sync(MV_FULL, excl, lo);
          kk[u] = e < T ? part[o + (e - ex)] : MV_KEY_PAD;
        }
#pragma unroll
        for (int u = 0; u < kUnroll; ++u)
          if (e00 + 32 * u < T) f(kk[u]);  // warp-uniform
      }
    }
  };
  // pass 1: each lane's R smallest keys
  uint64_t t[R];
#pragma unroll
  for (int r = 0; r < R; ++r) t[r] = MV_KEY_PAD;
  for_each_chunk([&](uint64_t key) {
    if (key < t[R - 1]) {
      t[R - 1] = key;
#pragma unroll
      for (int r = R - 1; r > 0; --r)
        if (t[r] < t[r - 1]) {
          const uint64_t x = t[r];
          t[r] = t[r - 1];
          t[r - 1] = x;
        }
    }
  });
  warp_bitonic_sort<R>(t);
  uint64_t bsel = t[0];
#pragma unroll
  for (int r = 1; r < R; ++r)
    if (r == ((k - 1) >> 5)) bsel = t[r];
  const uint64_t bound = shfl64(bsel, (k - 1) & 31);  // PAD when fewer than k candidates
  // pass 2: keys <= bound -> staging -> sorted list (best[r] holds element r*32 + lane)
  uint64_t best[R];
#pragma unroll
  for (int r = 0; r < R; ++r) best[r] = MV_KEY_PAD;
  int ns = 0;
  auto flush32 = [&]() {
    uint64_t c[R];
    uint64_t c1[1] = {lane < ns ? stage[lane] : MV_KEY_PAD};
    warp_bitonic_sort<1>(c1);
    c[0] = c1[0];
#pragma unroll
    for (int r = 1; r < R; ++r) c[r] = MV_KEY_PAD;
    warp_merge_smallest<R>(best, c);
    const int rest = ns > 32 ? ns - 32 : 0;
    const uint64_t mv = lane < rest ? stage[32 + lane] : 0;
    __syncwarp();
    if (lane < rest) stage[lane] = mv;
    __syncwarp();
    ns = rest;
  };
  for_each_chunk([&](uint64_t key) {
    const bool ps = key != MV_KEY_PAD && key <= bound;
    const uint32_t m = __ballot_sync(MV_FULL, ps);
    if (ps) stage[ns + __popc(m & ((1u << lane) - 1))] = key;
    ns += __popc(m);
    __syncwarp();
    if (ns >= 32) flush32();
  });
  if (ns > 0) flush32();
  auto kth_of = [&]() {
    uint64_t v = best[0];
#pragma unroll
    for (int r = 1; r < R; ++r)
      if (r == ((k - 1) >> 5)) v = best[r];
    return shfl64(v, (k - 1) & 31);
  };
  if (tau_out) {  // seeding: the k-th best key of the first nuse[q] pairs bounds the query's top-k
    const uint64_t kth = kth_of();
    if (lane == 0 && kth != MV_KEY_PAD) tau_out[q] = kth;
    return;
  }
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const int i = r * 32 + lane;
    if (i < k) {
      const uint64_t key = best[r];
      float dv;
      int64_t iv;
      if (key != MV_KEY_PAD) {
        dv = key_dist((uint32_t)(key >> 32), metric);
        iv = rank_to_id(sorted_ids, key);
      } else {
        dv = metric == MV_L2 ? __int_as_float(0x7f800000) : __int_as_float(0xff800000);
        iv = -1;
      }
      out_d[q * k + i] = dv;
      out_i[q * k + i] = iv;
    }
  }
}

// k <= 256, filter mode, second kernel (the first is k_final_warp in tau mode: t~ = the exact
// k-th smallest approximate key): one pass over the query's keys; the band b~ <= t~ + 2 E_q is
// re-scored exactly (exact_badness4: four rows in flight), staged and merged into a sorted list
// of the k smallest exact keys, which is the answer.  Kept apart from the select
// so that each kernel has its own register budget (the selects run at full occupancy).
template <int R, int TYPE>
__global__ void __launch_bounds__(256) k_refine_band(const int64_t* __restrict__ poff, const int32_t* __restrict__ pcnt,
                                                     const uint64_t* __restrict__ part, int64_t nq, int npb, int k,
                                                     int metric, const int64_t* __restrict__ sorted_ids, float* out_d,
                                                     int64_t* out_i, const uint64_t* __restrict__ tau2,
                                                     const RefineArgs rf) {
  __shared__ uint64_t stage_all[8][64];
  // shared: SQ8's decode table (256), then per warp q (+ SQ8: vmin, vdiff), dpad floats each
  extern __shared__ __align__(16) float qsm[];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int64_t q = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int dpad = rf.dpad;
  float* stab = qsm;
  if (TYPE == MV_IVF_SQ8) {
    for (int i = threadIdx.x; i < 256; i += blockDim.x) stab[i] = rf.sq8_t[i];
    __syncthreads();
  }
  if (q >= nq || (rf.rgate && *rf.rgate == 0)) return;
  uint64_t* stage = stage_all[wib];
  float* sq = qsm + (TYPE == MV_IVF_SQ8 ? 256 + wib * 3 * dpad : wib * dpad);
  float* svm = sq + dpad;
  float* svd = svm + dpad;
  for (int j = lane; j < dpad; j += 32) {
    sq[j] = rf.qpad[q * dpad + j];
    if (TYPE == MV_IVF_SQ8) {
      svm[j] = rf.vmin[j];
      svd[j] = rf.vdiff[j];
    }
  }
  __syncwarp();
  const uint64_t kth = tau2[q];
  const float band =
      kth == MV_KEY_PAD ? __int_as_float(0x7f800000) : __fadd_ru(key2f((uint32_t)(kth >> 32)), 2.0f * rf.qerr[q]);
  uint64_t best[R];
#pragma unroll
  for (int r = 0; r < R; ++r) best[r] = MV_KEY_PAD;
  int ns = 0;
  // a flush re-scores the (up to) 32 staged band keys, one per lane -- every lane busy -- before the
  // sort + merge (re-scoring in the chunk loop would run a whole warp for one or two band keys)
  auto flush32 = [&]() {
    uint64_t c[R];
    uint64_t c1[1] = {MV_KEY_PAD};
    if (lane < ns) {
      const uint64_t key = stage[lane];
      const int64_t row = (int64_t)__ldg(rf.row_of_rank + (uint32_t)key);
      const float b = lane_exact_badness<TYPE>(row, sq, svm, svd, dpad, metric == MV_L2, rf.payload, stab);
      c1[0] = ((uint64_t)f2key(b) << 32) | (uint32_t)key;
    }
    warp_bitonic_sort<1>(c1);
    c[0] = c1[0];
#pragma unroll
    for (int r = 1; r < R; ++r) c[r] = MV_KEY_PAD;
    warp_merge_smallest<R>(best, c);
    const int rest = ns > 32 ? ns - 32 : 0;
    const uint64_t mv = lane < rest ? stage[32 + lane] : 0;
    __syncwarp();
    if (lane < rest) stage[lane] = mv;
    __syncwarp();
    ns = rest;
  };
  for (int g = 0; g < npb; g += 32) {
    const int j = g + lane;
    const int cnt = j < npb ? pcnt[q * npb + j] : 0;
    const int64_t off = j < npb ? poff[q * npb + j] : 0;
    int incl = cnt;
    for (int o = 1; o < 32; o <<= 1) {
      const int v = __shfl_up_sync(MV_FULL, incl, o);
      if (lane >= o) incl += v;
    }
    const int excl = incl - cnt;
    const int T = __shfl_sync(MV_FULL, incl, 31);
    for (int e00 = 0; e00 < T; e00 += 32 * kUnroll) {
      uint64_t kk[kUnroll];
#pragma unroll
      for (int u = 0; u < kUnroll; ++u) {  // kUnroll chunks' loads in flight (as k_final_warp)
        const int e = e00 + 32 * u + lane;
        int lo = 0;
#pragma unroll
        for (int step = 16; step > 0; step >>= 1) {
          const int ex = __shfl_sync(MV_FULL, excl, (lo + step) & 31);
          if (lo + step < 32 && ex <= e) lo += step;
        }
        const int64_t addr = __shfl_sync(MV_FULL, off, lo) + (e - __shfl_sync(MV_FULL, excl, lo));
        kk[u] = e < T ? part[addr] : MV_KEY_PAD;
      }
#pragma unroll
      for (int u = 0; u < kUnroll; ++u) {
        if (e00 + 32 * u >= T) break;  // warp-uniform
        const uint64_t key = kk[u];
        const bool ps = key != MV_KEY_PAD && key2f((uint32_t)(key >> 32)) <= band;
        const uint32_t m = __ballot_sync(MV_FULL, ps);
        if (ps) stage[ns + __popc(m & ((1u << lane) - 1))] = key;  // re-scored at the flush
        ns += __popc(m);
        __syncwarp();
        if (ns >= 32) flush32();
      }
    }
  }
  if (ns > 0) flush32();
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const int i = r * 32 + lane;
    if (i < k) {
      const uint64_t key = best[r];
      float dv;
      int64_t iv;
      if (key != MV_KEY_PAD) {
        dv = key_dist((uint32_t)(key >> 32), metric);
        iv = rank_to_id(sorted_ids, key);
      } else {
        dv = metric == MV_L2 ? __int_as_float(0x7f800000) : __int_as_float(0xff800000);
        iv = -1;
      }
      out_d[q * k + i] = dv;
      out_i[q * k + i] = iv;
    }
  }
}

// k <= 256: the warp kernel with a 32R-entry register list (R = 1, 2, 4, 8)
static bool launch_warp_select(const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq, int npb,
                               int k, int metric, const int64_t* sorted_ids, float* out_d, int64_t* out_i,
                               const int32_t* nuse, uint64_t* tau, const int* gate, cudaStream_t st) {
  const unsigned grid = (unsigned)((nq * 32 + 255) / 256);
  if (k <= 32)
    k_final_warp<1><<<grid, 256, 0, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d, out_i, nuse, tau,
                                         gate);
  else if (k <= 64)
    k_final_warp<2><<<grid, 256, 0, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d, out_i, nuse, tau,
                                         gate);
  else if (k <= 128)
    k_final_warp<4><<<grid, 256, 0, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d, out_i, nuse, tau,
                                         gate);
  else if (k <= 256)
    k_final_warp<8><<<grid, 256, 0, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d, out_i, nuse, tau,
                                         gate);
  else
    return false;
  return true;
}

// k <= 256 with the filter mode's refine: k_final_warp in tau mode (t~ = the k-th approximate key)
// then k_refine_band; an exact search (rgate set and *rgate == 0) takes the plain final select
__global__ void k_not(const int* __restrict__ g, int* __restrict__ out) { *out = g ? (*g == 0) : 0; }

cudaError_t launch_final_refine(int type, const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq,
                                int npb, int k, int metric, const int64_t* sorted_ids, float* out_d, int64_t* out_i,
                                const float* qerr, const float* qpad, int dpad, const void* payload,
                                const uint32_t* row_of_rank, const float* vmin, const float* vdiff, const float* sq8_t,
                                const int* rgate, uint64_t* tau2, int* notgate, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  if (k > 256 || dpad > 512 || dpad % 4) return cudaErrorInvalidValue;
  const RefineArgs rf{qerr, qpad, dpad, payload, row_of_rank, vmin, vdiff, sq8_t, rgate};
  const unsigned grid = (unsigned)((nq * 32 + 255) / 256);
  cudaError_t e;
  // shared: (SQ8: the 256-entry decode table +) per warp q (, vmin, vdiff)
  const size_t qsm = ((type == MV_IVF_SQ8 ? 256 : 0) + (size_t)8 * (type == MV_IVF_SQ8 ? 3 : 1) * dpad) * sizeof(float);
  if (rgate) {  // exact searches: the plain select, gated by !*rgate
    k_not<<<1, 1, 0, st>>>(rgate, notgate);
    if (!launch_warp_select(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d, out_i, nullptr, nullptr, notgate,
                            st))
      return cudaErrorInvalidValue;
  }
  if ((e = cudaMemsetAsync(tau2, 0xff, sizeof(uint64_t) * nq, st)) != cudaSuccess) return e;
  launch_warp_select(poff, pcnt, part, nq, npb, k, MV_L2, nullptr, nullptr, nullptr, nullptr, tau2, rgate, st);
#define MV_REFINE_LAUNCH(R)                                                                                           \
  if (type == MV_IVF_FLAT) {                                                                                          \
    k_refine_band<R, MV_IVF_FLAT><<<grid, 256, qsm, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d,    \
                                                          out_i, tau2, rf);                                           \
  } else {                                                                                                            \
    if ((e = cudaFuncSetAttribute(k_refine_band<R, MV_IVF_SQ8>, cudaFuncAttributeMaxDynamicSharedMemorySize,         \
                                  (int)qsm)) != cudaSuccess)                                                          \
      return e;                                                                                                       \
    k_refine_band<R, MV_IVF_SQ8><<<grid, 256, qsm, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d,     \
                                                         out_i, tau2, rf);                                            \
  }
  if (k <= 32) { MV_REFINE_LAUNCH(1) }
  else if (k <= 64) { MV_REFINE_LAUNCH(2) }
  else if (k <= 128) { MV_REFINE_LAUNCH(4) }
  else { MV_REFINE_LAUNCH(8) }
#undef MV_REFINE_LAUNCH
  return cudaGetLastError();
}

cudaError_t launch_final_select(const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq, int npb,
                                int k, int metric, const int64_t* sorted_ids, float* out_d, int64_t* out_i,
                                int64_t tmax, uint8_t* over, BigSel bsel, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  if (launch_warp_select(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d, out_i, nullptr, nullptr, nullptr,
                         st))
    return cudaGetLastError();
  return launch_big_select(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d, out_i, nullptr, nullptr, tmax,
                           over, nullptr, bsel, st);
}

cudaError_t launch_tau_select(const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq, int npb,
                              const int32_t* nuse, int k, uint64_t* tau, int64_t tmax, uint8_t* over,
                              const int* gate, BigSel bsel, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  if (launch_warp_select(poff, pcnt, part, nq, npb, k, MV_L2, nullptr, nullptr, nullptr, nuse, tau, gate, st))
    return cudaGetLastError();
  return launch_big_select(poff, pcnt, part, nq, npb, k, MV_L2, nullptr, nullptr, nullptr, nuse, tau, tmax, over, gate,
                           bsel, st);
}

// ------------------------------------------------------------------------------------------
// Exact re-scoring for the tensor-core scan's filter mode (DESIGN.md §5 "Filter mode").  The
// scan's keys carry the fp32 tensor-core badness b~ with |b~ - b| <= E_q (qerr[q], a rigorous
// bound), b the oracle's badness: FLAT when the stored vectors or the queries are not
// tf32-exact, SQ8 always.  With t~ = the k-th smallest b~ of the query (tau2[q]), every member of
// the exact top-k has b~ <= t~ + 2 E_q (k candidates have b <= t~ + E_q), and every candidate
// above that bound has b > t~ + E_q.  So the kernel recomputes b exactly for the candidates at or
// below the bound -- fp64 from the fp32 query and the stored row (FLAT: the fp32 vector; SQ8: the
// codes decoded in fp32 in the oracle's order, vmin + ((c + 0.5) / 255) vdiff), the definition of
// PAPER.md:290-294 (§2.1) -- rewrites their keys (exact fp32 distance key << 32 | id rank), and
// turns every other key into padding.  The final select then returns the exact top-k.  One warp
// per query; the query row lives in registers (dpad <= 512: <= 4 float4 per lane), each
// re-scored row is read as coalesced float4s (FLAT) or 4-code words (SQ8).
// ------------------------------------------------------------------------------------------
template <int TYPE>
__global__ void __launch_bounds__(256) k_rekey(const int64_t* __restrict__ poff, const int32_t* __restrict__ pcnt,
                                               uint64_t* __restrict__ part, int64_t nq, int npb,
                                               const uint64_t* __restrict__ tau2, const float* __restrict__ qerr,
                                               int metric, const float* __restrict__ qpad, int dpad,
                                               const void* __restrict__ payload,
                                               const uint32_t* __restrict__ row_of_rank,
                                               const float* __restrict__ vmin, const float* __restrict__ vdiff,
                                               const float* __restrict__ sq8_t, const int* __restrict__ gate) {
  const int lane = threadIdx.x & 31;
  const int64_t q = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (q >= nq || (gate && *gate == 0)) return;
  const uint64_t t = tau2[q];
  // bound in badness units, rounded up; fewer than k candidates (t = PAD): every candidate
  const float bound =
      t == MV_KEY_PAD ? __int_as_float(0x7f800000) : __fadd_ru(key2f((uint32_t)(t >> 32)), 2.0f * qerr[q]);
  QueryRegs qr;
  load_query_regs<TYPE>(qr, qpad + q * dpad, dpad, vmin, vdiff);
  const bool l2 = metric == MV_L2;
  for (int g = 0; g < npb; g += 32) {
    const int j = g + lane;
    const int cnt = j < npb ? pcnt[q * npb + j] : 0;
    const int64_t off = j < npb ? poff[q * npb + j] : 0;
    int incl = cnt;
    for (int o = 1; o < 32; o <<= 1) {
      const int v = __shfl_up_sync(MV_FULL, incl, o);
      if (lane >= o) incl += v;
    }
    const int excl = incl - cnt;
    const int T = __shfl_sync(MV_FULL, incl, 31);
    for (int e0 = 0; e0 < T; e0 += 32) {
      const int e = e0 + lane;
      int lo = 0;
#pragma unroll
      for (int step = 16; step > 0; step >>= 1) {
        const int ex = __shfl_sync(MV_FULL, excl, (lo + step) & 31);
        if (lo + step < 32 && ex <= e) lo += step;
      }
      const int64_t addr = __shfl_sync(MV_FULL, off, lo) + (e - __shfl_sync(MV_FULL, excl, lo));
      const uint64_t key = e < T ? part[addr] : MV_KEY_PAD;
      const bool band = key != MV_KEY_PAD && key2f((uint32_t)(key >> 32)) <= bound;
      uint64_t nk = key;
      uint32_t m = __ballot_sync(MV_FULL, band);
      while (m) {
        const int src = __ffs(m) - 1;
        m &= m - 1;
        const uint32_t rk = __shfl_sync(MV_FULL, (uint32_t)key, src);
        const float b = exact_badness<TYPE>(qr, (int64_t)__ldg(row_of_rank + rk), dpad, l2, payload, sq8_t);
        if (lane == src) nk = ((uint64_t)f2key(b) << 32) | rk;
      }
      // only the band is rewritten: its k smallest exact keys (<= t~ + E) are below every key left
      // approximate (> t~ + 2 E), so the final select returns the exact top-k
      if (band) part[addr] = nk;
    }
  }
}

cudaError_t launch_rekey(int type, const int64_t* poff, const int32_t* pcnt, uint64_t* part, int64_t nq, int npb,
                         const uint64_t* tau2, const float* qerr, int metric, const float* qpad, int dpad,
                         const void* payload, const uint32_t* row_of_rank, const float* vmin, const float* vdiff,
                         const float* sq8_t, const int* gate, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  if (dpad > 512 || dpad % 4) return cudaErrorInvalidValue;
  const unsigned grid = (unsigned)((nq * 32 + 255) / 256);
  if (type == MV_IVF_FLAT)
    k_rekey<MV_IVF_FLAT><<<grid, 256, 0, st>>>(poff, pcnt, part, nq, npb, tau2, qerr, metric, qpad, dpad, payload,
                                               row_of_rank, vmin, vdiff, sq8_t, gate);
  else
    k_rekey<MV_IVF_SQ8><<<grid, 256, 0, st>>>(poff, pcnt, part, nq, npb, tau2, qerr, metric, qpad, dpad, payload,
                                              row_of_rank, vmin, vdiff, sq8_t, gate);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------
// merge of two best-first lists per query (stable: A before B on equal (distance, id))
// ------------------------------------------------------------------------------------------
struct MKey {
  uint32_t dk;
  int64_t id;
};
__device__ __forceinline__ MKey mkey(const float* d, const int64_t* i, int x, int metric) {
  const int64_t id = i[x];
  if (id == -1) return {0xffffffffu, (int64_t)0x7fffffffffffffffll};
  return {dist_key(d[x], metric), id};
}
__device__ __forceinline__ bool mle(const MKey& a, const MKey& b) {  // a <= b
  return a.dk < b.dk || (a.dk == b.dk && a.id <= b.id);
}

__global__ void k_merge2(int metric, const float* __restrict__ ad, const int64_t* __restrict__ ai,
                         const float* __restrict__ bd, const int64_t* __restrict__ bi, int64_t nq, int k,
                         float* od, int64_t* oi) {
  const int64_t total = nq * k;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t q = t / k;
    const int i = (int)(t - q * k);
    const float* A = ad + q * k; const int64_t* AI = ai + q * k;
    const float* B = bd + q * k; const int64_t* BI = bi + q * k;
    int lo = max(0, i - k), hi = min(i, k);
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if (mle(mkey(A, AI, mid, metric), mkey(B, BI, i - mid - 1, metric))) lo = mid + 1; else hi = mid;
    }
    const int a = lo, b = i - a;
    const bool takeA = a < k && (b >= k || mle(mkey(A, AI, a, metric), mkey(B, BI, b, metric)));
    od[t] = takeA ? A[a] : B[b];
    oi[t] = takeA ? AI[a] : BI[b];
  }
}

cudaError_t launch_merge2(int metric, const float* ad, const int64_t* ai, const float* bd, const int64_t* bi,
                          int64_t nq, int k, float* od, int64_t* oi, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  const int grid = (int)min64(kNumSMs * 8, (nq * k + 255) / 256);
  k_merge2<<<grid, 256, 0, st>>>(metric, ad, ai, bd, bi, nq, k, od, oi);
  return cudaGetLastError();
}

__global__ void k_fill_pad(int64_t n, int metric, float* d, int64_t* i) {
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
    d[t] = metric == MV_L2 ? __int_as_float(0x7f800000) : __int_as_float(0xff800000);
    i[t] = -1;
  }
}

cudaError_t launch_fill_pad(int64_t n, int metric, float* d, int64_t* i, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  const int grid = (int)min64(kNumSMs * 8, (n + 255) / 256);
  k_fill_pad<<<grid, 256, 0, st>>>(n, metric, d, i);
  return cudaGetLastError();
}

}  // namespace mv
