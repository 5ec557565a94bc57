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
                                                      uint64_t* tau_out) {
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
      iv = sorted_ids[(uint32_t)(key & 0xffffffffu)];
    } else {
      dv = metric == MV_L2 ? __int_as_float(0x7f800000) : __int_as_float(0xff800000);
      iv = -1;
    }
    out_d[q * k + i] = dv;
    out_i[q * k + i] = iv;
  }
}

// k <= 32: one warp per query.  The pairs' regions are walked in 32-key chunks (a flattened index
// over groups of 32 pairs, located by a shuffle binary search); a chunk is skipped unless some key
// beats the running k-th best, else it is bitonic-sorted and merged into the sorted register list.
__global__ void __launch_bounds__(256) k_final_small(const int64_t* __restrict__ poff, const int32_t* __restrict__ pcnt,
                                                     const uint64_t* __restrict__ part, int64_t nq, int npb, int k,
                                                     int metric, const int64_t* __restrict__ sorted_ids, float* out_d,
                                                     int64_t* out_i, const int32_t* __restrict__ nuse,
                                                     uint64_t* tau_out) {
  const int lane = threadIdx.x & 31;
  const int64_t q = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (q >= nq) return;
  const int stride = npb;
  if (nuse) npb = nuse[q];
  uint64_t best[1] = {MV_KEY_PAD};  // ascending: lane i holds the i-th best so far
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
    for (int e0 = 0; e0 < T; e0 += 32) {
      const int e = e0 + lane;
      // pair holding element e: the largest s with excl[s] <= e
      int lo = 0;
#pragma unroll
      for (int step = 16; step > 0; step >>= 1) {
        const int ex = __shfl_sync(MV_FULL, excl, lo + step);
        if (lo + step < 32 && ex <= e) lo += step;
      }
      const int64_t o = __shfl_sync(MV_FULL, off, lo);
      const int ex = __shfl_sync(MV_FULL, excl, lo);
      uint64_t v[1] = {e < T ? part[o + (e - ex)] : MV_KEY_PAD};
      const uint64_t kth = shfl64(best[0], k - 1);
      if (!(v[0] < kth)) v[0] = MV_KEY_PAD;
      if (__any_sync(MV_FULL, v[0] != MV_KEY_PAD)) {
        warp_bitonic_sort<1>(v);
        warp_merge_smallest<1>(best, v);
      }
    }
  }
  if (tau_out) {  // seeding: the k-th best key of the first nuse[q] pairs bounds the query's top-k
    const uint64_t kth = shfl64(best[0], k - 1);
    if (lane == 0 && kth != MV_KEY_PAD) tau_out[q] = kth;
    return;
  }
  if (lane < k) {
    const uint64_t key = best[0];
    float dv;
    int64_t iv;
    if (key != MV_KEY_PAD) {
      dv = key_dist((uint32_t)(key >> 32), metric);
      iv = sorted_ids[(uint32_t)(key & 0xffffffffu)];
    } else {
      dv = metric == MV_L2 ? __int_as_float(0x7f800000) : __int_as_float(0xff800000);
      iv = -1;
    }
    out_d[q * k + lane] = dv;
    out_i[q * k + lane] = iv;
  }
}

cudaError_t launch_final_select(const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq, int npb,
                                int k, int metric, const int64_t* sorted_ids, float* out_d, int64_t* out_i,
                                cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  if (k <= 32) {
    k_final_small<<<(unsigned)((nq * 32 + 255) / 256), 256, 0, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids,
                                                                     out_d, out_i, nullptr, nullptr);
    return cudaGetLastError();
  }
  const int selcap = max(4096, next_pow2(k));
  size_t smem = (size_t)(selcap + kBoundCap) * 8 + (size_t)(npb + 1) * 4 + 256 * 4 + 8 * 4 + 64;
  cudaError_t e = cudaFuncSetAttribute(k_final_select, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k_final_select<<<(unsigned)nq, 256, smem, st>>>(poff, pcnt, part, nq, npb, k, metric, sorted_ids, out_d, out_i,
                                                  selcap, nullptr, nullptr);
  return cudaGetLastError();
}

cudaError_t launch_tau_select(const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq, int npb,
                              const int32_t* nuse, int k, uint64_t* tau, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  if (k <= 32) {
    k_final_small<<<(unsigned)((nq * 32 + 255) / 256), 256, 0, st>>>(poff, pcnt, part, nq, npb, k, MV_L2, nullptr,
                                                                     nullptr, nullptr, nuse, tau);
    return cudaGetLastError();
  }
  const int selcap = max(4096, next_pow2(k));
  size_t smem = (size_t)(selcap + kBoundCap) * 8 + (size_t)(npb + 1) * 4 + 256 * 4 + 8 * 4 + 64;
  cudaError_t e = cudaFuncSetAttribute(k_final_select, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k_final_select<<<(unsigned)nq, 256, smem, st>>>(poff, pcnt, part, nq, npb, k, MV_L2, nullptr, nullptr, nullptr,
                                                  selcap, nuse, tau);
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
