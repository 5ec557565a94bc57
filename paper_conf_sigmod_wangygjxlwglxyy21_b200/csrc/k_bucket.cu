// k_bucket.cu -- §8 row a4: invert the (query, probed list) pairs into per-list query buckets
// and work items.  The grouping is the B200 form of the paper's cache-aware idea: "reuse the
// accessed data vectors as much as possible for multiple queries" (§3.2.1),
// because in step 2 "different queries do not necessarily access the same buckets"
// (§3.4).  A counting sort by list id: histogram, exclusive scan, scatter.
// Also the per-pair candidate-region offsets for the scan's partial top-k output.
#include "mv_internal.cuh"

namespace mv {

// Single-CTA exclusive scan (n up to a few million): out[0..n], out[n] = total.
template <typename T>
__global__ void __launch_bounds__(1024) k_scan_single(const T* __restrict__ in, int64_t n, T* __restrict__ out) {
  __shared__ T part[1024];
  const int tid = threadIdx.x;
  const int64_t per = (n + 1023) / 1024;
  const int64_t s = tid * per, e = min64(n, s + per);
  T acc = 0;
  for (int64_t i = s; i < e; ++i) acc += in[i];
  part[tid] = acc;
  __syncthreads();
  for (int off = 1; off < 1024; off <<= 1) {  // Hillis-Steele inclusive scan of 1024 partials
    T v = tid >= off ? part[tid - off] : (T)0;
    __syncthreads();
    part[tid] += v;
    __syncthreads();
  }
  T run = tid ? part[tid - 1] : (T)0;
  for (int64_t i = s; i < e; ++i) {
    out[i] = run;
    run += in[i];
  }
  if (tid == 1023) out[n] = part[1023];
}

cudaError_t launch_scan_i32(const int32_t* in, int n, int32_t* out, cudaStream_t st) {
  k_scan_single<int32_t><<<1, 1024, 0, st>>>(in, n, out);
  return cudaGetLastError();
}
cudaError_t launch_scan_i64(const int64_t* in, int64_t n, int64_t* out, cudaStream_t st) {
  k_scan_single<int64_t><<<1, 1024, 0, st>>>(in, n, out);
  return cudaGetLastError();
}

// Virtual list of pair p = q*npb + r: its list l, or l + nlist for the pairs of the second phase
// when the seeding phase is on (ra != nullptr): phase A = the ra[q] nearest lists of query q,
// scanned first so that their k-th best bounds tau_q before the other lists are scanned.
__device__ __forceinline__ int vlist_of(const int32_t* probes, int64_t p, int npb, int nlist, const int32_t* ra) {
  const int l = probes[p];
  return (ra && (int)(p % npb) >= ra[p / npb]) ? l + nlist : l;
}

__global__ void k_count_pairs(const int32_t* __restrict__ probes, int64_t npairs, int npb, int nlist,
                              const int32_t* __restrict__ ra, int32_t* counts) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < npairs; p += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(counts + vlist_of(probes, p, npb, nlist, ra), 1);
}

__global__ void k_bucket_fill(const int32_t* __restrict__ probes, int64_t npairs, int npb, int nlist,
                              const int32_t* __restrict__ ra, const int32_t* __restrict__ boff, int32_t* bfill,
                              int32_t* bq) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < npairs; p += (int64_t)gridDim.x * blockDim.x) {
    const int l = vlist_of(probes, p, npb, nlist, ra);
    const int pos = boff[l] + atomicAdd(bfill + l, 1);
    bq[pos] = (int32_t)p;
  }
}

// one warp per query: ra[q] = the fewest nearest lists holding >= need candidates (at most npb)
__global__ void k_seed_ranks(const int32_t* __restrict__ probes, int64_t nq, int npb,
                             const int64_t* __restrict__ list_off, int64_t need, int32_t* ra) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t q = warp; q < nq; q += nwarps) {
    int64_t run = 0;
    int r = npb;
    for (int j0 = 0; j0 < npb; j0 += 32) {
      const int j = j0 + lane;
      int64_t c = 0;
      if (j < npb) {
        const int l = probes[q * npb + j];
        c = list_off[l + 1] - list_off[l];
      }
      int64_t incl = c;
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t v = __shfl_up_sync(MV_FULL, incl, o);
        if (lane >= o) incl += v;
      }
      const uint32_t hit = __ballot_sync(MV_FULL, j < npb && run + incl >= need);
      if (hit) {
        r = j0 + __ffs(hit);  // ranks 0 .. first hit
        break;
      }
      run += __shfl_sync(MV_FULL, incl, 31);
    }
    if (lane == 0) ra[q] = r;
  }
}

// qcfg = {query chunk, query planes}: the split (two-plane) shape when *qlo_any, else the exact one
__global__ void k_scan_cfg(const int* qlo_any, int qc_exact, int p_exact, int qc_split, int p_split, int32_t* qcfg) {
  const bool sp = qlo_any != nullptr && *qlo_any != 0;
  qcfg[0] = sp ? qc_split : qc_exact;
  qcfg[1] = sp ? p_split : p_exact;
}

cudaError_t launch_scan_cfg(const int* qlo_any, int qc_exact, int p_exact, int qc_split, int p_split, int32_t* qcfg,
                            cudaStream_t st) {
  k_scan_cfg<<<1, 1, 0, st>>>(qlo_any, qc_exact, p_exact, qc_split, p_split, qcfg);
  return cudaGetLastError();
}

cudaError_t launch_seed_ranks(const int32_t* probes, int64_t nq, int npb, const int64_t* list_off, int64_t need,
                              int32_t* ra, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  const int grid = (int)min64(kNumSMs * 8, (nq * 32 + 255) / 256);
  k_seed_ranks<<<grid, 256, 0, st>>>(probes, nq, npb, list_off, need, ra);
  return cudaGetLastError();
}

__global__ void k_work_count(const int32_t* __restrict__ lcount, int nlist, const int32_t* __restrict__ qcfg,
                             int32_t* wcount) {
  const int l = blockIdx.x * blockDim.x + threadIdx.x;
  const int qchunk = qcfg[0];
  if (l < nlist) wcount[l] = (lcount[l] + qchunk - 1) / qchunk;
}

__global__ void k_work_fill(const int32_t* __restrict__ wcount, const int32_t* __restrict__ woff,
                            const int32_t* __restrict__ boff, int nlist, const int32_t* __restrict__ qcfg,
                            int2* witems) {
  const int l = blockIdx.x * blockDim.x + threadIdx.x;
  const int qchunk = qcfg[0];
  if (l >= nlist) return;
  const int n = wcount[l], o = woff[l], b = boff[l];
  for (int c = 0; c < n; ++c) witems[o + c] = make_int2(l, b + c * qchunk);
}

// Longest-first order for the persistent scan's static round-robin: a single-CTA counting sort of
// the work items by descending cost key = 64 * tiles + queries (tiles = ceil(|list| / 128)); with
// the seeding split, every phase-A item (virtual list < nlist) precedes every phase-B item.
__global__ void __launch_bounds__(1024) k_sort_work(const int2* __restrict__ in, const int32_t* __restrict__ nwork_p,
                                                    const int32_t* __restrict__ boff, const int64_t* __restrict__ list_off,
                                                    int nlist, const int32_t* __restrict__ qcfg,
                                                    int2* __restrict__ out) {
  constexpr int NB = 8192, HB = 4096;
  const int qchunk = qcfg[0];
  __shared__ int hist[NB];
  __shared__ int part[1024];
  const int nwork = *nwork_p, tid = threadIdx.x;
  for (int i = tid; i < NB; i += 1024) hist[i] = 0;
  __syncthreads();
  auto key = [&](int w) {
    const int2 it = in[w];
    const int l = it.x >= nlist ? it.x - nlist : it.x;
    const int nq = min(qchunk, boff[it.x + 1] - it.y);
    const int64_t len = list_off[l + 1] - list_off[l];
    const int tiles = (int)min64((len + 127) / 128, 63);
    return (it.x >= nlist ? HB : 0) + HB - 1 - min(HB - 1, tiles * 64 + min(nq, 63));  // descending cost
  };
  for (int w = tid; w < nwork; w += 1024) atomicAdd(&hist[key(w)], 1);
  __syncthreads();
  // exclusive scan of 8192 bins: 8 per thread
  int loc[8], acc = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    loc[j] = acc;
    acc += hist[tid * 8 + j];
  }
  part[tid] = acc;
  __syncthreads();
  for (int off = 1; off < 1024; off <<= 1) {
    const int v = tid >= off ? part[tid - off] : 0;
    __syncthreads();
    part[tid] += v;
    __syncthreads();
  }
  const int base = tid ? part[tid - 1] : 0;
  __syncthreads();
#pragma unroll
  for (int j = 0; j < 8; ++j) hist[tid * 8 + j] = base + loc[j];
  __syncthreads();
  for (int w = tid; w < nwork; w += 1024) out[atomicAdd(&hist[key(w)], 1)] = in[w];
}

cudaError_t launch_bucket(const int32_t* probes, int64_t nq, int npb, int nlist, const int64_t* list_off, int k,
                          const int32_t* qcfg, const int32_t* ra, const Bucketing& b, cudaStream_t st) {
  (void)k;
  const int64_t npairs = nq * npb;
  const int nv = ra ? 2 * nlist : nlist;  // virtual lists
  cudaMemsetAsync(b.lcount, 0, sizeof(int32_t) * nv, st);
  cudaMemsetAsync(b.bfill, 0, sizeof(int32_t) * nv, st);
  cudaMemsetAsync(b.counter, 0, sizeof(int32_t), st);
  const int grid = (int)min64(kNumSMs * 8, (npairs + 255) / 256);
  if (npairs) k_count_pairs<<<grid, 256, 0, st>>>(probes, npairs, npb, nlist, ra, b.lcount);
  cudaError_t e;
  if ((e = launch_scan_i32(b.lcount, nv, b.boff, st)) != cudaSuccess) return e;
  if (npairs) k_bucket_fill<<<grid, 256, 0, st>>>(probes, npairs, npb, nlist, ra, b.boff, b.bfill, b.bq);
  k_work_count<<<(nv + 255) / 256, 256, 0, st>>>(b.lcount, nv, qcfg, b.wcount);
  if ((e = launch_scan_i32(b.wcount, nv, b.woff, st)) != cudaSuccess) return e;
  k_work_fill<<<(nv + 255) / 256, 256, 0, st>>>(b.wcount, b.woff, b.boff, nv, qcfg, b.witems_unsorted);
  k_sort_work<<<1, 1024, 0, st>>>(b.witems_unsorted, b.woff + nv, b.boff, list_off, nlist, qcfg, b.witems);
  return cudaGetLastError();
}

// Region capacity of pair (q, j): min(capk, |list|) when the SIMT scan selects locally (k <= 1024,
// capk > 0), else |list| (every candidate that survives the bitset may be emitted).
__device__ __forceinline__ int64_t pair_cap(int64_t len, int k, int capk) {
  return (capk > 0 && k <= kLocalSelectMaxK) ? min64(capk, len) : len;
}

// one warp per query: qtot[q] = sum_j cap(q, j)
__global__ void k_query_tot(const int32_t* __restrict__ probes, int64_t nq, int npb,
                            const int64_t* __restrict__ list_off, int k, int capk, int64_t* qtot) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t q = warp; q < nq; q += nwarps) {
    int64_t acc = 0;
    for (int j = lane; j < npb; j += 32) {
      const int l = probes[q * npb + j];
      acc += pair_cap(list_off[l + 1] - list_off[l], k, capk);
    }
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(MV_FULL, acc, o);
    if (lane == 0) qtot[q] = acc;
  }
}

// one warp per query: poff[q*npb + j] = qbase[q] + sum_{j' < j} cap(q, j')
__global__ void k_pair_off(const int32_t* __restrict__ probes, int64_t nq, int npb, const int64_t* __restrict__ list_off,
                           int k, int capk, const int64_t* __restrict__ qbase, int64_t* poff) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t q = warp; q < nq; q += nwarps) {
    int64_t run = qbase[q];
    for (int j0 = 0; j0 < npb; j0 += 32) {
      const int j = j0 + lane;
      int64_t c = 0;
      if (j < npb) {
        const int l = probes[q * npb + j];
        c = pair_cap(list_off[l + 1] - list_off[l], k, capk);
      }
      int64_t incl = c;
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t v = __shfl_up_sync(MV_FULL, incl, o);
        if (lane >= o) incl += v;
      }
      if (j < npb) poff[q * npb + j] = run + incl - c;
      run += __shfl_sync(MV_FULL, incl, 31);
    }
  }
}

cudaError_t launch_pair_offsets(const int32_t* probes, int64_t nq, int npb, const int64_t* list_off, int k, int capk,
                                const Bucketing& b, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  const int grid = (int)min64(kNumSMs * 8, (nq * 32 + 255) / 256);
  int64_t* qbase = b.qtot + (nq + 1);  // second half of the qtot allocation
  k_query_tot<<<grid, 256, 0, st>>>(probes, nq, npb, list_off, k, capk, b.qtot);
  cudaError_t e = launch_scan_i64(b.qtot, nq, qbase, st);
  if (e != cudaSuccess) return e;
  k_pair_off<<<grid, 256, 0, st>>>(probes, nq, npb, list_off, k, capk, qbase, b.poff);
  return cudaGetLastError();
}

}  // namespace mv
