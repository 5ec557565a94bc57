// k_bucket.cu -- §8 row a4: invert the (query, probed list) pairs into per-list query buckets
// and work items.  The grouping is the B200 form of the paper's cache-aware idea: "reuse the
// accessed data vectors as much as possible for multiple queries" (§3.2.1),
// because in step 2 "different queries do not necessarily access the same buckets"
// (§3.4).  A counting sort by list id: histogram, exclusive scan, scatter.
// Also the per-pair candidate-region offsets, the seeding split and the work-item order.
//
// One cooperative launch (grid-wide barriers between the steps) replaces a dozen small kernels:
//   0  zero the counters; the work-item shape {query chunk, planes} (qlo_any decides FLAT's)
//   1  per query (warp): ra[q] = the fewest nearest lists holding >= need candidates (seeding),
//      the query's region capacity, and the pair counts per virtual list
//   2  grid-wide exclusive scans: pair counts -> bucket offsets, capacities -> query bases
//   3  per query: pair region offsets + bucket fill; per virtual list: work-item counts
//   4  grid-wide exclusive scan of the work-item counts
//   5  work items (virtual list, first bucket position) + histogram of their cost keys
//   6  longest-first order (counting sort by cost, seeding phase first: block 0 scans the
//      histogram, every block scatters)
#include <cooperative_groups.h>

#include "mv_internal.cuh"

namespace cg = cooperative_groups;

namespace mv {

constexpr int kPlanThreads = 1024;

// With the seeding split (ra != nullptr) every pair p = q*npb + r of list l is an entry of virtual
// list l + nlist (phase B, region capacity |l|), and the pairs of query q with r < ra[q] are also
// entries of virtual list l (phase A: the first min(|l|, capA) rows, region capacity the same,
// pair id npairs + p).  Without it, pair p is an entry of virtual list l.

// Region capacity of a pair: |list| (every candidate that survives the bitset may be emitted).

// single-block exclusive scan out[0..n] (out[n] = total) with all kPlanThreads threads
template <typename T>
__device__ void block_exclusive_scan(const T* __restrict__ in, int64_t n, T* __restrict__ out, T* part) {
  const int tid = threadIdx.x;
  const int64_t per = (n + kPlanThreads - 1) / kPlanThreads;
  const int64_t s = tid * per, e = min64(n, s + per);
  T acc = 0;
  for (int64_t i = s; i < e; ++i) acc += in[i];
  part[tid] = acc;
  __syncthreads();
  for (int off = 1; off < kPlanThreads; off <<= 1) {
    const T v = tid >= off ? part[tid - off] : (T)0;
    __syncthreads();
    part[tid] += v;
    __syncthreads();
  }
  T run = tid ? part[tid - 1] : (T)0;
  for (int64_t i = s; i < e; ++i) {
    out[i] = run;
    run += in[i];
  }
  if (tid == kPlanThreads - 1) out[n] = part[kPlanThreads - 1];
  __syncthreads();
}

// Grid-wide exclusive scan out[0..n] (out[n] = total) in two passes separated by a grid barrier:
// block b owns the contiguous segment [b*seg, (b+1)*seg).  Pass 1 writes the segment sum to
// bsum[b]; pass 2 adds the sums of the earlier segments and scans the segment 1024 entries at a
// time (coalesced loads, warp shuffles).  All threads of every block must call both passes.
__device__ __forceinline__ void plan_segment(int64_t n, int64_t& s, int64_t& e) {
  const int64_t seg = (n + gridDim.x - 1) / gridDim.x;
  s = min64(n, (int64_t)blockIdx.x * seg);
  e = min64(n, s + seg);
}

// block-wide sum, returned to every thread (red: 32 shared slots)
__device__ __forceinline__ int64_t plan_block_sum(int64_t v, int64_t* red) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(MV_FULL, v, o);
  __syncthreads();
  if (lane == 0) red[warp] = v;
  __syncthreads();
  int64_t t = lane < (kPlanThreads >> 5) ? red[lane] : 0;
  for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(MV_FULL, t, o);
  return t;
}

template <typename T>
__device__ void grid_scan_pass1(const T* __restrict__ in, int64_t n, int64_t* bsum, int64_t* red) {
  int64_t s, e;
  plan_segment(n, s, e);
  int64_t acc = 0;
  for (int64_t i = s + threadIdx.x; i < e; i += kPlanThreads) acc += in[i];
  acc = plan_block_sum(acc, red);
  if (threadIdx.x == 0) bsum[blockIdx.x] = acc;
}

template <typename T>
__device__ void grid_scan_pass2(const T* __restrict__ in, int64_t n, T* __restrict__ out, const int64_t* bsum,
                                int64_t* red) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  int64_t s, e;
  plan_segment(n, s, e);
  int64_t off = 0;
  for (int i = threadIdx.x; i < (int)blockIdx.x; i += kPlanThreads) off += bsum[i];
  off = plan_block_sum(off, red);
  for (int64_t c = s; c < e; c += kPlanThreads) {
    const int64_t i = c + threadIdx.x;
    const int64_t v = i < e ? (int64_t)in[i] : 0;
    int64_t incl = v;
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t u = __shfl_up_sync(MV_FULL, incl, o);
      if (lane >= o) incl += u;
    }
    __syncthreads();
    if (lane == 31) red[warp] = incl;
    __syncthreads();
    if (warp == 0) {
      int64_t w = red[lane];
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t u = __shfl_up_sync(MV_FULL, w, o);
        if (lane >= o) w += u;
      }
      red[lane] = w;
    }
    __syncthreads();
    if (i < e) out[i] = (T)(off + (warp ? red[warp - 1] : 0) + incl - v);
    off += red[31];
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) out[n] = (T)off;
}

__global__ void __launch_bounds__(kPlanThreads) k_plan(const PlanArgs a) {
  cg::grid_group grid = cg::this_grid();
  __shared__ int64_t part64[kPlanThreads];
  __shared__ int64_t red[32];
  const int tid = threadIdx.x, lane = tid & 31;
  const int64_t gtid = blockIdx.x * (int64_t)blockDim.x + tid;
  const int64_t gthreads = (int64_t)gridDim.x * blockDim.x;
  const int64_t gwarp = gtid >> 5, gwarps = gthreads >> 5;
  const int nq_i = (int)a.nq, npb = a.npb, nlist = a.nlist;
  const int nv = a.split ? 2 * nlist : nlist;
  const Bucketing& b = a.b;

  // 0 ---------------------------------------------------------------------------------------
  for (int64_t i = gtid; i < nv; i += gthreads) {
    b.lcount[i] = 0;
    b.bfill[i] = 0;
  }
  for (int64_t i = gtid; i < kPlanCostBins; i += gthreads) b.whist[i] = 0;
  if (gtid == 0) {
    const bool sp = a.qlo_any != nullptr && *a.qlo_any != 0;
    a.qcfg[0] = sp ? a.qc_split : a.qc_exact;
    a.qcfg[1] = sp ? a.p_split : a.p_exact;
    b.counter[0] = 0;
    b.counter[1] = 0;
  }
  grid.sync();
  const int qchunk = a.qcfg[0];
  int32_t* ra = a.split ? a.ra : nullptr;

  // 1 ---------------------------------------------------------------------------------------
  for (int64_t q = gwarp; q < nq_i; q += gwarps) {
    const int32_t* pq = a.probes + q * npb;
    int64_t run = 0, capsum = 0;
    int r = npb;
    for (int j0 = 0; j0 < npb; j0 += 32) {
      const int j = j0 + lane;
      int64_t len = 0;
      if (j < npb) {
        const int l = pq[j];
        len = a.list_off[l + 1] - a.list_off[l];
        capsum += len;
        if (a.split) len = min64(len, a.capA);  // phase A reads a prefix of each list
      }
      int64_t incl = len;
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t v = __shfl_up_sync(MV_FULL, incl, o);
        if (lane >= o) incl += v;
      }
      const uint32_t hit = __ballot_sync(MV_FULL, j < npb && run + incl >= a.need);
      if (hit && r == npb) r = j0 + __ffs(hit);  // ranks 0 .. first hit
      run += __shfl_sync(MV_FULL, incl, 31);
    }
    // phase-A regions: the prefixes of the ra nearest lists
    for (int j = lane; j < r && ra; j += 32) {
      const int l = pq[j];
      capsum += min64(a.list_off[l + 1] - a.list_off[l], a.capA);
    }
    for (int o = 16; o > 0; o >>= 1) capsum += __shfl_xor_sync(MV_FULL, capsum, o);
    if (lane == 0) {
      if (ra) ra[q] = r;
      b.qtot[q] = capsum;
    }
    for (int j = lane; j < npb; j += 32) {
      const int l = pq[j];
      if (ra) {
        atomicAdd(b.lcount + l + nlist, 1);
        if (j < r) atomicAdd(b.lcount + l, 1);
      } else {
        atomicAdd(b.lcount + l, 1);
      }
    }
  }
  grid.sync();

  // 2 ---------------------------------------------------------------------------------------
  grid_scan_pass1<int32_t>(b.lcount, nv, b.bsum, red);
  grid_scan_pass1<int64_t>(b.qtot, a.nq, b.bsum + kPlanMaxBlocks, red);
  grid.sync();
  grid_scan_pass2<int32_t>(b.lcount, nv, b.boff, b.bsum, red);
  grid_scan_pass2<int64_t>(b.qtot, a.nq, b.qtot + (a.nq + 1), b.bsum + kPlanMaxBlocks, red);
  grid.sync();

  // 3 ---------------------------------------------------------------------------------------
  const int64_t* qbase = b.qtot + (a.nq + 1);
  for (int64_t q = gwarp; q < nq_i; q += gwarps) {
    const int32_t* pq = a.probes + q * npb;
    const int r = ra ? ra[q] : npb;
    int64_t run = qbase[q];
    for (int j0 = 0; j0 < npb; j0 += 32) {
      const int j = j0 + lane;
      int64_t c = 0;
      if (j < npb) {
        const int l = pq[j];
        c = a.list_off[l + 1] - a.list_off[l];
        const int v = ra ? l + nlist : l;
        b.bq[b.boff[v] + atomicAdd(b.bfill + v, 1)] = (int32_t)(q * npb + j);
      }
      int64_t incl = c;
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t v = __shfl_up_sync(MV_FULL, incl, o);
        if (lane >= o) incl += v;
      }
      if (j < npb) b.poff[q * npb + j] = run + incl - c;
      run += __shfl_sync(MV_FULL, incl, 31);
    }
    // phase-A entries (pair id npairs + q*npb + j), regions after the query's phase-B regions
    for (int j0 = 0; ra && j0 < r; j0 += 32) {
      const int j = j0 + lane;
      int64_t c = 0;
      if (j < r) {
        const int l = pq[j];
        c = min64(a.list_off[l + 1] - a.list_off[l], a.capA);
        b.bq[b.boff[l] + atomicAdd(b.bfill + l, 1)] = (int32_t)(a.nq * npb + q * npb + j);
      }
      int64_t incl = c;
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t v = __shfl_up_sync(MV_FULL, incl, o);
        if (lane >= o) incl += v;
      }
      if (j < r) b.poff[a.nq * npb + q * npb + j] = run + incl - c;
      run += __shfl_sync(MV_FULL, incl, 31);
    }
  }
  {  // work-item counts over this block's segment, and their sum (pass 1 of step 4's scan)
    int64_t s, e, acc = 0;
    plan_segment(nv, s, e);
    for (int64_t v = s + tid; v < e; v += kPlanThreads) {
      const int c = (b.lcount[v] + qchunk - 1) / qchunk;
      b.wcount[v] = c;
      acc += c;
    }
    acc = plan_block_sum(acc, red);
    if (tid == 0) b.bsum[blockIdx.x] = acc;
  }
  grid.sync();

  // 4 ---------------------------------------------------------------------------------------
  grid_scan_pass2<int32_t>(b.wcount, nv, b.woff, b.bsum, red);
  grid.sync();

  // 5 ---------------------------------------------------------------------------------------
  // work items, and the histogram of their cost keys: descending cost = 64 * tiles + queries
  // (tiles = ceil(|list| / 128), queries of the list's first item); every phase-A item (virtual
  // list < nlist) precedes every phase-B item.  A list's items (several when more than qchunk
  // queries probe it) get one key and consecutive places in the order, so the static schedule
  // runs them at the same time on neighbouring CTAs and the siblings' tile reads hit L2 (round 2
  // sorted items one by one: c4's phase B read 1.83x its algorithmic bytes from DRAM)
  constexpr int HB = kPlanCostBins / 2;
  auto key = [&](int v) {
    const int l = v >= nlist ? v - nlist : v;
    const int nqw = min(qchunk, b.boff[v + 1] - b.boff[v]);
    int64_t len = a.list_off[l + 1] - a.list_off[l];
    if (a.split && v < nlist) len = min64(len, a.capA);
    const int tiles = (int)min64((len + 127) / 128, 63);
    return (v >= nlist ? HB : 0) + HB - 1 - min(HB - 1, tiles * 64 + min(nqw, 63));
  };
  for (int64_t v = gtid; v < nv; v += gthreads) {
    const int n = b.wcount[v];
    if (n) atomicAdd(b.whist + key((int)v), n);
  }
  grid.sync();

  // 6 ---------------------------------------------------------------------------------------
  // counting sort by the cost key: block 0 scans the histogram, then every list reserves its
  // items' places in one piece (kItemMulti marks the items of a list with siblings)
  if (blockIdx.x == 0) {
    int loc[8], acc = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      loc[j] = acc;
      acc += b.whist[tid * 8 + j];
    }
    int32_t* p32 = reinterpret_cast<int32_t*>(part64);
    p32[tid] = acc;
    __syncthreads();
    for (int off = 1; off < kPlanThreads; off <<= 1) {
      const int v = tid >= off ? p32[tid - off] : 0;
      __syncthreads();
      p32[tid] += v;
      __syncthreads();
    }
    const int base = tid ? p32[tid - 1] : 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) b.whist[tid * 8 + j] = base + loc[j];
  }
  grid.sync();
  for (int64_t v = gtid; v < nv; v += gthreads) {
    const int n = b.wcount[v], bb = b.boff[v];
    if (!n) continue;
    const int o = atomicAdd(b.whist + key((int)v), n);
    const int x = (int)v | (n > 1 ? kItemMulti : 0);
    for (int c = 0; c < n; ++c) b.witems[o + c] = make_int2(x, bb + c * qchunk);
  }
}

// single-CTA exclusive scan for the add path (n up to a few million)
template <typename T>
__global__ void __launch_bounds__(kPlanThreads) k_scan_single(const T* __restrict__ in, int64_t n, T* __restrict__ out) {
  __shared__ T part[kPlanThreads];
  block_exclusive_scan<T>(in, n, out, part);
}

cudaError_t launch_scan_i32(const int32_t* in, int n, int32_t* out, cudaStream_t st) {
  k_scan_single<int32_t><<<1, kPlanThreads, 0, st>>>(in, n, out);
  return cudaGetLastError();
}
cudaError_t launch_scan_i64(const int64_t* in, int64_t n, int64_t* out, cudaStream_t st) {
  k_scan_single<int64_t><<<1, kPlanThreads, 0, st>>>(in, n, out);
  return cudaGetLastError();
}

cudaError_t launch_plan(const PlanArgs& a, cudaStream_t st) {
  static int grid = 0;
  if (grid == 0) {
    int dev = 0, nsm = kNumSMs, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_plan, kPlanThreads, 0);
    // two blocks per SM (grid-wide barriers cost more with more blocks)
    grid = std::min(kPlanMaxBlocks, nsm * std::max(1, std::min(per, 2)));
  }
  PlanArgs args = a;
  void* kargs[] = {&args};
  return cudaLaunchCooperativeKernel((const void*)k_plan, dim3(grid), dim3(kPlanThreads), kargs, 0, st);
}

}  // namespace mv
