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
constexpr int kMaxD = 512;            // the tensor-core kernels stage query operands of <= 512 dims
constexpr int kMaxNprobe = 1024;      // ranked probes per query (k_probe_select's register list)
constexpr int kNumSMs = 148;
// SQ8 query-side digit planes (kind::i8, base 2^7): the scan is a filter whose error bound E_q
// includes the last digit's residual; the band is re-scored exactly, so two planes
// suffice (round 1 used four for an exact in-scan fp64 value)
constexpr int kSq8Planes = 2;
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
// Per-index tuning options (mv_index_set_option).  None of them changes a result: they pick
// launch shapes and the seeding sample.  0 = automatic.
// ------------------------------------------------------------------------------------------
namespace mv {
struct Options {
  int seeding = 1;          // 0: no seeding phase (phase B alone, every candidate emitted)
  int64_t need = 0;         // seeding sample size (candidates); clamped to >= max(2k, k + 32)
  int64_t capa = 0;         // rows per list of the seeding sample (16-row multiple)
  int sq8_qc = 0;           // SQ8 queries per scan work item (16..64)
  int flat_qc = 0;          // FLAT queries per scan work item (16..128)
  int coarse_nqb = 0, coarse_cs = 0, coarse_epi = 0, coarse_nacc = 0;  // coarse GEMM launch shape
  int64_t workspace = 0;    // per-search scratch budget in bytes (0: half of the free device memory)
  int64_t scan_trace = 0;   // -DMV_SCAN_TRACE builds: device address of the phase-B timeline buffer
  int async_host = 0;       // 1: searches with pinned host buffers return without synchronising
  int large_k_select = 0;   // k > 256: 0 streaming select (staged radix fallback), 1 sample-threshold select, 2 staged radix only
  int big_ctas = 0;         // k > 256 staged select: CTAs per SM of its first launch (1..4; 0 = 2)
  int64_t big_cap = 0;      // ... and its stage capacity in keys (0: the most that fits big_ctas per SM)
};

// k > 256 select launch choices: Options::large_k_select / big_ctas, and a lower bound on the
// candidates per query when the caller knows one (the seeding sample: >= need)
struct BigSel {
  int mode = 0;
  int ctas = 0;
  int64_t cap = 0;
  int64_t tlo = 0;
  // streaming select (k_select_stream, mode 0): the seeding select writes each query's smallest
  // key to kmin; the final select bins the keys over [kmin, khi] (khi = the seeding bound tau)
  uint64_t* kmin = nullptr;
  const uint64_t* khi = nullptr;
};
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
                                int64_t* sorted_ids, uint32_t* row_of_rank, cudaStream_t st);
// profiling counters: *out += sum of v[0..n) / += n
cudaError_t launch_sum_i32(const int32_t* v, int64_t n, int npb, const int32_t* ra, unsigned long long* out,
                           cudaStream_t st);
cudaError_t launch_count_add(int64_t n, unsigned long long* out, cudaStream_t st);
// *out = max(*out, max_i v[i]) for non-negative doubles (atomicMax on the bit patterns)
cudaError_t launch_max_f64(const double* v, int64_t n, unsigned long long* out, cudaStream_t st);
cudaError_t launch_check_ids(const int64_t* ids, int64_t n, int* flag, cudaStream_t st);
cudaError_t launch_new_sizes(const int32_t* add, int nlist, const int64_t* old_off, int64_t* out, cudaStream_t st);
cudaError_t launch_iota_i32(int32_t* out, int64_t n, cudaStream_t st);

// k_coarse.cu
cudaError_t launch_query_prep(const float* q, int64_t nq, int d, int dpad, float* qpad, float* qnorm, cudaStream_t st);
cudaError_t launch_centroid_prep(const float* c, int nlist, int d, int dpad, float* cpad, float* cnorm, cudaStream_t st);
// nprobe >= nlist: every bucket, in id order
cudaError_t launch_all_lists(int64_t nq, int nlist, int32_t* probes, cudaStream_t st);

// k_bucket.cu
struct Bucketing {
  int32_t* lcount;   // nlist      pairs per list
  int32_t* boff;     // nlist+1    exclusive scan of lcount
  int32_t* bfill;    // nlist      scratch
  int32_t* bq;       // nq*npb (x2 with seeding)  pair ids grouped by list
  int32_t* wcount;   // nlist      work items per list
  int32_t* woff;     // nlist+1
  int2* witems;      // <= nlist + nq*npb   (list | kItemMulti, first bucket position), longest first
  int64_t* qtot;     // nq+1       per-query candidate capacity, then exclusive scan
  int64_t* poff;     // nq*npb (x2 with seeding: phase-A entries at nq*npb + p)  region offset per pair
  int32_t* pcnt;     // nq*npb (x2 with seeding)  candidates written per pair
  int32_t* counter;  // 2          scan work-item counters (phase A, phase B)
  int32_t* whist;    // kPlanCostBins  work-item cost histogram, then its exclusive scan
  int64_t* bsum;     // 2 x kPlanMaxBlocks  per-block partial sums of the grid-wide scans
};
constexpr int kPlanCostBins = 8192;
// work-item flag (bit 30 of the virtual list): the list has several items (sibling reads share L2)
constexpr int kItemMulti = 1 << 30;
constexpr int kPlanMaxBlocks = 1024;
// a4 in one cooperative launch (k_bucket.cu).  With the seeding split the pairs of query q with
// probe rank < ra[q] form a first phase (virtual lists 0..nlist-1, work items first) and the
// others a second (virtual lists nlist..2*nlist-1); arrays are then sized for 2*nlist lists.
struct PlanArgs {
  const int32_t* probes;   // nq x npb, best-first
  int64_t nq;
  int npb, nlist, k;
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

// k_kmeans.cu: Lloyd k-means accumulation and update
cudaError_t launch_kmeans_accum(const float* x, int64_t n, int d, const int32_t* lists, double* sums,
                                unsigned long long* cnt, cudaStream_t st);
cudaError_t launch_kmeans_update(const double* sums, const unsigned long long* cnt, int nlist, int d, int spherical,
                                 float* c, cudaStream_t st);
// k_pq.cu: IVF_PQ encode (add path) and the query-major ADC scan
struct PqScanParams {
  int metric, dpad, M, dsub, npb, phase, rowcap;
  int64_t nq;
  const float* qpad;        // nq x dpad
  const float* codebooks;   // [M][256][dsub]
  const int32_t* probes;    // nq x npb
  const int32_t* ra;        // phase A: the query's seeding lists
  const uint64_t* tau;      // phase B: emit keys <= tau_q
  const int64_t* list_off;
  const uint8_t* codes;     // ntotal x M, list-major
  const uint32_t* rank;
  const int64_t* ids;
  const uint8_t* bitset;
  int64_t nbits;
  const int64_t* poff;
  int32_t* pcnt;
  uint64_t* part;
};
cudaError_t launch_pq_encode(const float* xpad, const int64_t* ids, const int32_t* sorted_idx,
                             const int32_t* sorted_list, int64_t n, int dpad, int M, int dsub, const float* cb,
                             const int64_t* new_off, const int64_t* old_off, const int32_t* add_off, uint8_t* payload,
                             double* norms, int64_t* out_ids, cudaStream_t st);
cudaError_t launch_pq_scan(const PqScanParams& p, cudaStream_t st);
cudaError_t launch_check_identity(const int64_t* sorted_ids, int64_t n, int* flag, cudaStream_t st);
// k_filter.cu: strategy E's range bitmap and vector fusion
cudaError_t launch_attr_bitset(const int64_t* ids, const int64_t* attr, int64_t n, int64_t lo, int64_t hi,
                               uint8_t* bitset, int64_t nbits, cudaStream_t st);
constexpr int kMaxFuse = 16;  // vectors per entity (mv_fuse_rows)
struct FuseArgs {
  const float* part[kMaxFuse];
  int dim[kMaxFuse], off[kMaxFuse];
  float w[kMaxFuse];
  int m, dtot;
};
cudaError_t launch_fuse_rows(const FuseArgs& a, int64_t n, float* out, cudaStream_t st);

// k_scan_tc.cu (tcgen05 path): a filter-and-emit scan run in two phases
struct TcScanParams {
  int type, metric, dpad, k, npb, qchunk, nchunks, nstage, ncol, tmem_cols, nacc, atom;
  int qchunk_split;        // FLAT: queries per work item when the queries need the lo plane (P = 2)
  const int32_t* cfg;      // device {query chunk, planes} of this search (launch_scan_cfg)
  int nlist;               // virtual list v >= nlist is list v - nlist (phase-B pairs)
  int phase;               // 0: seeding phase A (emit every candidate); 1: phase B (emit keys <= tau_q)
  int key32;               // phase A: emit 4-byte distance keys into a u32 view of the regions (k > 256)
  int rowcap;              // rows scanned per list in this launch (phase A: capA; else INT_MAX)
  int64_t nq;              // FLAT query planes are plane-major [2][nq][dpad]
  int off_x, off_q, q_bytes, off_meta, meta_bytes, off_side, off_bar, smem_total;
  int nts, side_bytes;     // side-data ring: slots and bytes per slot
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
  int64_t nbq;             // entries of bq
  const int32_t* boff;
  const int2* witems;
  const int32_t* wbeg;     // device: first work item of this launch (nullable = 0)
  const int32_t* nwitems;  // device: one past the last work item of this launch
  int32_t* counter;        // device: work items taken so far in this launch (zeroed by k_plan)
  const int64_t* poff;     // per pair: output region (capacity = the list length)
  int32_t* pcnt;           // per pair: keys emitted
  uint64_t* part;
  const uint64_t* tau;     // nq: per-query bound for phase B (exact k-th key of phase A)
  int approx_always;       // FLAT: stored values not tf32-exact -> filter mode for every search (SQ8: always)
  const float* qerr;       // filter mode: E_q, the bound on |approximate - exact badness|
  unsigned long long* prof;  // -DMV_SCAN_TRACE builds only: CTA-0 timeline
};
bool tc_scan_plan(int type, int dpad, int k, double qpl, bool ids, const Options& o, TcScanParams& p);  // qpl: queries per probed list
// the payload's tensor maps: boxes of 128, 64, 32, 16 rows (one swizzle atom wide)
struct XMaps {
  CUtensorMap m[4];
};
cudaError_t launch_scan_tc(const XMaps& xm, const TcScanParams& p, cudaStream_t st);
// filter-mode error model: FLAT ex / eq = relative representation error of the
// stored value / of the query as the MMA sees them; xmax2 = max ||x||^2 (SQ8: ||x_hat||^2) over the
// index
struct FlatErr {
  double ex, eq, xmax2;
  int metric;
};
cudaError_t launch_qplanes(int type, const float* qpad, int64_t nq, int dpad, const float* vmin, const float* vdiff,
                           uint8_t* out, float* qscale, double* qa, double* qnorm, const FlatErr* fe, float* qerr,
                           cudaStream_t st);
cudaError_t launch_tf32_check(const float* x, int64_t n, int* flag, cudaStream_t st);

// k_coarse_tc.cu (tcgen05 coarse GEMM -> score matrix S, then a warp-per-query top-nprobe)
// The coarse step never materialises the nq x nlist score matrix: the same GEMM runs twice
// (bitwise-identical scores).  Pass 0 writes only the minimum score key of every 32-centroid group
// (G); k_group_bound picks, per query, the nprobe-th smallest (group minimum, group id) pair; pass
// 1 appends the (score key, centroid) keys at or below it -- at most 32 nprobe per query -- and a
// warp per query sorts out the nprobe best (k_probe_final).
struct CoarseParams {
  int64_t nq;
  int nlist, nchunks, nstage, nprobe, nqb, csplit, tmem_cols, metric, smem_total;
  int nepi, nacc;          // epilogue warps (multiple of 4, <= 16), TMEM accumulators (<= 4)
  int mode;                // 0: group minima -> G; 1: the selected groups' keys -> cand
  int qm;                  // 1: k_coarse_qm (queries on the MMA's M side, dpad <= 128)
  const float* cnorm;
  uint32_t* G;             // nq x ldg: minimum score key of each 32-centroid group (ldg = 4 ceil(nlist/128))
  int64_t ldg;
  uint64_t* gbound;        // nq: (bound score key << 32) | bound group id
  int16_t* gslot;          // nq x ceil(nlist/32): rank of the group among the query's nprobe selected, or -1
  uint64_t* cand;          // nq x ccap: per selected group 32 slots, its passing (score key << 32 | centroid) first
  uint8_t* ccnt;           // nq x nprobe: passing keys per slot group
  int ccap;                // 32 nprobe
  const int* qlo_any;      // device: some query needs its lo plane (nullable = yes)
  int32_t* probes;
};
bool coarse_tc_plan(int dpad, int nprobe, int64_t nq, int nlist, int nsm, const Options& o, CoarseParams& p);
cudaError_t launch_coarse_tc(const CUtensorMap* cmap, const CUtensorMap* qmap, const CoarseParams& p, int64_t nq,
                             cudaStream_t st);
// plane-major tf32 split of n rows; *lo_any (nullable) |= 1 when some lo element is nonzero
cudaError_t launch_hilo(const float* x, int64_t n, int d, int dpad, float* out, int* lo_any, cudaStream_t st);

// k_select.cu
// final select over the pairs of each query; with tau != nullptr instead: tau[q] = the k-th best
// key over the first nuse[q] pairs of query q (left untouched when they hold fewer than k).
// tmax bounds the candidates of one query; over (nq bytes, nullable) is scratch for k > 256.
// big_mode (k > 256): 0 = the staged radix select (default), 1 = the sample-threshold select with
// the staged radix select as its fallback.  over: 2 nq bytes of scratch for k > 256.
cudaError_t launch_final_select(const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq, int npb,
                                int k, int metric, const int64_t* sorted_ids, float* out_d, int64_t* out_i,
                                int64_t tmax, uint8_t* over, BigSel bsel, cudaStream_t st);
// k > 256 seeding bound from phase A's 4-byte distance keys (scan key32); tmax bounds a query's sample
cudaError_t launch_tau32(const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq, int npb,
                         const int32_t* nuse, int k, uint64_t* tau, uint64_t* kmin, int64_t tmax, cudaStream_t st);
cudaError_t launch_tau_select(const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq, int npb,
                              const int32_t* nuse, int k, uint64_t* tau, int64_t tmax, uint8_t* over,
                              const int* gate, BigSel bsel, cudaStream_t st);
// k <= 256: the final select with the filter mode's fused exact re-scoring (k_final_warp<R, type>);
// rgate (nullable = always): refine only when *rgate != 0, else the plain exact select
cudaError_t launch_final_refine(int type, const int64_t* poff, const int32_t* pcnt, const uint64_t* part, int64_t nq,
                                int npb, int k, int metric, const int64_t* sorted_ids, float* out_d, int64_t* out_i,
                                const float* qerr, const float* qpad, int dpad, const void* payload,
                                const uint32_t* row_of_rank, const float* vmin, const float* vdiff, const float* sq8_t,
                                const int* rgate, uint64_t* tau2, int* notgate, cudaStream_t st);
// k > 256, filter mode: exact fp64 re-scoring in place of the keys at or below tau2[q] + 2 qerr[q];
// gate (nullable): skipped when *gate == 0
cudaError_t launch_rekey(int type, const int64_t* poff, const int32_t* pcnt, uint64_t* part, int64_t nq, int npb,
                         const uint64_t* tau2, const float* qerr, int metric, const float* qpad, int dpad,
                         const void* payload, const uint32_t* row_of_rank, const float* vmin, const float* vdiff,
                         const float* sq8_t, const int* gate, cudaStream_t st);
cudaError_t launch_fill_pad(int64_t n, int metric, float* d, int64_t* i, cudaStream_t st);
cudaError_t launch_merge2(int metric, const float* ad, const int64_t* ai, const float* bd, const int64_t* bi,
                          int64_t nq, int k, float* od, int64_t* oi, cudaStream_t st);

}  // namespace mv
