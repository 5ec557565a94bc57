// k_add.cu -- build side of the boundary (§8 row a0): SQ8 train/encode, norms, list-major
// scatter, id ranks.  Not in the timed search path.
//
// PAPER.md:503-514 (§3.1): each vector goes to the bucket of its closest centroid (the
// assignment itself reuses the coarse kernel with nprobe = 1, k_coarse.cu).
// PAPER.md:516-520 (§3.1), 803: SQ8 stores one byte per dimension; the formula is reading O3
// (DESIGN.md §2): code = floor(255 * clamp((x - vmin) / vdiff, 0, 1)), fp32, one rounding per
// operation -- bit-exact with oracle.sq8_encode.
#include "mv_internal.cuh"

namespace mv {

__global__ void k_sq8_minmax(const float* __restrict__ x, int64_t n, int d, uint32_t* kmin, uint32_t* kmax) {
  const int j = blockIdx.x * 32 + threadIdx.x;
  if (j >= d) return;
  uint32_t lo = 0xffffffffu, hi = 0u;
  for (int64_t r = (int64_t)blockIdx.y * blockDim.y + threadIdx.y; r < n; r += (int64_t)gridDim.y * blockDim.y) {
    const uint32_t kk = f2key(x[r * d + j]);
    lo = min(lo, kk);
    hi = max(hi, kk);
  }
  atomicMin(kmin + j, lo);
  atomicMax(kmax + j, hi);
}

__global__ void k_sq8_finish(const uint32_t* kmin, const uint32_t* kmax, int d, float* vmin, float* vdiff) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= d) return;
  const float lo = key2f(kmin[j]), hi = key2f(kmax[j]);
  vmin[j] = lo;
  vdiff[j] = __fsub_rn(hi, lo);
}

cudaError_t launch_sq8_minmax(const float* x, int64_t n, int d, float* vmin, float* vdiff, cudaStream_t st) {
  uint32_t* keys = nullptr;
  cudaError_t e = cudaMallocAsync(&keys, sizeof(uint32_t) * 2 * d, st);
  if (e != cudaSuccess) return e;
  cudaMemsetAsync(keys, 0xff, sizeof(uint32_t) * d, st);
  cudaMemsetAsync(keys + d, 0, sizeof(uint32_t) * d, st);
  dim3 blk(32, 8);
  int gy = (int)min64(1024, (n + 7) / 8);
  k_sq8_minmax<<<dim3((d + 31) / 32, max(gy, 1)), blk, 0, st>>>(x, n, d, keys, keys + d);
  k_sq8_finish<<<(d + 127) / 128, 128, 0, st>>>(keys, keys + d, d, vmin, vdiff);
  e = cudaGetLastError();
  cudaFreeAsync(keys, st);
  return e;
}

__global__ void k_prep_rows(const float* __restrict__ x, int64_t n, int d, int dpad, float* __restrict__ out) {
  const int64_t total = n * dpad;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = t / dpad;
    const int j = (int)(t - r * dpad);
    out[t] = j < d ? x[r * d + j] : 0.0f;
  }
}

cudaError_t launch_prep_rows(const float* x, int64_t n, int d, int dpad, float* out, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  int grid = (int)min64(kNumSMs * 16, (n * dpad + 255) / 256);
  k_prep_rows<<<grid, 256, 0, st>>>(x, n, d, dpad, out);
  return cudaGetLastError();
}

__global__ void k_count_lists(const int32_t* __restrict__ lists, int64_t n, int32_t* counts) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(counts + lists[i], 1);
}

cudaError_t launch_count_lists(const int32_t* lists, int64_t n, int32_t* counts, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  int grid = (int)min64(kNumSMs * 8, (n + 255) / 256);
  k_count_lists<<<grid, 256, 0, st>>>(lists, n, counts);
  return cudaGetLastError();
}

// One warp per new row: write its payload (fp32 copy or SQ8 codes), its norm and its id at
// its list-major position new_off[l] + oldlen[l] + (rank among the new rows of list l).
__global__ void k_store_rows(int type, int metric, const float* __restrict__ xpad, const int64_t* __restrict__ ids,
                             const int32_t* __restrict__ sorted_idx, const int32_t* __restrict__ sorted_list, int64_t n,
                             int dpad, const int64_t* __restrict__ new_off, const int64_t* __restrict__ old_off,
                             const int32_t* __restrict__ add_off, void* payload, double* norms, int64_t* out_ids,
                             const float* __restrict__ vmin, const float* __restrict__ vdiff,
                             const float* __restrict__ sq8_t) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t t = warp; t < n; t += nwarps) {
    const int i = sorted_idx[t];
    const int l = sorted_list[t];
    const int64_t pos = new_off[l] + (old_off[l + 1] - old_off[l]) + (t - add_off[l]);
    const float* src = xpad + (int64_t)i * dpad;
    double acc = 0.0;
    if (type == MV_IVF_FLAT) {
      float* dst = reinterpret_cast<float*>(payload) + pos * dpad;
      for (int j = lane; j < dpad; j += 32) {
        const float v = src[j];
        dst[j] = v;
        acc = fma((double)v, (double)v, acc);
      }
    } else {
      uint8_t* dst = reinterpret_cast<uint8_t*>(payload) + pos * dpad;
      for (int j = lane; j < dpad; j += 32) {
        const float vd = vdiff[j], vm = vmin[j];
        float tt = 0.0f;
        if (vd > 0.0f) tt = __fdiv_rn(__fsub_rn(src[j], vm), vd);
        tt = fminf(fmaxf(tt, 0.0f), 1.0f);
        const int code = (int)floorf(__fmul_rn(255.0f, tt));
        dst[j] = (uint8_t)code;
        const float xh = __fadd_rn(__fmul_rn(sq8_t[code], vd), vm);  // decode, oracle op order
        acc = fma((double)xh, (double)xh, acc);
      }
    }
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(MV_FULL, acc, o);
    if (lane == 0) {
      norms[pos] = acc;
      out_ids[pos] = ids[i];
    }
  }
}

cudaError_t launch_store_rows(int type, int metric, const float* xpad, const int64_t* ids, const int32_t* sorted_idx,
                              const int32_t* sorted_list, int64_t n, int dpad, const int64_t* new_off,
                              const int64_t* old_off, const int32_t* add_off, void* payload, double* norms,
                              int64_t* out_ids, const float* vmin, const float* vdiff, const float* sq8_t,
                              cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  int grid = (int)min64(kNumSMs * 16, (n * 32 + 255) / 256);
  k_store_rows<<<grid, 256, 0, st>>>(type, metric, xpad, ids, sorted_idx, sorted_list, n, dpad, new_off, old_off,
                                     add_off, payload, norms, out_ids, vmin, vdiff, sq8_t);
  return cudaGetLastError();
}

// One block per list: move the list's previous rows to their new offsets.
__global__ void k_move_old(int esize, int dpad, const int64_t* __restrict__ old_off, const int64_t* __restrict__ new_off,
                           const uint8_t* __restrict__ old_payload, const double* __restrict__ old_norms,
                           const int64_t* __restrict__ old_ids, uint8_t* payload, double* norms, int64_t* ids) {
  const int l = blockIdx.x;
  const int64_t s = old_off[l], e = old_off[l + 1], ns = new_off[l];
  const int64_t row_bytes = (int64_t)esize * dpad;
  const int64_t nbytes = (e - s) * row_bytes;
  const uint8_t* src = old_payload + s * row_bytes;
  uint8_t* dst = payload + ns * row_bytes;
  for (int64_t b = threadIdx.x; b < nbytes; b += blockDim.x) dst[b] = src[b];
  for (int64_t r = s + threadIdx.x; r < e; r += blockDim.x) {
    norms[ns + (r - s)] = old_norms[r];
    ids[ns + (r - s)] = old_ids[r];
  }
}

cudaError_t launch_move_old(int type, int dpad, int nlist, const int64_t* old_off, const int64_t* new_off,
                            const void* old_payload, const double* old_norms, const int64_t* old_ids, int64_t old_n,
                            void* payload, double* norms, int64_t* ids, cudaStream_t st) {
  if (old_n == 0) return cudaSuccess;
  const int esize = type == MV_IVF_FLAT ? 4 : 1;
  k_move_old<<<nlist, 256, 0, st>>>(esize, dpad, old_off, new_off, (const uint8_t*)old_payload, old_norms, old_ids,
                                    (uint8_t*)payload, norms, ids);
  return cudaGetLastError();
}

__global__ void k_id_keys(const int64_t* __restrict__ ids, int64_t n, uint64_t* keys, uint32_t* vals) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    keys[i] = (uint64_t)ids[i] ^ 0x8000000000000000ull;  // signed order -> unsigned order
    vals[i] = (uint32_t)i;
  }
}

cudaError_t launch_id_keys(const int64_t* ids, int64_t n, uint64_t* keys, uint32_t* vals, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  int grid = (int)min64(kNumSMs * 8, (n + 255) / 256);
  k_id_keys<<<grid, 256, 0, st>>>(ids, n, keys, vals);
  return cudaGetLastError();
}

// rank[row] = position of (id, row) in sorted order; sorted_ids[rank] = id; row_of_rank[rank] =
// storage row (nullable: FLAT only, the filter mode's exact re-scoring reads the row back)
__global__ void k_rank_scatter(const uint64_t* __restrict__ skeys, const uint32_t* __restrict__ svals, int64_t n,
                               uint32_t* rank, int64_t* sorted_ids, uint32_t* row_of_rank) {
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
    rank[svals[t]] = (uint32_t)t;
    sorted_ids[t] = (int64_t)(skeys[t] ^ 0x8000000000000000ull);
    if (row_of_rank) row_of_rank[t] = svals[t];
  }
}

cudaError_t launch_rank_scatter(const uint64_t* skeys, const uint32_t* svals, int64_t n, uint32_t* rank,
                                int64_t* sorted_ids, uint32_t* row_of_rank, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  int grid = (int)min64(kNumSMs * 8, (n + 255) / 256);
  k_rank_scatter<<<grid, 256, 0, st>>>(skeys, svals, n, rank, sorted_ids, row_of_rank);
  return cudaGetLastError();
}

// profiling counters: *out += sum of v[q * npb + j] over j < (ra ? ra[q] : npb) / += n
__global__ void k_sum_i32(const int32_t* __restrict__ v, int64_t n, int npb, const int32_t* __restrict__ ra,
                          unsigned long long* out) {
  unsigned long long acc = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    if (!ra || (int)(i % npb) < ra[i / npb]) acc += (unsigned)v[i];
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(MV_FULL, acc, o);
  if ((threadIdx.x & 31) == 0 && acc) atomicAdd(out, acc);
}
__global__ void k_count_add(int64_t n, unsigned long long* out) { *out += (unsigned long long)n; }

cudaError_t launch_sum_i32(const int32_t* v, int64_t n, int npb, const int32_t* ra, unsigned long long* out,
                           cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  k_sum_i32<<<(int)min64(kNumSMs * 4, (n + 255) / 256), 256, 0, st>>>(v, n, npb, ra, out);
  return cudaGetLastError();
}
cudaError_t launch_count_add(int64_t n, unsigned long long* out, cudaStream_t st) {
  k_count_add<<<1, 1, 0, st>>>(n, out);
  return cudaGetLastError();
}

// max of non-negative doubles: their IEEE bit patterns order like unsigned integers
__global__ void k_max_f64(const double* __restrict__ v, int64_t n, unsigned long long* out) {
  unsigned long long m = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    m = max(m, (unsigned long long)__double_as_longlong(v[i]));
  for (int o = 16; o > 0; o >>= 1) m = max(m, __shfl_xor_sync(MV_FULL, m, o));
  if ((threadIdx.x & 31) == 0) atomicMax(out, m);
}

cudaError_t launch_max_f64(const double* v, int64_t n, unsigned long long* out, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  int grid = (int)min64(kNumSMs * 4, (n + 255) / 256);
  k_max_f64<<<grid, 256, 0, st>>>(v, n, out);
  return cudaGetLastError();
}

__global__ void k_check_ids(const int64_t* __restrict__ ids, int64_t n, int* flag) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    if (ids[i] == -1) *flag = 1;
}

cudaError_t launch_check_ids(const int64_t* ids, int64_t n, int* flag, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  int grid = (int)min64(kNumSMs * 8, (n + 255) / 256);
  k_check_ids<<<grid, 256, 0, st>>>(ids, n, flag);
  return cudaGetLastError();
}

// new list sizes (int64) = old sizes + added sizes
__global__ void k_new_sizes(const int32_t* __restrict__ add, int nlist, const int64_t* __restrict__ old_off,
                            int64_t* out) {
  const int l = blockIdx.x * blockDim.x + threadIdx.x;
  if (l < nlist) out[l] = (old_off[l + 1] - old_off[l]) + add[l];
}

cudaError_t launch_new_sizes(const int32_t* add, int nlist, const int64_t* old_off, int64_t* out, cudaStream_t st) {
  k_new_sizes<<<(nlist + 255) / 256, 256, 0, st>>>(add, nlist, old_off, out);
  return cudaGetLastError();
}

__global__ void k_iota_i32(int32_t* out, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = (int32_t)i;
}

cudaError_t launch_iota_i32(int32_t* out, int64_t n, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  int grid = (int)min64(kNumSMs * 8, (n + 255) / 256);
  k_iota_i32<<<grid, 256, 0, st>>>(out, n);
  return cudaGetLastError();
}

// any sorted_ids[t] != t?  (ids exactly 0..n-1: the selects map a rank to its id without a gather)
__global__ void k_check_identity(const int64_t* __restrict__ sorted_ids, int64_t n, int* flag) {
  bool bad = false;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    bad |= sorted_ids[i] != i;
  if (__syncthreads_or(bad) && threadIdx.x == 0) atomicOr(flag, 1);
}

cudaError_t launch_check_identity(const int64_t* sorted_ids, int64_t n, int* flag, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  const int grid = (int)min64(kNumSMs * 8, (n + 255) / 256);
  k_check_identity<<<grid, 256, 0, st>>>(sorted_ids, n, flag);
  return cudaGetLastError();
}

}  // namespace mv
