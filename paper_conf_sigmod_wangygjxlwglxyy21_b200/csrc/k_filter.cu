// k_filter.cu -- SURVEY §8(f) row f4: the two workloads the paper runs on top of the vector hot
// path, as device kernels behind the C ABI (mv_attr_bitset, mv_fuse_rows).
//
// * Strategy E (§4.1): partitions by the value range of a frequently searched
//   attribute; a partition whose range the query constraint only partly covers checks the
//   attribute with strategy B's bitmap -- mv_attr_bitset builds that bitmap
//   from the partition's (id, attribute) columns on the device; a covered partition needs none.
// * Vector fusion (§4.2): an entity's mu vectors are stored concatenated and a
//   query entity's vectors are scaled by the aggregation weights and concatenated, so that one
//   inner-product search computes the weighted sum of the per-vector inner products --
//   mv_fuse_rows writes [w_0 v_0 | w_1 v_1 | ...] row by row.
#include <cuda_runtime.h>
#include <stdint.h>

#include "mv_internal.cuh"

namespace mv {

// bit id of the 32-bit-word bitset is set (excluded, reading R6) when attr is outside [lo, hi]
__global__ void k_attr_bitset(const int64_t* __restrict__ ids, const int64_t* __restrict__ attr, int64_t n, int64_t lo,
                              int64_t hi, uint32_t* __restrict__ words, int64_t nbits) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t a = attr[i], id = ids[i];
    if ((a < lo || a > hi) && id >= 0 && id < nbits) atomicOr(words + (id >> 5), 1u << (id & 31));
  }
}

cudaError_t launch_attr_bitset(const int64_t* ids, const int64_t* attr, int64_t n, int64_t lo, int64_t hi,
                               uint8_t* bitset, int64_t nbits, cudaStream_t st) {
  const int64_t nwords = (nbits + 31) / 32;
  cudaError_t e = cudaMemsetAsync(bitset, 0, (size_t)nwords * 4, st);
  if (e != cudaSuccess || n == 0) return e;
  const int grid = (int)min64(kNumSMs * 8, (n + 255) / 256);
  k_attr_bitset<<<grid, 256, 0, st>>>(ids, attr, n, lo, hi, reinterpret_cast<uint32_t*>(bitset), nbits);
  return cudaGetLastError();
}

// out[r][off_i + j] = w_i * part_i[r][j]: one warp per row, the row's parts one after another
__global__ void k_fuse_rows(FuseArgs a, int64_t n, float* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t w0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = w0; r < n; r += nw) {
    float* o = out + r * a.dtot;
    for (int i = 0; i < a.m; ++i) {
      const float* src = a.part[i] + r * a.dim[i];
      const float w = a.w[i];
      for (int j = lane; j < a.dim[i]; j += 32) o[a.off[i] + j] = w * src[j];
    }
  }
}

cudaError_t launch_fuse_rows(const FuseArgs& a, int64_t n, float* out, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  const int grid = (int)min64(kNumSMs * 16, (n * 32 + 255) / 256);
  k_fuse_rows<<<grid, 256, 0, st>>>(a, n, out);
  return cudaGetLastError();
}

}  // namespace mv
