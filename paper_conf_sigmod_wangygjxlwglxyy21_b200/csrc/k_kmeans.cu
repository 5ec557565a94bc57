// k_kmeans.cu -- SURVEY §8(f) row f1 (the GPU build path): Lloyd k-means training of the coarse
// quantizer on the device.  PAPER.md:503-514 (§3.1): IVF "uses K-means to cluster" the vectors
// into nlist buckets whose centroids are the coarse codebook.  One Lloyd iteration = assign every
// training row to its closest centroid (mv_api.cu: the tensor-core coarse step with nprobe = 1, the
// assignment mv_index_add makes), then replace each centroid by the mean of its rows (fp64 sums,
// rounded to fp32 once); a centroid without rows keeps its position (reading R18);
// `spherical` re-normalises the centroids (unit-norm, inner-product data).
#include <cuda_runtime.h>
#include <stdint.h>

#include "mv_internal.cuh"

namespace mv {

// sums[l][j] += x[r][j], cnt[l] += 1 for l = lists[r]: one warp per row (coalesced row reads,
// fp64 atomics into the centroid's row)
__global__ void k_kmeans_accum(const float* __restrict__ x, int64_t n, int d, const int32_t* __restrict__ lists,
                               double* __restrict__ sums, unsigned long long* __restrict__ cnt) {
  const int lane = threadIdx.x & 31;
  const int64_t w0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = w0; r < n; r += nw) {
    const int l = lists[r];
    const float* xr = x + r * d;
    double* sr = sums + (int64_t)l * d;
    for (int j = lane; j < d; j += 32) atomicAdd(sr + j, (double)xr[j]);
    if (lane == 0) atomicAdd(cnt + l, 1ull);
  }
}

// c[l] = sums[l] / cnt[l] (fp64, rounded to fp32; optionally normalised in fp64 first); empty
// centroids keep c[l].  One warp per centroid.
__global__ void k_kmeans_update(const double* __restrict__ sums, const unsigned long long* __restrict__ cnt, int nlist,
                                int d, int spherical, float* __restrict__ c) {
  const int lane = threadIdx.x & 31;
  const int64_t w0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t l = w0; l < nlist; l += nw) {
    const unsigned long long m = cnt[l];
    if (m == 0) continue;
    const double* s = sums + l * d;
    double nn = 0.0;
    if (spherical) {
      for (int j = lane; j < d; j += 32) {
        const double v = s[j] / (double)m;
        nn = fma(v, v, nn);
      }
      for (int o = 16; o > 0; o >>= 1) nn += __shfl_xor_sync(MV_FULL, nn, o);
    }
    const double inv = spherical && nn > 0.0 ? 1.0 / sqrt(nn) : 1.0;
    for (int j = lane; j < d; j += 32) c[l * d + j] = (float)(s[j] / (double)m * inv);
  }
}

cudaError_t launch_kmeans_accum(const float* x, int64_t n, int d, const int32_t* lists, double* sums,
                                unsigned long long* cnt, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  const int grid = (int)min64(kNumSMs * 16, (n * 32 + 255) / 256);
  k_kmeans_accum<<<grid, 256, 0, st>>>(x, n, d, lists, sums, cnt);
  return cudaGetLastError();
}

cudaError_t launch_kmeans_update(const double* sums, const unsigned long long* cnt, int nlist, int d, int spherical,
                                 float* c, cudaStream_t st) {
  const int grid = (int)min64(kNumSMs * 16, ((int64_t)nlist * 32 + 255) / 256);
  k_kmeans_update<<<grid, 256, 0, st>>>(sums, cnt, nlist, d, spherical, c);
  return cudaGetLastError();
}

}  // namespace mv
