// k_coarse.cu -- §8 row a1 (query / centroid staging: zero-padded rows and norms) and the
// degenerate step (1) of PAPER.md:523-529 (§3.1) when nprobe >= nlist: every bucket is probed,
// listed in id order (no ranking is needed).  The ranked coarse step (a2 + a3) and the add path's
// assignment run on the tensor cores (k_coarse_tc.cu).
#include "mv_internal.cuh"

namespace mv {

// one warp per row: zero-padded copy and squared norm (fp32, fmaf chain per lane + xor tree)
__global__ void k_row_prep(const float* __restrict__ x, int64_t n, int d, int dpad, float* __restrict__ out,
                           float* __restrict__ norm) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = warp; r < n; r += nwarps) {
    float acc = 0.0f;
    for (int j = lane; j < dpad; j += 32) {
      const float v = j < d ? x[r * d + j] : 0.0f;
      out[r * dpad + j] = v;
      acc = fmaf(v, v, acc);
    }
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(MV_FULL, acc, o);
    if (lane == 0) norm[r] = acc;
  }
}

cudaError_t launch_query_prep(const float* q, int64_t nq, int d, int dpad, float* qpad, float* qnorm, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  int grid = (int)min64(kNumSMs * 16, (nq * 32 + 255) / 256);
  k_row_prep<<<grid, 256, 0, st>>>(q, nq, d, dpad, qpad, qnorm);
  return cudaGetLastError();
}

cudaError_t launch_centroid_prep(const float* c, int nlist, int d, int dpad, float* cpad, float* cnorm, cudaStream_t st) {
  return launch_query_prep(c, nlist, d, dpad, cpad, cnorm, st);
}

__global__ void k_all_lists(int64_t nq, int nlist, int32_t* probes) {
  const int64_t total = nq * nlist;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x)
    probes[t] = (int32_t)(t % nlist);
}

cudaError_t launch_all_lists(int64_t nq, int nlist, int32_t* probes, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  int grid = (int)min64(kNumSMs * 8, (nq * nlist + 255) / 256);
  k_all_lists<<<grid, 256, 0, st>>>(nq, nlist, probes);
  return cudaGetLastError();
}

}  // namespace mv
