// k_coarse.cu -- §8 rows a1 (query staging), a2 (Q x C^T coarse contraction) and a3 (fused
// per-query top-nprobe).  PAPER.md:523-529 (§3.1): "(1) Find the closest nprobe buckets based on
// the distance between q and the centroid of each bucket".  Score per (q, c):
//   L2: ||c||^2 - 2 q.c  (||q||^2 does not change the ranking),   IP: -(q.c)
// ordered by (score, centroid id).  Also serves the add path's assignment (nprobe = 1,
// I(v) = the closest centroid).
//
// v0 bring-up kernel: SIMT fp32 (CUDA cores).  The tcgen05 contraction replaces it.
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

template <int QB>
__global__ void __launch_bounds__(256) k_coarse_simt(const float* __restrict__ qpad, int64_t nq, int dpad,
                                                     const float* __restrict__ cpad, const float* __restrict__ cnorm,
                                                     int nlist, int metric, int nprobe, int32_t* __restrict__ probes) {
  constexpr int CT = 64;           // centroids per tile
  constexpr int QPT = QB / 16;     // queries per thread
  extern __shared__ __align__(16) uint8_t smem[];
  const int ld = dpad + 1;
  float* Qs = reinterpret_cast<float*>(smem);
  float* Cs = Qs + QB * ld;
  uint64_t* S = reinterpret_cast<uint64_t*>(Cs + CT * ld + ((QB * ld + CT * ld) & 1));
  uint64_t* lists = S + QB * CT;

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t q0 = (int64_t)blockIdx.x * QB;
  const int nqb = (int)min64(QB, nq - q0);

  for (int i = tid; i < QB * dpad; i += 256) {
    const int r = i / dpad, j = i - r * dpad;
    Qs[r * ld + j] = r < nqb ? qpad[(q0 + r) * dpad + j] : 0.0f;
  }
  for (int i = tid; i < QB * nprobe; i += 256) lists[i] = MV_KEY_PAD;

  const int tc = tid & 15, tq = tid >> 4;
  for (int c0 = 0; c0 < nlist; c0 += CT) {
    __syncthreads();
    const int nct = min(CT, nlist - c0);
    for (int i = tid; i < CT * dpad; i += 256) {
      const int r = i / dpad, j = i - r * dpad;
      Cs[r * ld + j] = r < nct ? cpad[(int64_t)(c0 + r) * dpad + j] : 0.0f;
    }
    __syncthreads();
    float acc[QPT][4];
#pragma unroll
    for (int a = 0; a < QPT; ++a)
#pragma unroll
      for (int b = 0; b < 4; ++b) acc[a][b] = 0.0f;
    for (int j = 0; j < dpad; ++j) {
      float qv[QPT], cv[4];
#pragma unroll
      for (int a = 0; a < QPT; ++a) qv[a] = Qs[(tq + 16 * a) * ld + j];
#pragma unroll
      for (int b = 0; b < 4; ++b) cv[b] = Cs[(tc + 16 * b) * ld + j];
#pragma unroll
      for (int a = 0; a < QPT; ++a)
#pragma unroll
        for (int b = 0; b < 4; ++b) acc[a][b] = fmaf(qv[a], cv[b], acc[a][b]);
    }
#pragma unroll
    for (int a = 0; a < QPT; ++a)
#pragma unroll
      for (int b = 0; b < 4; ++b) {
        const int cl = tc + 16 * b, c = c0 + cl, qi = tq + 16 * a;
        uint64_t key = MV_KEY_PAD;
        if (cl < nct && qi < nqb) {
          const float s = metric == MV_L2 ? __fsub_rn(cnorm[c], 2.0f * acc[a][b]) : -acc[a][b];
          key = ((uint64_t)f2key(s) << 32) | (uint32_t)c;
        }
        S[qi * CT + cl] = key;
      }
    __syncthreads();
    for (int qi = warp; qi < nqb; qi += 8) {
      warp_list_insert(lists + qi * nprobe, nprobe, S[qi * CT + lane], true);
      warp_list_insert(lists + qi * nprobe, nprobe, S[qi * CT + lane + 32], true);
    }
  }
  __syncthreads();
  for (int i = tid; i < nqb * nprobe; i += 256) {
    const int qi = i / nprobe, j = i - qi * nprobe;
    probes[(q0 + qi) * nprobe + j] = (int32_t)(uint32_t)(lists[qi * nprobe + j] & 0xffffffffu);
  }
}

__global__ void k_all_lists(int64_t nq, int nlist, int32_t* probes) {
  const int64_t total = nq * nlist;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x)
    probes[t] = (int32_t)(t % nlist);
}

template <int QB>
static cudaError_t run_coarse(const float* qpad, int64_t nq, int dpad, const float* cpad, const float* cnorm, int nlist,
                              int metric, int nprobe, int32_t* probes, cudaStream_t st) {
  const int ld = dpad + 1;
  size_t smem = (size_t)(QB + 64) * ld * 4 + 8 + (size_t)QB * 64 * 8 + (size_t)QB * nprobe * 8;
  cudaError_t e = cudaFuncSetAttribute(k_coarse_simt<QB>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  const int64_t grid = (nq + QB - 1) / QB;
  k_coarse_simt<QB><<<(unsigned)grid, 256, smem, st>>>(qpad, nq, dpad, cpad, cnorm, nlist, metric, nprobe, probes);
  return cudaGetLastError();
}

cudaError_t launch_coarse(const float* qpad, int64_t nq, int dpad, const float* cpad, const float* cnorm, int nlist,
                          int metric, int nprobe, int32_t* probes, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  if (nprobe >= nlist) {
    int grid = (int)min64(kNumSMs * 8, (nq * nlist + 255) / 256);
    k_all_lists<<<grid, 256, 0, st>>>(nq, nlist, probes);
    return cudaGetLastError();
  }
  if (nprobe <= 512) return run_coarse<32>(qpad, nq, dpad, cpad, cnorm, nlist, metric, nprobe, probes, st);
  return run_coarse<16>(qpad, nq, dpad, cpad, cnorm, nlist, metric, nprobe, probes, st);
}

}  // namespace mv
