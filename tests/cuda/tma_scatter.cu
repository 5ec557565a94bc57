// tma_scatter.cu -- is the list scan's HBM rate limited by WHERE its tiles lie?  148 CTAs stream
// 128-row tiles by TMA (one producer thread, a ring of stages, a consumer thread releasing them)
// from a buffer of G GiB, in sequential or hashed (random) tile order:
//   sq8-like : rows of 128 B, one 16 KB box per tile, 12 stages
//   flat-like: rows of 512 B, four {32 fp32, 128 rows} SW128 boxes per tile, 6 stages
// Usage: tma_scatter [GiB ...]
#include <cstdio>
#include <cstdlib>
#include <algorithm>
#include "sm100.cuh"
#include "tmap.h"
using namespace mv::sm100;

struct Args { int64_t nload, nbuf; int boxes, stage_bytes, nstage, random; };  // nload tile loads over nbuf tiles

__device__ __forceinline__ uint64_t mix(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__global__ void __launch_bounds__(64, 1) k_stream(const __grid_constant__ CUtensorMap m, Args a) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint64_t* full = reinterpret_cast<uint64_t*>(sm + a.nstage * a.stage_bytes);
  uint64_t* empty = full + a.nstage;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) { for (int s = 0; s < a.nstage; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); } fence_mbar_init(); }
  __syncthreads();
  if (warp == 0 && lane == 0) {
    uint32_t it = 0;
    for (int64_t i = blockIdx.x; i < a.nload; i += gridDim.x) {
      const int64_t t = a.random ? (int64_t)(mix((uint64_t)i) % (uint64_t)a.nbuf) : i % a.nbuf;
      for (int c = 0; c < a.boxes; ++c, ++it) {
        const uint32_t s = it % a.nstage, r = it / a.nstage;
        mbar_wait(&empty[s], (r & 1) ^ 1);
        mbar_expect_tx(&full[s], a.stage_bytes);
        tma_load_2d(sm + s * a.stage_bytes, &m, &full[s], c * 32, (int)(t * 128));
      }
    }
  } else if (warp == 1 && lane == 0) {
    uint32_t it = 0;
    for (int64_t i = blockIdx.x; i < a.nload; i += gridDim.x)
      for (int c = 0; c < a.boxes; ++c, ++it) {
        const uint32_t s = it % a.nstage;
        mbar_wait(&full[s], (it / a.nstage) & 1);
        mbar_arrive(&empty[s]);
      }
  }
  __syncthreads();
}

int main(int argc, char** argv) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int ai = 1; ai < argc; ++ai) {
    const int64_t gib = atoll(argv[ai]);
    const int64_t bytes = gib << 30;
    uint8_t* x;
    if (cudaMalloc(&x, bytes) != cudaSuccess) { printf("%lld GiB: alloc failed\n", (long long)gib); return 1; }
    cudaMemset(x, 0, bytes);
    for (int flat = 0; flat < 2; ++flat) {
      const int rowb = flat ? 512 : 128, ncol = rowb / 4;
      const int64_t rows = bytes / rowb;
      CUtensorMap m;
      mv::make_tmap_2d(&m, x, flat ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_UINT8,
                       flat ? ncol : rowb, rows, rowb, flat ? 32 : 128, 128, CU_TENSOR_MAP_SWIZZLE_128B);
      for (int nst : {flat ? 6 : 12, flat ? 12 : 6}) {
        for (int rnd = 0; rnd < 2; ++rnd) {
          const int64_t nbuf = rows / 128;
          const int64_t tiles = std::min<int64_t>(nbuf, (8ll << 30) / (128 * rowb));  // 8 GiB per run
          Args d{tiles, nbuf, flat ? 4 : 1, 16384, nst, rnd};
          const int smem = 16384 * nst + 1024;
          cudaFuncSetAttribute(k_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
          float ms = 0;
          for (int rep = 0; rep < 2; ++rep) {
            cudaEventRecord(e0);
            k_stream<<<148, 64, smem>>>(m, d);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            cudaEventElapsedTime(&ms, e0, e1);
          }
          printf("%3lld GiB %-9s %2d stages %-10s %7.1f GB/s (%s)\n", (long long)gib, flat ? "flat-like" : "sq8-like", nst,
                 rnd ? "random" : "sequential", tiles * 128.0 * rowb / (ms * 1e6), cudaGetErrorString(cudaGetLastError()));
        }
      }
    }
    cudaFree(x);
  }
  return 0;
}
