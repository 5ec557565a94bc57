// tma_bench.cu -- HBM streaming rate of the TMA load shapes the list scan can use (one producer
// thread per CTA, ring of stages, one consumer warp releasing stages), 148 CTAs, 1 GiB matrix.
//   mode 0: 2-D tensor box {32 fp32, 128 rows} SW128 (the current scan: 4 column-chunk boxes / tile)
//   mode 1: 2-D tensor box {32 fp32, 256 rows} SW128
//   mode 2: cp.async.bulk of contiguous 16 KB pieces (a tile-blocked payload layout)
//   mode 3: 3-D tensor box {32, 128 rows, 4 chunks} SW128 = one 64 KB tile per instruction
#include <cstdio>
#include <vector>
#include "sm100.cuh"
#include "tmap.h"
using namespace mv::sm100;

struct Args { const float* base; int64_t rows; int mode, stage_bytes, nstage; };

__global__ void __launch_bounds__(64, 1) k_stream(const __grid_constant__ CUtensorMap m2, const __grid_constant__ CUtensorMap m3, Args a) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint64_t* full = reinterpret_cast<uint64_t*>(sm + a.nstage * a.stage_bytes);
  uint64_t* empty = full + a.nstage;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) { for (int s = 0; s < a.nstage; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); } fence_mbar_init(); }
  __syncthreads();
  const int64_t tiles = a.rows / 128;            // 128-row tiles of 512 B rows = 64 KB
  const int per_tile = 65536 / a.stage_bytes;    // stages per tile
  if (warp == 0 && lane == 0) {
    uint32_t it = 0;
    for (int64_t t = blockIdx.x; t < tiles; t += gridDim.x)
      for (int c = 0; c < per_tile; ++c, ++it) {
        const uint32_t s = it % a.nstage, r = it / a.nstage;
        mbar_wait(&empty[s], (r & 1) ^ 1);
        mbar_expect_tx(&full[s], a.stage_bytes);
        uint8_t* dst = sm + s * a.stage_bytes;
        if (a.mode == 0) tma_load_2d(dst, &m2, &full[s], c * 32, (int)(t * 128));
        else if (a.mode == 1) tma_load_2d(dst, &m2, &full[s], (c & 3) * 32, (int)(t * 128 + (c >> 2) * 0));
        else if (a.mode == 2) bulk_g2s(dst, reinterpret_cast<const uint8_t*>(a.base) + t * 65536 + c * a.stage_bytes, a.stage_bytes, &full[s]);
        else asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];"
                          :: "r"(smem_u32(dst)), "l"(&m3), "r"(smem_u32(&full[s])), "r"(0), "r"((int)(t * 128)), "r"(0) : "memory");
      }
  } else if (warp == 1 && lane == 0) {
    uint32_t it = 0;
    for (int64_t t = blockIdx.x; t < tiles; t += gridDim.x)
      for (int c = 0; c < per_tile; ++c, ++it) {
        const uint32_t s = it % a.nstage;
        mbar_wait(&full[s], (it / a.nstage) & 1);
        mbar_arrive(&empty[s]);
      }
  }
  __syncthreads();
}

int main() {
  const int64_t rows = (1ll << 30) / 512;  // 1 GiB of 128-float rows
  float* x; cudaMalloc(&x, rows * 512); cudaMemset(x, 0, rows * 512);
  CUtensorMap m2a, m2b, m3;
  mv::make_tmap_2d(&m2a, x, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 128, rows, 512, 32, 128, CU_TENSOR_MAP_SWIZZLE_128B);
  mv::make_tmap_2d(&m2b, x, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 128, rows, 512, 32, 256, CU_TENSOR_MAP_SWIZZLE_128B);
  {  // 3-D view: {32 elems (128 B), rows (pitch 512 B), 4 chunks (pitch 128 B)}
    auto enc = mv::tmap_encoder();
    cuuint64_t dims[3] = {32, (cuuint64_t)rows, 4};
    cuuint64_t strides[2] = {512, 128};
    cuuint32_t box[3] = {32, 128, 4}, es[3] = {1, 1, 1};
    CUresult r = enc(&m3, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, x, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("3d map encode: %d\n", (int)r);
  }
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  struct Cfg { int mode, stage, nstage; const char* name; } cfgs[] = {
    {0, 16384, 6, "2D box 32x128 (16KB) x6"}, {0, 16384, 12, "2D box 32x128 (16KB) x12"},
    {1, 32768, 3, "2D box 32x256 (32KB) x3"}, {1, 32768, 6, "2D box 32x256 (32KB) x6"},
    {2, 16384, 6, "bulk 16KB contiguous x6"}, {2, 16384, 12, "bulk 16KB contiguous x12"}, {2, 65536, 3, "bulk 64KB contiguous x3"},
    {3, 65536, 2, "3D box 32x128x4 (64KB) x2"}, {3, 65536, 3, "3D box 32x128x4 (64KB) x3"}};
  for (auto& c : cfgs) {
    Args a{x, rows, c.mode, c.stage, c.nstage};
    const int smem = c.stage * c.nstage + 1024;
    cudaFuncSetAttribute(k_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    const CUtensorMap& m = c.mode == 1 ? m2b : m2a;
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(e0);
      k_stream<<<148, 64, smem>>>(m, m3, a);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
    }
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    printf("%-30s %7.1f GB/s  (%s)\n", c.name, (rows * 512.0) / (ms * 1e6), cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
