// umma_bench.cu -- measure tcgen05.mma throughput (cycles per instruction) for the shapes the
// scan/coarse kernels issue: kind::tf32 and kind::i8, M = 128, various N, operands in smem
// (SW128 tf32 / SW32 i8), back-to-back issue by one thread, completion via tcgen05.commit.
#include <cstdio>
#include "sm100.cuh"
using namespace mv::sm100;

template <bool I8>
__global__ void k_bench(int N, int iters, long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint64_t bar;
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x >> 5;
  const int atom = I8 ? 32 : 128;
  for (int i = threadIdx.x; i < (128 + 256) * 128 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = 0x3f800000u;
  fence_proxy_async();
  if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
  if (warp == 0) { tmem_alloc(&tslot, 512); tmem_relinquish(); }
  tc_fence_before(); __syncthreads(); tc_fence_after();
  if (threadIdx.x == 0) {
    const uint32_t idesc = I8 ? idesc_u8s8(N) : idesc_tf32(N);
    const uint32_t a = smem_u32(sm), b = smem_u32(sm + 128 * atom);
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const int ks = i & 3;
      if (I8) mma_i8(tslot, kmajor_desc(a + ks * 32 % atom, atom), kmajor_desc(b + ks * 32 % atom, atom), idesc, 1);
      else mma_tf32(tslot, kmajor_desc(a + ks * 32, atom), kmajor_desc(b + ks * 32, atom), idesc, 1);
    }
    long long t1 = clock64();
    mma_commit(&bar);
    mbar_wait(&bar, 0);
    long long t2 = clock64();
    out[0] = t1 - t0; out[1] = t2 - t0;
  }
  tc_fence_before(); __syncthreads();
  if (warp == 0) { tc_fence_after(); tmem_dealloc(tslot, 512); }
}

int main() {
  long long* d; cudaMalloc(&d, 16); long long h[2];
  for (int i8 = 0; i8 < 2; ++i8)
    for (int N : {32, 48, 64, 96, 128, 192, 256}) {
      const int iters = 4096;
      if (i8) { cudaFuncSetAttribute(k_bench<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200000); k_bench<true><<<1, 128, 200000>>>(N, iters, d); }
      else { cudaFuncSetAttribute(k_bench<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200000); k_bench<false><<<1, 128, 200000>>>(N, iters, d); }
      cudaError_t e = cudaDeviceSynchronize();
      cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
      const double macs = 128.0 * N * (i8 ? 32 : 8);
      printf("%s N=%3d: issue %.1f cyc/mma, complete %.1f cyc/mma -> %.0f MAC/cyc (%s)\n", i8 ? "i8  " : "tf32", N,
             (double)h[0] / iters, (double)h[1] / iters, macs * iters / h[1], cudaGetErrorString(e));
    }
  return 0;
}
