// umma_selftest.cu -- GPU self-test of the hand-written sm_100a building blocks (test
// infrastructure): TMA (SW128 / SW32) + tcgen05.mma kind::tf32 and kind::i8 (u8 x s8) + TMEM
// loads, on integer data whose products are exact, against a CPU int64 reference.
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "sm100.cuh"
#include "tmap.h"

using namespace mv::sm100;

template <bool I8>
__global__ void k_gemm(const __grid_constant__ CUtensorMap mapA, const uint8_t* Bg, int N, int K, int atom, int* Dout) {
  extern __shared__ __align__(1024) uint8_t sm[];
  const int es = I8 ? 1 : 4;
  const int chunks = K * es / atom;
  uint8_t* As = sm;
  uint8_t* Bs = sm + chunks * 128 * atom;
  __shared__ uint64_t bar[2];
  __shared__ uint32_t tslot;
  const int tid = threadIdx.x, warp = tid >> 5;
  if (tid == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    fence_mbar_init();
  }
  if (warp == 0) {
    tmem_alloc(&tslot, 256);
    tmem_relinquish();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tslot;
  if (tid == 0) {
    mbar_expect_tx(&bar[0], chunks * 128 * atom);
    for (int c = 0; c < chunks; ++c) tma_load_2d(As + c * 128 * atom, &mapA, &bar[0], c * atom / es, 0);
  }
  const int pieces = atom / 16;
  for (int i = tid; i < N * chunks * pieces; i += blockDim.x) {
    const int n = i / (chunks * pieces), r = i % (chunks * pieces), c = r / pieces, p = r % pieces;
    const uint4 v = *reinterpret_cast<const uint4*>(Bg + (size_t)n * K * es + c * atom + p * 16);
    *reinterpret_cast<uint4*>(Bs + c * N * atom + swz_off(n, p, atom)) = v;
  }
  fence_proxy_async();
  __syncthreads();
  if (tid == 0) {
    mbar_wait(&bar[0], 0);
    tc_fence_after();
    const uint32_t idesc = I8 ? idesc_u8s8(N) : idesc_tf32(N);
    for (int c = 0; c < chunks; ++c)
      for (int s = 0; s < atom / 32; ++s) {
        const uint64_t a = kmajor_desc(smem_u32(As + c * 128 * atom) + s * 32, atom);
        const uint64_t b = kmajor_desc(smem_u32(Bs + c * N * atom) + s * 32, atom);
        if (I8) mma_i8(tmem, a, b, idesc, (c | s) != 0);
        else mma_tf32(tmem, a, b, idesc, (c | s) != 0);
      }
    mma_commit(&bar[1]);
  }
  __syncwarp();
  mbar_wait(&bar[1], 0);
  tc_fence_after();
  const int row = (warp & 3) * 32 + (tid & 31);
  for (int c0 = 0; c0 < N; c0 += 16) {
    uint32_t r[16];
    tmem_ld16(tmem + ((uint32_t)((warp & 3) * 32) << 16) + c0, r);
    tmem_wait_ld();
    for (int j = 0; j < 16; ++j) {
      int v = I8 ? (int)r[j] : (int)__uint_as_float(r[j]);
      Dout[row * N + c0 + j] = v;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tmem, 256);
}

template <bool I8>
static int run(int N, int K, int atom) {
  const int es = I8 ? 1 : 4;
  std::vector<uint8_t> A(128 * K * es), B(N * K * es);
  std::vector<long long> ref(128 * N, 0);
  srand(1234 + N + K);
  std::vector<int> av(128 * K), bv(N * K);
  for (int i = 0; i < 128 * K; ++i) av[i] = I8 ? rand() % 256 : rand() % 256;
  for (int i = 0; i < N * K; ++i) bv[i] = I8 ? (rand() % 255) - 127 : rand() % 256;
  for (int i = 0; i < 128 * K; ++i) {
    if (I8) A[i] = (uint8_t)av[i];
    else { float f = (float)av[i]; memcpy(&A[i * 4], &f, 4); }
  }
  for (int i = 0; i < N * K; ++i) {
    if (I8) B[i] = (uint8_t)(int8_t)bv[i];
    else { float f = (float)bv[i]; memcpy(&B[i * 4], &f, 4); }
  }
  for (int m = 0; m < 128; ++m)
    for (int n = 0; n < N; ++n) {
      long long acc = 0;
      for (int k = 0; k < K; ++k) acc += (long long)av[m * K + k] * bv[n * K + k];
      ref[m * N + n] = acc;
    }
  uint8_t *dA, *dB;
  int* dD;
  cudaMalloc(&dA, A.size());
  cudaMalloc(&dB, B.size());
  cudaMalloc(&dD, 128 * N * 4);
  cudaMemcpy(dA, A.data(), A.size(), cudaMemcpyHostToDevice);
  cudaMemcpy(dB, B.data(), B.size(), cudaMemcpyHostToDevice);
  CUtensorMap map;
  CUtensorMapSwizzle sw = atom == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : (atom == 64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B);
  if (!mv::make_tmap_2d(&map, dA, I8 ? CU_TENSOR_MAP_DATA_TYPE_UINT8 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, K, 128, K * es,
                        atom / es, 128, sw)) {
    printf("tmap failed\n");
    return 1;
  }
  const int smem = (K * es / atom) * (128 + N) * atom + 1024;
  cudaFuncSetAttribute(k_gemm<I8>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  k_gemm<I8><<<1, 128, smem>>>(map, dB, N, K, atom, dD);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) {
    printf("%s N=%d K=%d atom=%d: CUDA error %s\n", I8 ? "i8" : "tf32", N, K, atom, cudaGetErrorString(e));
    return 1;
  }
  std::vector<int> D(128 * N);
  cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
  int bad = 0;
  for (int i = 0; i < 128 * N; ++i)
    if (D[i] != ref[i]) {
      if (bad < 5) printf("  mismatch m=%d n=%d got %d want %lld\n", i / N, i % N, D[i], ref[i]);
      ++bad;
    }
  printf("%s N=%d K=%d atom=%d: %s (%d mismatches)\n", I8 ? "i8(u8xs8)" : "tf32", N, K, atom, bad ? "FAIL" : "PASS", bad);
  cudaFree(dA); cudaFree(dB); cudaFree(dD);
  return bad != 0;
}

int main() {
  int fails = 0;
  fails += run<false>(64, 128, 128);
  fails += run<false>(16, 128, 128);
  fails += run<false>(256, 32, 128);
  fails += run<false>(48, 128, 128);
  fails += run<true>(64, 96, 32);
  fails += run<true>(16, 128, 32);
  fails += run<true>(80, 96, 32);
  fails += run<true>(64, 128, 128);
  printf(fails ? "SELFTEST FAIL\n" : "SELFTEST PASS\n");
  return fails;
}
