// select_bench.cu -- cycles per (query, tile) of the epilogue selection (warp_filter_group, G=4,
// k=10) on synthetic 128-candidate tiles held in shared memory like the scan's transposed tile.
// mode 0: keys random every tile (natural regime: survivors ~ k/t per tile after warm-up)
// mode 1: keys always above the threshold after the first tile (filter only)
#include <cstdio>
#include "mv_internal.cuh"
using namespace mv;

__device__ uint32_t hsh(uint32_t x) { x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16; return x; }

template <int G>
__global__ void __launch_bounds__(256, 1) k_sel(int ntiles, int nq, int k, int mode, long long* out) {
  __shared__ uint32_t Dt[48 * 129];
  __shared__ uint64_t lists[48 * 10], cbuf[48 * 32], scratch[8 * 32];
  __shared__ int cnb[64];
  __shared__ uint32_t cbnd[64];
  __shared__ uint32_t srank[128];
  __shared__ int ctr;
  const int tid = threadIdx.x, lane = tid & 31, ew = tid >> 5;
  for (int i = tid; i < 48 * 10; i += 256) lists[i] = MV_KEY_PAD;
  for (int i = tid; i < 64; i += 256) { cnb[i] = 0; cbnd[i] = 0xffffffffu; }
  for (int i = tid; i < 128; i += 256) srank[i] = i;
  __syncthreads();
  long long tsel = 0;
  for (int t = 0; t < ntiles; ++t) {
    for (int i = tid; i < nq * 128; i += 256) {
      const int q = i / 128, v = i % 128;
      uint32_t key = 0x40000000u + (hsh(t * 1000003u + q * 131u + v) >> 4);
      if (mode == 1 && t > 0) key = 0x7fffffffu;
      Dt[q * 129 + v] = key;
    }
    if (tid == 0) ctr = 0;
    __syncthreads();
    const long long t0 = clock64();
    for (;;) {
      int i0 = 0;
      if (lane == 0) i0 = atomicAdd(&ctr, G);
      i0 = __shfl_sync(MV_FULL, i0, 0);
      if (i0 >= nq) break;
      const int nvalid = min(G, nq - i0);
      warp_filter_group<G>(
          nvalid, k, [&](int g, int m) { return Dt[(i0 + g) * 129 + m * 32 + lane]; },
          [&](int g, uint64_t*& L, uint64_t*& B, int*& nb, uint32_t*& bnd, uint64_t& li) {
            const int i = i0 + g;
            L = lists + i * k; B = cbuf + i * 32; nb = cnb + i; bnd = cbnd + i; li = MV_KEY_PAD;
          },
          [&](int, int v) { return srank[v] + (uint32_t)t * 128u; }, [](int, uint32_t) {}, scratch);
    }
    __syncthreads();
    tsel += clock64() - t0;
  }
  if (tid == 0) out[blockIdx.x] = tsel;
}

int main() {
  long long* d; cudaMalloc(&d, 148 * 8); long long h[148];
  for (int mode = 0; mode < 2; ++mode)
    for (int nq : {8, 48}) {
      const int ntiles = 200;
      k_sel<4><<<148, 256>>>(ntiles, nq, 10, mode, d);
      cudaError_t e = cudaDeviceSynchronize();
      cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
      double avg = 0; for (int b = 0; b < 148; ++b) avg += h[b]; avg /= 148;
      printf("mode %d nq %2d: %.0f cycles per tile (%.0f per query-tile)  %s\n", mode, nq, avg / ntiles, avg / ntiles / nq * 8, cudaGetErrorString(e));
    }
  return 0;
}
