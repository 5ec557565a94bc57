// k_pq.cu -- SURVEY §8(f) row f3: IVF_PQ's fine quantizer on the device.
//
// PAPER.md:519-521 (§3.1): "IVF_PQ uses product quantization that splits each vector into
// multiple sub-vectors and applies k-means for each sub-space".  Reading R19: M
// sub-spaces of dsub = d / M dimensions, 256 sub-centroids each (one byte per sub-code), PQ of the
// vectors themselves; the search's step (2) computes the asymmetric distance
// from q to the decoded vector x_hat through a per-query table T[m][j] = badness of q's m-th
// sub-vector against sub-centroid j (L2: squared distance; IP: minus the inner product), summed
// over the M codes of a row.
//
//   k_pq_encode  add path: per row and sub-space the closest sub-centroid in fp64 (ties to the
//                smaller index, as the oracle), the codes stored list-major, ||x_hat||^2, ids
//   k_pq_scan    search: one CTA per query (the table is per query, 256 x M fp32 in shared
//                memory -- the ADC lookup has no reuse across queries, unlike the grouped SQ8 /
//                FLAT scans, so the work is query-major as in Faiss' GPU IVFPQ); the CTA walks the
//                query's probed lists of the phase (seeding phase A: the ra nearest lists' first
//                capA rows, every candidate emitted; phase B: every probed list, keys <= tau_q
//                emitted), a thread per row: M table lookups, the bitset, the key (badness key <<
//                32 | id rank), warp-aggregated appends into the pair's output region.  The keys
//                then go through the same selects as the other index types.
#include <cuda_runtime.h>
#include <stdint.h>

#include "mv_internal.cuh"

namespace mv {

// one warp per row: per sub-space every lane scores 8 of the 256 sub-centroids (fp64), a warp
// argmin (value, index) picks the code; the decoded row's norm in fp64
__global__ void k_pq_encode(const float* __restrict__ xpad, const int64_t* __restrict__ ids,
                            const int32_t* __restrict__ sorted_idx, const int32_t* __restrict__ sorted_list, int64_t n,
                            int dpad, int M, int dsub, const float* __restrict__ cb, const int64_t* __restrict__ new_off,
                            const int64_t* __restrict__ old_off, const int32_t* __restrict__ add_off,
                            uint8_t* __restrict__ payload, double* __restrict__ norms, int64_t* __restrict__ out_ids) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t t = warp; t < n; t += nwarps) {
    const int i = sorted_idx[t];
    const int l = sorted_list[t];
    const int64_t pos = new_off[l] + (old_off[l + 1] - old_off[l]) + (t - add_off[l]);
    const float* src = xpad + (int64_t)i * dpad;
    uint8_t* dst = payload + pos * M;
    double nrm = 0.0;
    for (int m = 0; m < M; ++m) {
      double best = 1e300;
      int bj = 0;
      for (int u = 0; u < 8; ++u) {
        const int j = u * 32 + lane;  // ascending per lane: the first minimum wins ties
        const float* c = cb + ((int64_t)m * 256 + j) * dsub;
        double dd = 0.0;
        for (int e = 0; e < dsub; ++e) {
          const double df = (double)src[m * dsub + e] - (double)c[e];
          dd = fma(df, df, dd);
        }
        if (dd < best) {
          best = dd;
          bj = j;
        }
      }
      for (int o = 16; o > 0; o >>= 1) {
        const double ob = __shfl_xor_sync(MV_FULL, best, o);
        const int oj = __shfl_xor_sync(MV_FULL, bj, o);
        if (ob < best || (ob == best && oj < bj)) {
          best = ob;
          bj = oj;
        }
      }
      if (lane == 0) dst[m] = (uint8_t)bj;
      const float* c = cb + ((int64_t)m * 256 + bj) * dsub;
      for (int e = lane; e < dsub; e += 32) nrm = fma((double)c[e], (double)c[e], nrm);
    }
    for (int o = 16; o > 0; o >>= 1) nrm += __shfl_xor_sync(MV_FULL, nrm, o);
    if (lane == 0) {
      norms[pos] = nrm;
      out_ids[pos] = ids[i];
    }
  }
}

cudaError_t launch_pq_encode(const float* xpad, const int64_t* ids, const int32_t* sorted_idx,
                             const int32_t* sorted_list, int64_t n, int dpad, int M, int dsub, const float* cb,
                             const int64_t* new_off, const int64_t* old_off, const int32_t* add_off, uint8_t* payload,
                             double* norms, int64_t* out_ids, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  const int grid = (int)min64(kNumSMs * 16, (n * 32 + 255) / 256);
  k_pq_encode<<<grid, 256, 0, st>>>(xpad, ids, sorted_idx, sorted_list, n, dpad, M, dsub, cb, new_off, old_off,
                                    add_off, payload, norms, out_ids);
  return cudaGetLastError();
}

// fp32 -> order-preserving u32 key (as f2key)
__device__ __forceinline__ uint32_t pq_f2key(float f) {
  const uint32_t b = __float_as_uint(__fadd_rn(f, 0.0f));
  return b ^ ((uint32_t)((int32_t)b >> 31) | 0x80000000u);
}

constexpr int kPqThreads = 256;

__global__ void __launch_bounds__(kPqThreads) k_pq_scan(const PqScanParams p) {
  extern __shared__ __align__(16) uint8_t smem[];
  float* T = reinterpret_cast<float*>(smem);           // [M][256]
  float* qs = T + p.M * 256;                           // dpad
  int* s_cnt = reinterpret_cast<int*>(qs + p.dpad);    // 1
  const int64_t q = blockIdx.x;
  const int tid = threadIdx.x, lane = tid & 31;
  const int M = p.M, dsub = p.dsub;
  for (int j = tid; j < p.dpad; j += kPqThreads) qs[j] = p.qpad[q * p.dpad + j];
  __syncthreads();
  // the query's table, fp64 per entry, rounded once
  for (int e = tid; e < M * 256; e += kPqThreads) {
    const int m = e >> 8;
    const float* c = p.codebooks + (int64_t)e * dsub;
    double acc = 0.0;
    if (p.metric == MV_L2) {
      for (int t = 0; t < dsub; ++t) {
        const double df = (double)qs[m * dsub + t] - (double)c[t];
        acc = fma(df, df, acc);
      }
    } else {
      for (int t = 0; t < dsub; ++t) acc = fma((double)qs[m * dsub + t], (double)c[t], acc);
      acc = -acc;
    }
    T[e] = (float)acc;
  }
  const bool phaseB = p.phase != 0;
  const int nr = phaseB ? p.npb : p.ra[q];
  const uint64_t tau = phaseB ? p.tau[q] : MV_KEY_PAD;
  const int64_t npairs = p.nq * (int64_t)p.npb;
  const int words = M >> 2;  // M is a multiple of 4: the codes are read as 32-bit words
  for (int r = 0; r < nr; ++r) {
    const int64_t pr = q * p.npb + r;
    const int64_t pair = phaseB ? pr : npairs + pr;
    const int l = p.probes[pr];
    const int64_t l0 = p.list_off[l];
    const int64_t len = min64(p.list_off[l + 1] - l0, (int64_t)p.rowcap);
    uint64_t* out = p.part + p.poff[pair];
    if (tid == 0) *s_cnt = 0;
    __syncthreads();
    for (int64_t b0 = 0; b0 < len; b0 += kPqThreads) {
      const int64_t i = b0 + tid;
      bool pass = false;
      uint64_t key = 0;
      if (i < len) {
        const int64_t row = l0 + i;
        float acc = 0.0f;
        if ((M & 15) == 0) {  // 16 sub-codes per 16-byte load
          const uint4* cq = reinterpret_cast<const uint4*>(p.codes + row * M);
          for (int w4 = 0; w4 < (M >> 4); ++w4) {
            const uint4 v4 = __ldg(cq + w4);
            const uint32_t vv[4] = {v4.x, v4.y, v4.z, v4.w};
#pragma unroll
            for (int w = 0; w < 4; ++w)
#pragma unroll
              for (int u = 0; u < 4; ++u)
                acc = __fadd_rn(acc, T[((w4 * 4 + w) * 4 + u) * 256 + ((vv[w] >> (8 * u)) & 0xff)]);
          }
        } else {
          const uint32_t* cw = reinterpret_cast<const uint32_t*>(p.codes + row * M);
          for (int w = 0; w < words; ++w) {
            const uint32_t v = __ldg(cw + w);
#pragma unroll
            for (int u = 0; u < 4; ++u) acc = __fadd_rn(acc, T[(w * 4 + u) * 256 + ((v >> (8 * u)) & 0xff)]);
          }
        }
        bool valid = true;
        if (p.bitset) valid = !bit_excluded(p.bitset, p.nbits, p.ids[row]);
        key = ((uint64_t)pq_f2key(acc) << 32) | p.rank[row];
        pass = valid && key <= tau;
      }
      const uint32_t bal = __ballot_sync(MV_FULL, pass);
      int base = 0;
      if (lane == 0 && bal) base = atomicAdd(s_cnt, __popc(bal));
      base = __shfl_sync(MV_FULL, base, 0);
      if (pass) out[base + __popc(bal & ((1u << lane) - 1))] = key;
    }
    __syncthreads();
    if (tid == 0) p.pcnt[pair] = *s_cnt;
  }
}

cudaError_t launch_pq_scan(const PqScanParams& p, cudaStream_t st) {
  if (p.nq == 0) return cudaSuccess;
  const size_t smem = (size_t)p.M * 256 * 4 + (size_t)p.dpad * 4 + 16;
  cudaError_t e = cudaFuncSetAttribute(k_pq_scan, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k_pq_scan<<<(unsigned)p.nq, kPqThreads, smem, st>>>(p);
  return cudaGetLastError();
}

}  // namespace mv
