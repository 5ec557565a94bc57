// k_scan.cu -- §8 rows a5 (grouped list scan: FLAT fp32 / SQ8 decoded, L2 / IP, bitset) and a6
// (per-(query, list) partial top-k fused into the scan).
//
// PAPER.md:529-532 (§3.1): "(2) Search within each of the nprobe relevant buckets based on
// different fine quantizers ... IVF_FLAT ... needs to scan the vectors".
// (§4.1, strategy B): the bitmap is checked "whenever a vector is encountered"; only passing
// vectors reach the top-k.  PAPER.md:590-596 (§3.2.1): per-thread heaps, merged at the end --
// here: one sorted list per (query, list) work item, merged by the final select (k_select.cu).
//
// Work item = (list l, a chunk of <= qchunk queries of l's bucket).  A persistent grid pulls
// work items from an atomic counter.  Per 64-vector tile: stage the vectors in shared memory
// (SQ8 codes decoded in-register with the oracle's op order), compute the 64 x nqc distance
// tile, then one warp per query filters the 64 candidates against its current k-th best and
// inserts the survivors.  v0 producer: SIMT fp32; DESIGN.md §5 describes the tcgen05 producer.
#include "mv_internal.cuh"

namespace mv {

constexpr int kVT = 64;      // vectors per tile
constexpr int kQCMax = 64;   // queries per work item (max)

template <int TYPE>
__global__ void __launch_bounds__(256) k_scan_simt(const ScanArgs a) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int dpad = a.dpad, ld = dpad + 1, k = a.k;
  float* Xs = reinterpret_cast<float*>(smem);
  float* Qs = Xs + kVT * ld;
  float* Dt = Qs + kQCMax * ld;                       // [kQCMax][kVT + 1]
  float* lut = Dt + kQCMax * (kVT + 1);               // 256
  uint32_t* rrank = reinterpret_cast<uint32_t*>(lut + 256);
  uint32_t* rvalid = rrank + kVT;
  int32_t* qpair = reinterpret_cast<int32_t*>(rvalid + kVT);
  int32_t* qcnt = qpair + kQCMax;
  int32_t* s_misc = qcnt + kQCMax;                    // [0] = work item
  uint64_t* lists = reinterpret_cast<uint64_t*>(s_misc + 4);  // 16-byte aligned by construction

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (TYPE == MV_IVF_SQ8)
    for (int i = tid; i < 256; i += 256) lut[i] = a.sq8_t[i];
  const int nwork = *a.nwitems;
  const int tv = tid & 15, tq = tid >> 4;

  for (;;) {
    __syncthreads();
    if (tid == 0) s_misc[0] = atomicAdd(a.counter, 1);
    __syncthreads();
    const int w = s_misc[0];
    if (w >= nwork) break;
    const int2 it = a.witems[w];
    const int l = it.x, bstart = it.y;
    const int nqc = min(a.qchunk, a.boff[l + 1] - bstart);
    const int64_t lstart = a.list_off[l];
    const int len = (int)(a.list_off[l + 1] - lstart);
    const bool sel = (k <= kLocalSelectMaxK) && (len > k);

    for (int i = tid; i < nqc; i += 256) {
      qpair[i] = a.bq[bstart + i];
      qcnt[i] = 0;
    }
    __syncthreads();
    for (int i = tid; i < kQCMax * dpad; i += 256) {
      const int r = i / dpad, j = i - r * dpad;
      float v = 0.0f;
      if (r < nqc) v = a.qpad[(int64_t)(qpair[r] / a.npb) * dpad + j];
      Qs[r * ld + j] = v;
    }
    if (sel)
      for (int i = tid; i < nqc * k; i += 256) lists[i] = MV_KEY_PAD;

    for (int t0 = 0; t0 < len; t0 += kVT) {
      __syncthreads();
      const int nv = min(kVT, len - t0);
      const int64_t row0 = lstart + t0;
      if (TYPE == MV_IVF_FLAT) {
        const float* src = reinterpret_cast<const float*>(a.payload) + row0 * dpad;
        for (int i = tid; i < kVT * dpad / 4; i += 256) {
          const int r = (i * 4) / dpad, j = i * 4 - r * dpad;
          float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
          if (r < nv) v = __ldg(reinterpret_cast<const float4*>(src + (int64_t)r * dpad + j));
          float* x = Xs + r * ld + j;
          x[0] = v.x; x[1] = v.y; x[2] = v.z; x[3] = v.w;
        }
      } else {
        const uint8_t* src = reinterpret_cast<const uint8_t*>(a.payload) + row0 * dpad;
        for (int i = tid; i < kVT * dpad / 4; i += 256) {
          const int r = (i * 4) / dpad, j = i * 4 - r * dpad;
          uint32_t c4 = 0;
          if (r < nv) c4 = __ldg(reinterpret_cast<const uint32_t*>(src + (int64_t)r * dpad + j));
          float* x = Xs + r * ld + j;
#pragma unroll
          for (int b = 0; b < 4; ++b) {
            const int c = (c4 >> (8 * b)) & 0xff;
            x[b] = r < nv ? __fadd_rn(__fmul_rn(lut[c], a.vdiff[j + b]), a.vmin[j + b]) : 0.0f;
          }
        }
      }
      for (int r = tid; r < kVT; r += 256) {
        bool ok = r < nv;
        if (ok && a.bitset) ok = !bit_excluded(a.bitset, a.nbits, a.ids[row0 + r]);
        rvalid[r] = ok;
        rrank[r] = ok ? a.rank[row0 + r] : 0u;
      }
      __syncthreads();
      // distance tile: thread (tv, tq) -> vectors tv + 16 i, queries tq + 16 jq
      for (int jq = 0; jq < 4 && 16 * jq < nqc; ++jq) {
        float acc[4] = {0.f, 0.f, 0.f, 0.f};
        const float* qrow = Qs + (tq + 16 * jq) * ld;
        for (int j = 0; j < dpad; ++j) {
          const float qv = qrow[j];
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const float xv = Xs[(tv + 16 * i) * ld + j];
            if (a.metric == MV_L2) {
              const float df = qv - xv;
              acc[i] = fmaf(df, df, acc[i]);
            } else {
              acc[i] = fmaf(qv, xv, acc[i]);
            }
          }
        }
#pragma unroll
        for (int i = 0; i < 4; ++i) Dt[(tq + 16 * jq) * (kVT + 1) + tv + 16 * i] = acc[i];
      }
      __syncthreads();
      for (int qi = warp; qi < nqc; qi += 8) {
        const int64_t p = qpair[qi];
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int v = lane + 32 * h;
          const bool ok = rvalid[v];
          const uint32_t k32 = dist_key(Dt[qi * (kVT + 1) + v], a.metric);
          const uint64_t key = ((uint64_t)k32 << 32) | rrank[v];
          if (sel) {
            uint64_t* L = lists + (int64_t)qi * k;
            warp_list_insert(L, k, key, ok);
          } else {
            const uint32_t m = __ballot_sync(MV_FULL, ok);
            const int pos = qcnt[qi] + __popc(m & ((1u << lane) - 1));
            if (ok) a.part[a.poff[p] + pos] = key;
            __syncwarp();
            if (lane == 0) qcnt[qi] += __popc(m);
            __syncwarp();
          }
        }
      }
    }
    __syncthreads();
    for (int qi = warp; qi < nqc; qi += 8) {
      const int64_t p = qpair[qi];
      if (sel) {
        const uint64_t* L = lists + (int64_t)qi * k;
        int c = 0;
        for (int j0 = 0; j0 < k; j0 += 32) {  // warp-uniform trip count: every lane reaches the ballot
          const int j = j0 + lane;
          const uint64_t v = j < k ? L[j] : MV_KEY_PAD;
          if (v != MV_KEY_PAD) a.part[a.poff[p] + j] = v;
          c += __popc(__ballot_sync(MV_FULL, v != MV_KEY_PAD));
        }
        if (lane == 0) a.pcnt[p] = c;
      } else if (lane == 0) {
        a.pcnt[p] = qcnt[qi];
      }
    }
  }
}

static size_t scan_smem(int dpad, int k, int qchunk) {
  const int ld = dpad + 1;
  size_t b = (size_t)(kVT + kQCMax) * ld * 4 + (size_t)kQCMax * (kVT + 1) * 4 + 256 * 4 + kVT * 8 +
             kQCMax * 8 + 16;
  b = (b + 15) & ~(size_t)15;
  if (k <= kLocalSelectMaxK) b += (size_t)qchunk * k * 8;
  return b;
}

cudaError_t launch_scan(const ScanArgs& a, cudaStream_t st) {
  const size_t smem = scan_smem(a.dpad, a.k, a.qchunk);
  auto kern = a.type == MV_IVF_FLAT ? k_scan_simt<MV_IVF_FLAT> : k_scan_simt<MV_IVF_SQ8>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 256, smem);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = kNumSMs;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  kern<<<nsm * max(per_sm, 1), 256, smem, st>>>(a);
  return cudaGetLastError();
}

}  // namespace mv
