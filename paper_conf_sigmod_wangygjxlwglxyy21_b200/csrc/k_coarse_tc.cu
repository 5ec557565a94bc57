// k_coarse_tc.cu -- §8 rows a2 + a3 on the tensor cores: the queries x centroids contraction with
// the per-query top-nprobe fused into its epilogue (the score matrix never reaches HBM).
//
// PAPER.md:523-529 (§3.1) step (1): "find the closest nprobe buckets based on the distance between
// q and the centroid of each bucket"; PAPER.md:838-843 (§3.4): this step "has a much higher
// computation-to-I/O ratio than step 2 ... all the queries compare against the same K centroids".
//
// CTA = one block of NQB queries (B operand: tf32 hi/lo planes, loaded once by TMA) streaming all
// centroid tiles (A operand: 128 centroids, tf32 hi and lo planes, TMA ring).  Per K-step two MMAs:
//   D[:, 0:2NQB] (=) C_hi . [Q_hi ; Q_lo]^T        D[:, 0:NQB] += C_lo . Q_hi^T
// so dot = D[:, j] + D[:, NQB + j] = q.c up to the dropped lo x lo term (~2^-22 relative).
// Score = ||c||^2 - 2 q.c (L2) or -q.c (IP), key = (score key << 32) | centroid id; the epilogue
// (8 warps, two per TMEM lane quarter) transposes the tile through shared memory and folds it into
// each query's running top-nprobe with warp_select_tile (shared with the list scan).
#include "mv_internal.cuh"
#include "sm100.cuh"

namespace mv {
using namespace sm100;

namespace {
constexpr int kCEpi = 8;
constexpr int kCThreads = 64 + 32 * kCEpi;  // warp 0 TMA, warp 1 MMA, warps 2..9 epilogue
constexpr int kCDLD = 129;

__device__ __forceinline__ void cbar(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }
}  // namespace

template <int NQB>
constexpr uint32_t coarse_tmem_cols() {
  return 4 * NQB <= 128 ? 128 : (4 * NQB <= 256 ? 256 : 512);
}

template <int NQB>
__global__ void __launch_bounds__(kCThreads, 1)
    k_coarse_tc(const __grid_constant__ CUtensorMap cmap, const __grid_constant__ CUtensorMap qmap, const CoarseParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  constexpr int ATOM = 128;            // tf32: 32 fp32 per 128-B swizzle atom row
  constexpr int ABYTES = 128 * ATOM;   // one 128-centroid chunk of one plane
  constexpr int BROWS = 2 * NQB;       // hi rows then lo rows
  const int nchunks = p.nchunks, nstage = p.nstage, nprobe = p.nprobe;
  const int ntiles = (p.nlist + 127) >> 7;
  const int q0 = blockIdx.x * NQB;

  uint8_t* Bs = sm;                                       // nchunks x BROWS x 128 B
  uint8_t* As = Bs + nchunks * BROWS * ATOM;              // nstage x (hi chunk, lo chunk)
  uint32_t* Dt = reinterpret_cast<uint32_t*>(As + nstage * 2 * ABYTES);  // NQB x kCDLD
  uint64_t* lists = reinterpret_cast<uint64_t*>(Dt + NQB * kCDLD + (NQB * kCDLD & 1));  // NQB x nprobe
  uint64_t* scratch = lists + NQB * nprobe;               // 32 per epilogue warp
  uint64_t* cbuf = scratch + 32 * kCEpi;                  // NQB x 32 survivor buffers (nprobe <= 32)
  int* cnb = reinterpret_cast<int*>(cbuf + NQB * 32);     // NQB buffer counts
  uint32_t* cbnd = reinterpret_cast<uint32_t*>(cnb + NQB);  // NQB running bounds
  uint64_t* bars = reinterpret_cast<uint64_t*>(cbnd + NQB);
  uint64_t* full_a = bars;
  uint64_t* empty_a = bars + nstage;
  uint64_t* full_b = empty_a + nstage;
  uint64_t* tfull = full_b + 1;
  uint64_t* tempty = tfull + 2;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < nstage; ++s) {
      mbar_init(&full_a[s], 1);
      mbar_init(&empty_a[s], 1);
    }
    mbar_init(full_b, 1);
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], kCEpi);
    }
    fence_mbar_init();
  }
  if (warp == 1) {
    tmem_alloc(tslot, coarse_tmem_cols<NQB>());
    tmem_relinquish();
  }
  if (warp == 0 && lane == 0) {
    tma_prefetch(&cmap);
    tma_prefetch(&qmap);
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tslot;

  if (warp == 0) {
    if (lane == 0) {
      // query block: hi rows [q0, q0+NQB) and lo rows [nq + q0, ...) of the plane-major matrix
      mbar_expect_tx(full_b, nchunks * BROWS * ATOM);
      for (int c = 0; c < nchunks; ++c) {
        tma_load_2d(Bs + c * BROWS * ATOM, &qmap, full_b, c * 32, q0);
        tma_load_2d(Bs + c * BROWS * ATOM + NQB * ATOM, &qmap, full_b, c * 32, p.nq + q0);
      }
      uint32_t it = 0;
      for (int t = 0; t < ntiles; ++t)
        for (int c = 0; c < nchunks; ++c, ++it) {
          const uint32_t s = it % nstage, r = it / nstage;
          mbar_wait(&empty_a[s], (r & 1) ^ 1);
          mbar_expect_tx(&full_a[s], 2 * ABYTES);
          tma_load_2d(As + s * 2 * ABYTES, &cmap, &full_a[s], c * 32, t * 128);
          tma_load_2d(As + s * 2 * ABYTES + ABYTES, &cmap, &full_a[s], c * 32, p.nlist + t * 128);
        }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      mbar_wait(full_b, 0);
      tc_fence_after();
      const uint32_t id_full = idesc_tf32(BROWS), id_hi = idesc_tf32(NQB);
      uint32_t it = 0;
      for (int t = 0; t < ntiles; ++t) {
        const uint32_t a = t & 1;
        mbar_wait(&tempty[a], ((t >> 1) & 1) ^ 1);
        tc_fence_after();
        const uint32_t d = tmem + a * 2 * NQB;
        for (int c = 0; c < nchunks; ++c, ++it) {
          const uint32_t s = it % nstage;
          mbar_wait(&full_a[s], (it / nstage) & 1);
          tc_fence_after();
          const uint32_t ah = smem_u32(As + s * 2 * ABYTES), al = ah + ABYTES;
          const uint32_t bb = smem_u32(Bs + c * BROWS * ATOM);
#pragma unroll
          for (int ks = 0; ks < 4; ++ks) {
            mma_tf32(d, kmajor_desc(ah + ks * 32, ATOM), kmajor_desc(bb + ks * 32, ATOM), id_full, (c | ks) != 0);
            mma_tf32(d, kmajor_desc(al + ks * 32, ATOM), kmajor_desc(bb + ks * 32, ATOM), id_hi, 1);
          }
          mma_commit(&empty_a[s]);
        }
        mma_commit(&tfull[a]);
      }
    }
  } else {
    // ------------------------------------------------------------------ epilogue
    const int ew = warp - 2;             // 0..7
    const int quarter = warp & 3;
    const int half = ew >> 2;
    const int row = quarter * 32 + lane;  // centroid within the tile
    const int et = threadIdx.x - 64;
    uint64_t* wscr = scratch + ew * 32;
    const int nqv = (int)min64(NQB, p.nq - q0);
    for (int i = et; i < NQB * nprobe; i += 32 * kCEpi) lists[i] = MV_KEY_PAD;
    for (int i = et; i < NQB; i += 32 * kCEpi) {
      cnb[i] = 0;
      cbnd[i] = 0xffffffffu;
    }
    float cn_next = (row < p.nlist && p.metric == MV_L2) ? __ldg(p.cnorm + row) : 0.0f;
    cbar(1, 32 * kCEpi);
    for (int t = 0; t < ntiles; ++t) {
      const uint32_t a = t & 1;
      const int cid = t * 128 + row;
      const bool valid = cid < p.nlist;
      const float cn = cn_next;
      const int nid = cid + 128;
      cn_next = (nid < p.nlist && p.metric == MV_L2) ? __ldg(p.cnorm + nid) : 0.0f;  // prefetch next tile
      mbar_wait(&tfull[a], (t >> 1) & 1);
      tc_fence_after();
      const uint32_t tb = tmem + a * 2 * NQB + ((uint32_t)(quarter * 32) << 16);
#pragma unroll
      for (int qc = half * 16; qc < ((p.dbg & 2) ? 0 : NQB); qc += 32) {
        uint32_t rh[16], rl[16];
        tmem_ld16(tb + qc, rh);
        tmem_ld16(tb + NQB + qc, rl);
        tmem_wait_ld();
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          const float dot = __uint_as_float(rh[j]) + __uint_as_float(rl[j]);
          const float sc = p.metric == MV_L2 ? cn - 2.0f * dot : -dot;
          Dt[(qc + j) * kCDLD + row] = valid ? f2key(sc) : 0xffffffffu;
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[a]);
      cbar(1, 32 * kCEpi);
      const uint32_t cbase = t * 128;
      if (nprobe <= 32) {
        constexpr int G = 4;
        for (int j0 = ew; j0 < ((p.dbg & 1) ? 0 : nqv); j0 += kCEpi * G) {
          const int nvalid = min(G, (nqv - j0 + kCEpi - 1) / kCEpi);
          warp_filter_group<G>(
              nvalid, nprobe, [&](int g, int m) { return Dt[(j0 + g * kCEpi) * kCDLD + m * 32 + lane]; },
              [&](int g, uint64_t*& L, uint64_t*& B, int*& nb, uint32_t*& bnd, uint64_t& li) {
                const int j = j0 + g * kCEpi;
                L = lists + (int64_t)j * nprobe;
                B = cbuf + j * 32;
                nb = cnb + j;
                bnd = cbnd + j;
                li = MV_KEY_PAD;
              },
              [&](int, int v) { return cbase + (uint32_t)v; }, [](int, uint32_t) {}, wscr);
        }
      } else {
        // 32 < nprobe <= 128: filter against the list's nprobe-th best, buffered merges
        for (int j = ew; j < ((p.dbg & 1) ? 0 : nqv); j += kCEpi) {
          uint64_t* L = lists + (int64_t)j * nprobe;
          const uint32_t thr32 = (uint32_t)(L[nprobe - 1] >> 32);
          uint32_t k32[4];
          bool pass[4];
          int npass = 0;
#pragma unroll
          for (int m = 0; m < 4; ++m) {
            k32[m] = Dt[j * kCDLD + m * 32 + lane];
            pass[m] = k32[m] != 0xffffffffu && k32[m] <= thr32;
            npass += __popc(__ballot_sync(MV_FULL, pass[m]));
          }
          if (npass == 0) continue;
          auto low = [&](int v) { return cbase + (uint32_t)v; };
          if (nprobe <= 64) warp_collect_R<2>(L, cbuf + j * 32, cnb + j, nprobe, k32, pass, npass, low);
          else warp_collect_R<4>(L, cbuf + j * 32, cnb + j, nprobe, k32, pass, npass, low);
        }
      }
      cbar(1, 32 * kCEpi);
    }
    for (int j = ew; j < nqv; j += kCEpi) {
      uint64_t* L = lists + (int64_t)j * nprobe;
      if (nprobe <= 32) warp_flush_buffer(L, cbuf + j * 32, cnb + j, cbnd + j, nprobe, MV_KEY_PAD);
      else if (nprobe <= 64) warp_flush_buffer_R<2>(L, cbuf + j * 32, cnb + j, nprobe);
      else warp_flush_buffer_R<4>(L, cbuf + j * 32, cnb + j, nprobe);
    }
    cbar(1, 32 * kCEpi);
    for (int i = et; i < nqv * nprobe; i += 32 * kCEpi) {
      const int j = i / nprobe, r = i - j * nprobe;
      const uint64_t key = lists[i];  // PAD only in MV_COARSE_DEBUG runs: keep the probe ids in range
      p.probes[(int64_t)(q0 + j) * nprobe + r] = key == MV_KEY_PAD ? r % p.nlist : (int32_t)(uint32_t)(key & 0xffffffffu);
    }
  }
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem, coarse_tmem_cols<NQB>());
  }
}

// plane-major tf32 split: out[0][r][:] = hi(x_r), out[1][r][:] = x_r - hi(x_r)
// tf32 round-to-nearest (ties away): the value with the low 13 mantissa bits cleared nearest to v
__device__ __forceinline__ float tf32_rn(float v) {
  const uint32_t b = __float_as_uint(v);
  if ((b & 0x7f800000u) == 0x7f800000u) return __uint_as_float(b & 0xffffe000u);  // inf / nan
  return __uint_as_float((b + 0x1000u) & 0xffffe000u);
}

// Both planes are tf32-representable (the MMA's operand truncation is then exact): hi = rn(x) and
// lo = rn(x - hi), |lo| <= 2^-11 |x|, so hi + lo = x to ~2^-22 relative with unbiased rounding.
__global__ void k_hilo(const float* __restrict__ x, int64_t n, int d, int dpad, float* __restrict__ out, int* lo_any) {
  const int64_t total = n * dpad;
  bool nz = false;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = t / dpad;
    const int j = (int)(t - r * dpad);
    const float v = j < d ? x[r * d + j] : 0.0f;
    const float hi = tf32_rn(v);
    const float lo = tf32_rn(v - hi);
    out[t] = hi;
    out[total + t] = lo;
    nz |= lo != 0.0f;
  }
  if (lo_any && __syncthreads_or(nz) && threadIdx.x == 0) atomicOr(lo_any, 1);
}

cudaError_t launch_hilo(const float* x, int64_t n, int d, int dpad, float* out, int* lo_any, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  const int grid = (int)min64(kNumSMs * 16, (n * dpad + 255) / 256);
  k_hilo<<<grid, 256, 0, st>>>(x, n, d, dpad, out, lo_any);
  return cudaGetLastError();
}

static int coarse_fixed_smem(int nqb, int nchunks, int nprobe) {
  return nchunks * 2 * nqb * 128 + nqb * kCDLD * 4 + 8 + nqb * nprobe * 8 + 32 * kCEpi * 8 + nqb * 32 * 8 + nqb * 8 + 256;
}

// Query-block size: the one that minimises (waves x block size) -- a second, mostly empty wave
// doubles the coarse time -- among the shapes whose shared memory fits with >= 2 centroid stages.
bool coarse_tc_plan(int dpad, int nprobe, int64_t nq, int nsm, CoarseParams& p) {
  if (dpad % 32 != 0 || nprobe > 128) return false;
  p.nchunks = dpad / 32;
  p.nprobe = nprobe;
  const int budget = 227 * 1024 - 1024;
  const int stage = 2 * 128 * 128;
  int best = -1;
  int64_t best_cost = 0;
  for (int nqb : {32, 48, 64, 80}) {
    if (nprobe > 32 && nqb > 32) continue;
    const int fixed = coarse_fixed_smem(nqb, p.nchunks, nprobe);
    if ((budget - fixed) / stage < 2) continue;
    const int64_t blocks = (nq + nqb - 1) / nqb;
    const int64_t cost = ((blocks + nsm - 1) / nsm) * (int64_t)(nqb + 32);  // + fixed per-CTA streaming
    if (best < 0 || cost < best_cost) {
      best = nqb;
      best_cost = cost;
    }
  }
  if (best < 0) return false;
  p.nqb = best;
  const int fixed = coarse_fixed_smem(best, p.nchunks, nprobe);
  p.nstage = std::min(4, (budget - fixed) / stage);
  p.smem_total = fixed + p.nstage * stage + 1024;
  return p.smem_total <= 227 * 1024;
}

template <int NQB>
static cudaError_t run_coarse_tc(const CUtensorMap* cmap, const CUtensorMap* qmap, const CoarseParams& p, unsigned grid,
                                 cudaStream_t st) {
  cudaError_t e = cudaFuncSetAttribute(k_coarse_tc<NQB>, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_total);
  if (e != cudaSuccess) return e;
  k_coarse_tc<NQB><<<grid, kCThreads, p.smem_total, st>>>(*cmap, *qmap, p);
  return cudaGetLastError();
}

cudaError_t launch_coarse_tc(const CUtensorMap* cmap, const CUtensorMap* qmap, const CoarseParams& p, int64_t nq,
                             cudaStream_t st) {
  const unsigned grid = (unsigned)((nq + p.nqb - 1) / p.nqb);
  switch (p.nqb) {
    case 32: return run_coarse_tc<32>(cmap, qmap, p, grid, st);
    case 48: return run_coarse_tc<48>(cmap, qmap, p, grid, st);
    case 64: return run_coarse_tc<64>(cmap, qmap, p, grid, st);
    default: return run_coarse_tc<80>(cmap, qmap, p, grid, st);
  }
}

}  // namespace mv
