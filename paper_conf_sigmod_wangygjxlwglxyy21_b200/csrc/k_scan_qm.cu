// k_scan_qm.cu -- §8 rows a5 + a6 for IVF_FLAT on the 5th-generation tensor cores (sm_100a),
// queries on the MMA's M side.
//
// PAPER.md:529-532 (§3.1) step (2): scan the nprobe probed buckets; PAPER.md:916-922 (§4.1 B): the
// bitmap is checked for every encountered vector before the top-k; PAPER.md:569-575 (§3.2.1): one
// loaded list tile is reused by every query of the list's bucket (one tensor-core contraction).
//
// Orientation.  D[128 query lanes x N vectors] = Qplanes[128 x K] . X_tile[N x K]^T: the bucket's
// queries are the A operand (gathered once per work item), the list tile is the B operand (TMA,
// N = 128 rows, or roundup16 of the list's tail).  Every epilogue thread owns one query (one TMEM
// lane) and walks its row of distances: the threshold tau_q, ||q||^2 and the output region live in
// registers, survivors are counted per 32 columns and appended with one shared atomic -- no
// ballots, no per-column shuffles.  The tf32 hi and lo query planes of a split query accumulate into
// the same lanes (two MMAs, one accumulator), so the epilogue reads one value per distance.
//
// Work item = (list l, <= QC queries probing l).  QC = 96 queries of one plane (tf32-exact queries)
// or 48 of two; rows QC..127 of the A operand are whatever follows in shared memory (their lanes
// are never read).  Persistent CTA per SM, warp-specialised:
//   warp 0     TMA producer: list tiles (128 rows, or 16-row boxes for the list's tail, so the
//              over-read past a list end is < 16 rows) + the tiles' side data (norms, id ranks,
//              ids) by bulk copy
//   warp 1     TMEM owner + single-thread tcgen05.mma issuer; 4 accumulator buffers of 128 columns
//   warps 2-3  query gatherer: the bucket's query planes -> swizzled K-major smem, and the
//              per-query metadata -- both double-buffered
//   warps 4-11 epilogue, two warps per TMEM lane quarter (64 columns each)
// Phases as in k_scan_tc.cu: phase A emits every candidate of a prefix of each query's nearest
// lists, phase B emits keys <= tau_q over all probed lists.
#include "mv_internal.cuh"
#include "sm100.cuh"

namespace mv {
using namespace sm100;

namespace {
__device__ __forceinline__ void named_bar(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }

constexpr int kQmNTS = 4;         // side-data ring slots = TMEM accumulator buffers
constexpr int kQmAcc = 4;
// side slot: norms f64 [1152 B] | rank u32 [640 B] | ids i64 [1152 B] | bias f32 [512 B]
constexpr int kQmSide = 3584;
constexpr int kQmRank = 1152, kQmIds = 1792, kQmBias = 3072;
constexpr int kQmEpi = 8;
constexpr int kQmThreads = 128 + 32 * kQmEpi;
constexpr int kQmMetaPerQuery = 32;  // pair i32, cnt i32, thf f32, qnf f32, tau u64, base i64 (+ 32-B header)

struct QmWork {
  int nqc, len, ntiles, bstart;
  int64_t lstart;
};
// per-buffer metadata: the work item's header, then per query pair, cnt, thf, qnf, tau, base
struct QmMeta {
  QmWork* wi;
  int32_t* pair;
  int32_t* cnt;
  float* thf;
  float* qnf;
  uint64_t* tau;
  int64_t* base;
};
__device__ __forceinline__ QmMeta qm_meta(uint8_t* m, int QC) {
  QmMeta r;
  r.wi = reinterpret_cast<QmWork*>(m);
  r.pair = reinterpret_cast<int32_t*>(m + 32);
  r.cnt = r.pair + QC;
  r.thf = reinterpret_cast<float*>(r.cnt + QC);
  r.qnf = r.thf + QC;
  r.tau = reinterpret_cast<uint64_t*>(r.qnf + QC);
  r.base = reinterpret_cast<int64_t*>(r.tau + QC);
  return r;
}

// work item w = witems[w] = (virtual list, first bucket position) -> its list range and queries
__device__ __forceinline__ QmWork qm_work(const TcScanParams& p, int2 it, int qc) {
  QmWork wi;
  const int l = it.x >= p.nlist ? it.x - p.nlist : it.x;
  wi.bstart = it.y;
  wi.nqc = min(qc, p.boff[it.x + 1] - wi.bstart);
  wi.lstart = p.list_off[l];
  wi.len = (int)min64(p.list_off[l + 1] - wi.lstart, p.rowcap);
  wi.ntiles = (wi.len + 127) >> 7;
  return wi;
}
}  // namespace

__global__ void __launch_bounds__(kQmThreads, 1)
    k_scan_qm(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ CUtensorMap xmap16, const TcScanParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  constexpr int ATOM = 128;            // 32 fp32 per swizzle-atom row
  constexpr int STAGE = 128 * ATOM;    // one K-chunk of one 128-row tile
  const int nstage = p.nstage, nchunks = p.nchunks;
  const int QCMAX = p.qchunk;          // A-operand rows per buffer (96)
  const int P = p.cfg[1];              // 1: tf32-exact queries (QC = 96), 2: hi + lo planes (QC = 48)
  const int QC = p.cfg[0];
  const int rowbytes = p.dpad * 4;
  const bool use_norms = p.metric == MV_L2;
  const bool use_ids = p.bitset != nullptr;
  const bool phaseB = p.phase != 0;

  uint8_t* As = sm + p.off_q;          // 2 buffers x nchunks x QCMAX rows x 128 B
  uint8_t* Xs = sm + p.off_x;
  uint8_t* metab = sm + p.off_meta;
  uint8_t* side = sm + p.off_side;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + p.off_bar);
  uint64_t* full_x = bars;
  uint64_t* empty_x = bars + nstage;
  uint64_t* full_q = empty_x + nstage;
  uint64_t* empty_q = full_q + 2;
  uint64_t* empty_m = empty_q + 2;
  uint64_t* tfull = empty_m + 2;
  uint64_t* tempty = tfull + kQmAcc;
  uint64_t* full_t = tempty + kQmAcc;
  uint64_t* empty_t = full_t + kQmNTS;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(empty_t + kQmNTS);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < nstage; ++s) {
      mbar_init(&full_x[s], 1);
      mbar_init(&empty_x[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&full_q[b], 64);
      mbar_init(&empty_q[b], 1);
      mbar_init(&empty_m[b], kQmEpi);
    }
    for (int a = 0; a < kQmAcc; ++a) {
      mbar_init(&tfull[a], 1);
      mbar_init(&tempty[a], kQmEpi);
    }
    for (int s = 0; s < kQmNTS; ++s) {
      mbar_init(&full_t[s], 1);
      mbar_init(&empty_t[s], kQmEpi);
    }
    fence_mbar_init();
  }
  if (warp == 1) {
    tmem_alloc(tslot, 512);
    tmem_relinquish();
  }
  if (warp == 0 && lane == 0) {
    tma_prefetch(&xmap);
    tma_prefetch(&xmap16);
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tslot;
  const int nwork = *p.nwitems;
  const int w0 = (p.wbeg ? *p.wbeg : 0) + blockIdx.x;
  const int abuf = nchunks * QCMAX * ATOM;  // bytes per A buffer

  if (warp == 0) {
    // ------------------------------------------------------------------ TMA producer
    if (lane == 0) {
      uint32_t it = 0, tcount = 0;
      const bool side_on = !(p.dbg & 32);
      const uint32_t side_tx = side_on ? 528 + (use_norms ? 1040 : 0) + (use_ids ? 1040 : 0) : 0;
      // two-deep prefetch: the next item's list range and the one after's (list, bucket) pair are
      // in flight while this item's tiles are issued, so no dependent load sits between items
      const int G = gridDim.x;
      int2 itn = w0 + G < nwork ? p.witems[w0 + G] : make_int2(0, 0);
      QmWork wn = w0 < nwork ? qm_work(p, p.witems[w0], QC) : QmWork{};
      for (int w = w0; w < nwork; w += G) {
        const QmWork wi = wn;
        if (w + G < nwork) wn = qm_work(p, itn, QC);
        if (w + 2 * G < nwork) itn = p.witems[w + 2 * G];
        for (int t = 0; t < wi.ntiles; ++t, ++tcount) {
          const int row0 = (int)(wi.lstart + t * 128);
          const int rows = min(128, wi.len - t * 128);
          const int nb16 = (rows + 15) >> 4;
          const uint32_t ts = tcount % kQmNTS, tr = tcount / kQmNTS;
          mbar_wait(&empty_t[ts], (tr & 1) ^ 1);
          mbar_expect_tx(&full_t[ts], side_tx);
          uint8_t* sd = side + ts * kQmSide;
          if (side_on) {
            bulk_g2s(sd + kQmRank, p.rank + (row0 & ~3), 528, &full_t[ts]);
            if (use_norms) bulk_g2s(sd, p.norms + (row0 & ~1), 1040, &full_t[ts]);
            if (use_ids) bulk_g2s(sd + kQmIds, p.ids + (row0 & ~1), 1040, &full_t[ts]);
          }
          for (int c = 0; c < nchunks; ++c, ++it) {
            const uint32_t s = it % nstage, r = it / nstage;
            mbar_wait(&empty_x[s], (r & 1) ^ 1);
            uint8_t* dst = Xs + s * STAGE;
            if (rows == 128 || (p.dbg & 8)) {
              mbar_expect_tx(&full_x[s], STAGE);
              tma_load_2d(dst, &xmap, &full_x[s], c * 32, row0);
            } else {
              // the list's tail: 16-row boxes, so at most 15 rows past the list end are read
              mbar_expect_tx(&full_x[s], nb16 * 16 * ATOM);
              for (int b16 = 0; b16 < nb16; ++b16)
                tma_load_2d(dst + b16 * 16 * ATOM, &xmap16, &full_x[s], c * 32, row0 + 16 * b16);
            }
          }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------------ MMA issuer
    if (lane == 0) {
      uint32_t it = 0, titer = 0, wcount = 0;
      for (int w = w0; w < nwork; w += gridDim.x, ++wcount) {
        const uint32_t b = wcount & 1;
        mbar_wait(&full_q[b], (wcount >> 1) & 1);
        tc_fence_after();
        const QmWork wi = *qm_meta(metab + b * p.meta_bytes, QCMAX).wi;
        const uint32_t abase = smem_u32(As + b * abuf);
        for (int t = 0; t < wi.ntiles; ++t, ++titer) {
          const int rows = min(128, wi.len - t * 128);
          const uint32_t idesc = idesc_tf32((rows + 15) & ~15);
          const uint32_t a = titer % kQmAcc;
          mbar_wait(&tempty[a], ((titer / kQmAcc) & 1) ^ 1);
          tc_fence_after();
          const uint32_t dcol = tmem + a * 128;
          for (int c = 0; c < nchunks; ++c, ++it) {
            const uint32_t s = it % nstage;
            mbar_wait(&full_x[s], (it / nstage) & 1);
            tc_fence_after();
            const uint32_t xb = smem_u32(Xs + s * STAGE);
            const uint32_t qb = abase + c * QCMAX * ATOM;
#pragma unroll
            for (int ks = 0; ks < ATOM / 32; ++ks) {
              if (p.dbg & 16) break;
              const uint64_t bd = kmajor_desc(xb + ks * 32, ATOM);
              mma_tf32(dcol, kmajor_desc(qb + ks * 32, ATOM), bd, idesc, (c | ks) != 0);
              if (P == 2) mma_tf32(dcol, kmajor_desc(qb + QC * ATOM + ks * 32, ATOM), bd, idesc, 1);
            }
            mma_commit(&empty_x[s]);
          }
          mma_commit(&tfull[a]);
        }
        mma_commit(&empty_q[b]);
      }
    }
  } else if (warp < 4) {
    // ------------------------------------------------------------------ query gatherer (64 thr)
    const int tq = threadIdx.x - 64;
    const int G = gridDim.x;
    // the next item's list range and per-query metadata are loaded into registers before waiting
    // for its buffers, so only the plane copies sit on the critical path once a buffer frees
    struct Pref {
      QmWork wi;
      int pr[2], q[2];
      uint64_t tau[2];
      double qn[2];
      int64_t base[2];
    };
    auto prefetch = [&](int w) {
      Pref f;
      f.wi = qm_work(p, p.witems[w], QC);
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        const int i = tq + 64 * u;
        if (i < f.wi.nqc) {
          f.pr[u] = p.bq[f.wi.bstart + i];
          // phase-A entries carry pair id npairs + p (their own output regions)
          const int64_t npairs = p.nq * p.npb;
          f.q[u] = (int)((f.pr[u] >= npairs ? f.pr[u] - npairs : f.pr[u]) / p.npb);
          f.tau[u] = phaseB ? p.tau[f.q[u]] : MV_KEY_PAD;
          f.qn[u] = p.qnorm[f.q[u]];
          f.base[u] = p.poff[f.pr[u]];
        }
      }
      return f;
    };
    Pref cur;
    if (w0 < nwork) cur = prefetch(w0);
    uint32_t wcount = 0;
    for (int w = w0; w < nwork; w += G, ++wcount) {
      Pref nxt;
      if (w + G < nwork) nxt = prefetch(w + G);
      const QmWork wi = cur.wi;
      const uint32_t b = wcount & 1, r = wcount >> 1;
      mbar_wait(&empty_q[b], (r & 1) ^ 1);
      mbar_wait(&empty_m[b], (r & 1) ^ 1);
      const QmMeta mt = qm_meta(metab + b * p.meta_bytes, QCMAX);
      if (tq == 0) *mt.wi = wi;
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        const int i = tq + 64 * u;
        if (i < wi.nqc) {
          const uint64_t t = cur.tau[u];
          const uint32_t t32 = (uint32_t)(t >> 32);
          mt.pair[i] = cur.pr[u];
          mt.cnt[i] = 0;
          mt.tau[i] = t;
          mt.thf[i] = t32 >= 0xff800000u ? __int_as_float(0x7f800000) : key2f(t32);
          mt.qnf[i] = (float)cur.qn[u];
          mt.base[i] = cur.base[u];
        }
      }
      named_bar(2, 64);
      uint8_t* Ab = As + b * abuf;
      constexpr int PIECES = ATOM / 16;
      const int total = (p.dbg & 4) ? 0 : wi.nqc * P * nchunks * PIECES;
      for (int idx = tq; idx < total; idx += 64) {
        const int pc = idx % PIECES;
        int rest = idx / PIECES;
        const int c = rest % nchunks;
        rest /= nchunks;
        const int pl = rest % P;
        const int i = rest / P;
        const int q = (int)((mt.pair[i] >= p.nq * p.npb ? mt.pair[i] - p.nq * p.npb : mt.pair[i]) / p.npb);
        cp_async16(Ab + c * QCMAX * ATOM + swz_off(pl * QC + i, pc, ATOM),
                   p.qplanes + ((int64_t)pl * p.nq + q) * rowbytes + c * ATOM + pc * 16);
      }
      cp_async_wait_all();
      fence_proxy_async();
      mbar_arrive(&full_q[b]);
      cur = nxt;
    }
  } else {
    // ------------------------------------------------------------------ epilogue (8 warps)
    const int ew = warp - 4;             // 0..7
    const int quarter = warp & 3;        // TMEM lane quarter this warp may access
    const int half = ew >> 2;            // columns [64 half, 64 half + 64) of each tile
    const int qi = quarter * 32 + lane;  // this thread's query within the work item
    const int et = threadIdx.x - 128;    // 0..255
    uint32_t titer = 0, wcount = 0;
    for (int w = w0; w < nwork; w += gridDim.x, ++wcount) {
      const uint32_t b = wcount & 1;
      mbar_wait(&full_q[b], (wcount >> 1) & 1);
      const QmMeta mt = qm_meta(metab + b * p.meta_bytes, QCMAX);
      const QmWork wi = *mt.wi;
      const bool active = qi < wi.nqc;
      const bool warp_active = quarter * 32 < wi.nqc && !(p.dbg & 2);
      float qn = 0.f, thf = 0.f;
      uint64_t tau = 0;
      int64_t base = 0;
      if (active) {
        qn = mt.qnf[qi];
        thf = mt.thf[qi];
        tau = mt.tau[qi];
        base = mt.base[qi];
      }
      if (!active) thf = __int_as_float(0xff800000u);  // -inf: nothing passes
      for (int t = 0; t < wi.ntiles; ++t, ++titer) {
        const uint32_t a = titer % kQmAcc;
        const uint32_t ts = titer % kQmNTS;
        const int rows = min(128, wi.len - t * 128);
        const int row0 = (int)(wi.lstart + t * 128);
        mbar_wait(&full_t[ts], (titer / kQmNTS) & 1);
        uint8_t* sd = side + ts * kQmSide;
        float* bias = reinterpret_cast<float*>(sd + kQmBias);
        const uint32_t* rk = reinterpret_cast<const uint32_t*>(sd + kQmRank) + (row0 & 3);
        if (et < 128) {
          // per-row term of the distance: ||x||^2 (L2) or 0 (IP); NaN for rows past the list end
          // and for rows the bitset excludes, so no comparison passes for them
          bool valid = et < rows;
          if (valid && use_ids)
            valid = !bit_excluded(p.bitset, p.nbits, reinterpret_cast<const int64_t*>(sd + kQmIds)[(row0 & 1) + et]);
          const float xn = use_norms ? (float)reinterpret_cast<const double*>(sd)[(row0 & 1) + et] : 0.0f;
          bias[et] = valid ? xn : __int_as_float(0x7fffffff);
        }
        named_bar(1, 32 * kQmEpi);
        mbar_wait(&tfull[a], (titer / kQmAcc) & 1);
        tc_fence_after();
        const uint32_t tbase = tmem + a * 128 + ((uint32_t)(quarter * 32) << 16);
        if (warp_active) {
          for (int c0 = half * 64; c0 < min(half * 64 + 64, rows); c0 += 32) {
            uint32_t r[32];
            tmem_ld32(tbase + c0, r);
            float bv[32];
#pragma unroll
            for (int v = 0; v < 8; ++v) {
              const float4 b4 = reinterpret_cast<const float4*>(bias + c0)[v];
              bv[4 * v] = b4.x; bv[4 * v + 1] = b4.y; bv[4 * v + 2] = b4.z; bv[4 * v + 3] = b4.w;
            }
            tmem_wait_ld();
            float dv[32];
            uint32_t m = 0;
#pragma unroll
            for (int j = 0; j < 32; ++j) {
              const float dot = __uint_as_float(r[j]);
              // exact for tf32-representable data; same operation order as the SIMT path
              dv[j] = use_norms ? (qn + bv[j]) - 2.0f * dot : bv[j] - dot;
              if (dv[j] <= thf) m |= 1u << j;
            }
            if (m && !(p.dbg & 1)) {
              uint32_t m2 = 0;
              uint64_t kk[32];
#pragma unroll
              for (int j = 0; j < 32; ++j) {
                kk[j] = ((uint64_t)f2key(dv[j]) << 32) | rk[c0 + j];
                if (((m >> j) & 1) && (!phaseB || kk[j] <= tau)) m2 |= 1u << j;
              }
              if (m2) {
                int pos = atomicAdd(mt.cnt + qi, __popc(m2));
                uint64_t* dst = p.part + base;
#pragma unroll
                for (int j = 0; j < 32; ++j)
                  if ((m2 >> j) & 1) dst[pos++] = kk[j];
              }
            }
          }
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          mbar_arrive(&tempty[a]);
          mbar_arrive(&empty_t[ts]);
        }
      }
      // every epilogue warp is done with this work item: publish the pairs' counts, free the metadata
      named_bar(1, 32 * kQmEpi);
      for (int i = et; i < wi.nqc; i += 32 * kQmEpi) p.pcnt[mt.pair[i]] = mt.cnt[i];
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty_m[b]);
    }
  }
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem, 512);
  }
}

// Shared-memory plan: [A0 | A1 | X ring | side ring | metadata x 2 | barriers].  The MMA reads 128
// A rows from each chunk block, i.e. up to 16 KB past a block start: the blocks are followed by
// more shared memory (A1, then the X ring), so those reads stay inside the allocation.
bool qm_scan_plan(int dpad, int k, TcScanParams& p) {
  if (dpad % 32 != 0) return false;
  auto up = [](int x, int a) { return (x + a - 1) / a * a; };
  const int qc = 96;
  p.type = MV_IVF_FLAT;
  p.k = k;
  p.dpad = dpad;
  p.nchunks = dpad / 32;
  p.qchunk = qc;
  p.qchunk_split = qc / 2;
  p.ncol = 128;
  p.tmem_cols = 512;
  p.q_bytes = p.nchunks * qc * 128;
  p.meta_bytes = up(32 + kQmMetaPerQuery * qc, 16);
  p.off_q = 0;
  p.off_x = 2 * p.q_bytes;
  const int fixed_tail = kQmNTS * kQmSide + 2 * p.meta_bytes + 256 + 1024;
  const int budget = 227 * 1024;
  int ns = (budget - p.off_x - fixed_tail) / (128 * 128);
  ns = std::min(ns, 8);
  if (ns < 3) return false;
  p.nstage = ns;
  p.off_side = p.off_x + ns * 128 * 128;
  p.off_meta = p.off_side + kQmNTS * kQmSide;
  p.off_bar = up(p.off_meta + 2 * p.meta_bytes, 16);
  p.smem_total = p.off_bar + (2 * ns + 6 + 2 * kQmAcc + 2 * kQmNTS) * 8 + 16 + 1024;
  // the last chunk block of A1 reads 128 rows past its lo-plane start (row qc/2): inside the allocation
  return p.smem_total <= budget && p.off_q + 2 * p.q_bytes - qc * 128 + (qc / 2 + 128) * 128 <= p.off_bar;
}

cudaError_t launch_scan_qm(const CUtensorMap* xmap, const CUtensorMap* xmap16, const TcScanParams& p, cudaStream_t st) {
  cudaError_t e = cudaFuncSetAttribute(k_scan_qm, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_total);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = kNumSMs;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  k_scan_qm<<<nsm, kQmThreads, p.smem_total, st>>>(*xmap, *xmap16, p);
  return cudaGetLastError();
}

}  // namespace mv
