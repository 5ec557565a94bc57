// k_scan_tc.cu -- §8 rows a5 + a6 on the 5th-generation tensor cores (sm_100a).
//
// PAPER.md:529-532 (§3.1) step (2): scan the nprobe probed buckets with the fine quantizer;
// PAPER.md:916-922 (§4.1 B): the bitmap is checked for every encountered vector before the
// top-k; PAPER.md:590-596 (§3.2.1): per-worker heaps merged at the end.  PAPER.md:569-575: the
// loaded data vectors are reused for many queries -- here one 128-vector list tile in shared
// memory meets every query of that list's bucket in one tensor-core contraction.
//
// Work item = (list l, <= qchunk queries probing l).  Persistent CTA per SM, warp-specialised:
//   warp 0     TMA producer: list tiles (128 rows x one 128-B / 32-B swizzle atom per stage)
//   warp 1     TMEM owner + single-thread tcgen05.mma issuer
//              D[128 vectors x N] (+)= X_tile[128 x K] . Qplanes[N x K]^T, N = P x roundup16(nq)
//   warps 2-3  query gatherer: the bucket's query planes -> swizzled K-major smem (double buffer)
//   warps 4-7  epilogue: tcgen05.ld (row per thread) -> distance -> bitset -> transposed keys in
//              smem -> one warp per query filters against its running k-th best (and the global
//              per-query threshold tau) and inserts survivors (a6).
// FLAT (kind::tf32): X = fp32 payload used as tf32 -- exact when the stored values are
//   tf32-representable (integer SIFT data; the index checks this at add time); the query is
//   split into hi + lo tf32 planes (P = 2), so the query side is exact to ~2^-22.
// SQ8 (kind::i8): X = u8 codes straight from HBM; the query-side weights w_j = q_j * vdiff_j/255
//   are expanded into P = 3 signed 8-bit digit planes with a per-query scale, so
//   q.x_hat = q.a + s (D0 + D1/2^7 + D2/2^14) with int32-exact partials; no decode instructions.
#include "mv_internal.cuh"
#include "sm100.cuh"

namespace mv {
using namespace sm100;

__device__ __forceinline__ void named_bar(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }

// CTA-0 event timeline for MV_SCAN_TRACE (row r holds up to 1024 clock64 stamps)
#define MV_TRACE(row, idx)                                                                      \
  do {                                                                                        \
    if (p.prof && blockIdx.x == 0 && (idx) < 1024) p.prof[(row) * 1024 + (idx)] = clock64();  \
  } while (0)

struct WorkInfo {
  int l, bstart, nqc, len, ntiles;
  int64_t lstart;
};

__device__ __forceinline__ WorkInfo work_info(const TcScanParams& p, int w) {
  WorkInfo wi;
  const int2 it = p.witems[w];
  wi.l = it.x;
  wi.bstart = it.y;
  wi.nqc = min(p.qchunk, p.boff[wi.l + 1] - wi.bstart);
  wi.lstart = p.list_off[wi.l];
  wi.len = (int)(p.list_off[wi.l + 1] - wi.lstart);
  wi.ntiles = (wi.len + 127) >> 7;
  return wi;
}

constexpr int kNTS = 4;          // per-tile side-data ring slots
// side slot: norms f64 [1152 B] | rank u32 [640 B] | ids i64 [1152 B]; each copied as the 16-B aligned
// superset of the tile's 128 rows (the arrays are padded at allocation so the copy stays in bounds)
constexpr int kSideBytes = 3072;
constexpr int kSideRank = 1152, kSideIds = 1792;
constexpr int kEpiWarps = 8;      // two epilogue warps per TMEM lane quarter
constexpr int kThreads = 128 + 32 * kEpiWarps;
constexpr int kDLD = 129;         // padded transpose stride (conflict-free row and column access)

template <int TYPE>
__global__ void __launch_bounds__(kThreads, 1) k_scan_tc(const __grid_constant__ CUtensorMap xmap, const TcScanParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  constexpr int ESZ = TYPE == MV_IVF_FLAT ? 4 : 1;
  constexpr int ATOM = TYPE == MV_IVF_FLAT ? 128 : 32;
  constexpr int P = TYPE == MV_IVF_FLAT ? 2 : 4;
  const int nstage = p.nstage, nchunks = p.nchunks, QC = p.qchunk, k = p.k;
  const int rowbytes = p.dpad * ESZ;
  const bool use_norms = p.metric == MV_L2;
  const bool use_ids = p.bitset != nullptr;

  uint8_t* Xs = sm + p.off_x;
  uint8_t* Qs = sm + p.off_q;
  uint32_t* Dt = reinterpret_cast<uint32_t*>(sm + p.off_dt);
  uint64_t* lists = reinterpret_cast<uint64_t*>(sm + p.off_lists);
  uint8_t* metab = sm + p.off_meta;
  int32_t* ecnt = reinterpret_cast<int32_t*>(sm + p.off_misc);
  uint64_t* scratch = reinterpret_cast<uint64_t*>(sm + p.off_misc + 256);  // 32 per epilogue warp
  uint64_t* cbuf = scratch + 32 * kEpiWarps;                               // QC x 32 (k <= 32)
  int* cnb = reinterpret_cast<int*>(cbuf + 32 * QC);                       // QC counts
  uint32_t* cbnd = reinterpret_cast<uint32_t*>(cnb + QC);                  // QC running bounds
  int* selctr = reinterpret_cast<int*>(sm + p.off_ctr);                    // per-tile slot dispenser
  uint8_t* side = sm + p.off_side;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + p.off_bar);
  uint64_t* full_x = bars;
  uint64_t* empty_x = bars + nstage;
  uint64_t* full_q = empty_x + nstage;
  uint64_t* empty_q = full_q + 2;
  uint64_t* empty_m = empty_q + 2;
  uint64_t* tfull = empty_m + 2;
  uint64_t* tempty = tfull + 2;
  uint64_t* full_t = tempty + 2;
  uint64_t* empty_t = full_t + kNTS;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(empty_t + kNTS);

  // metadata per Q buffer: pair[QC] i32 | qs[QC] f32 | (8-B aligned) lim[QC] u64 | qn[QC] f64 | qa[QC] f64
  auto m_pair = [&](int b) { return reinterpret_cast<int32_t*>(metab + b * p.meta_bytes); };
  auto m_qs = [&](int b) { return reinterpret_cast<float*>(metab + b * p.meta_bytes) + QC; };
  auto m_lim = [&](int b) { return reinterpret_cast<uint64_t*>(metab + b * p.meta_bytes + p.meta_lim_off); };
  auto m_qn = [&](int b) { return reinterpret_cast<double*>(metab + b * p.meta_bytes + p.meta_lim_off) + QC; };
  auto m_qa = [&](int b) { return reinterpret_cast<double*>(metab + b * p.meta_bytes + p.meta_lim_off) + 2 * QC; };

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < nstage; ++s) {
      mbar_init(&full_x[s], 1);
      mbar_init(&empty_x[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&full_q[b], 64);
      mbar_init(&empty_q[b], 1);
      mbar_init(&empty_m[b], kEpiWarps);
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], kEpiWarps);
    }
    for (int s = 0; s < kNTS; ++s) {
      mbar_init(&full_t[s], 1);
      mbar_init(&empty_t[s], kEpiWarps);
    }
    fence_mbar_init();
  }
  if (warp == 1) {
    tmem_alloc(tslot, p.tmem_cols);
    tmem_relinquish();
  }
  if (warp == 0 && lane == 0) tma_prefetch(&xmap);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tslot;
  const int nwork = *p.nwitems;
  unsigned long long gt0 = 0;
  if (p.prof) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt0));

  if (warp == 0) {
    // ------------------------------------------------------------------ TMA producer
    if (lane == 0) {
      uint32_t it = 0, tcount = 0;
      const uint32_t side_tx = 528 + (use_norms ? 1040 : 0) + (use_ids ? 1040 : 0);
      for (int w = blockIdx.x; w < nwork; w += gridDim.x) {
        const WorkInfo wi = work_info(p, w);
        for (int t = 0; t < wi.ntiles; ++t, ++tcount) {
          const int row0 = (int)(wi.lstart + t * 128);
          const uint32_t ts = tcount % kNTS, tr = tcount / kNTS;
          mbar_wait(&empty_t[ts], (tr & 1) ^ 1);
          mbar_expect_tx(&full_t[ts], side_tx);
          uint8_t* sd = side + ts * kSideBytes;
          bulk_g2s(sd + kSideRank, p.rank + (row0 & ~3), 528, &full_t[ts]);
          if (use_norms) bulk_g2s(sd, p.norms + (row0 & ~1), 1040, &full_t[ts]);
          if (use_ids) bulk_g2s(sd + kSideIds, p.ids + (row0 & ~1), 1040, &full_t[ts]);
          for (int c = 0; c < nchunks; ++c, ++it) {
            const uint32_t s = it % nstage, r = it / nstage;
            mbar_wait(&empty_x[s], (r & 1) ^ 1);
            MV_TRACE(0, it);
            mbar_expect_tx(&full_x[s], 128 * ATOM);
            tma_load_2d(Xs + s * 128 * ATOM, &xmap, &full_x[s], c * ATOM / ESZ, row0);
          }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------------ MMA issuer
    if (lane == 0) {
      uint32_t it = 0, titer = 0, wcount = 0;
      for (int w = blockIdx.x; w < nwork; w += gridDim.x, ++wcount) {
        const WorkInfo wi = work_info(p, w);
        const int NQ = (wi.nqc + 15) & ~15;
        const int N = P * NQ;
        const uint32_t idesc = TYPE == MV_IVF_FLAT ? idesc_tf32(N) : idesc_u8s8(N);
        const uint32_t b = wcount & 1;
        mbar_wait(&full_q[b], (wcount >> 1) & 1);
        MV_TRACE(1, wcount);
        tc_fence_after();
        const uint32_t qbase = smem_u32(Qs + b * p.q_bytes);
        for (int t = 0; t < wi.ntiles; ++t, ++titer) {
          const uint32_t a = titer & 1;
          mbar_wait(&tempty[a], ((titer >> 1) & 1) ^ 1);
          MV_TRACE(2, titer);
          tc_fence_after();
          const uint32_t dcol = tmem + a * p.ncol;
          for (int c = 0; c < nchunks; ++c, ++it) {
            const uint32_t s = it % nstage;
            mbar_wait(&full_x[s], (it / nstage) & 1);
            tc_fence_after();
            const uint32_t xb = smem_u32(Xs + s * 128 * ATOM);
            const uint32_t qb = qbase + c * N * ATOM;
#pragma unroll
            for (int ks = 0; ks < ATOM / 32; ++ks) {
              const uint64_t ad = kmajor_desc(xb + ks * 32, ATOM);
              const uint64_t bd = kmajor_desc(qb + ks * 32, ATOM);
              if (TYPE == MV_IVF_FLAT) mma_tf32(dcol, ad, bd, idesc, (c | ks) != 0);
              else mma_i8(dcol, ad, bd, idesc, (c | ks) != 0);
            }
            mma_commit(&empty_x[s]);
          }
          mma_commit(&tfull[a]);
          MV_TRACE(3, titer);
        }
        mma_commit(&empty_q[b]);
      }
    }
  } else if (warp < 4) {
    // ------------------------------------------------------------------ query gatherer (64 thr)
    const int tq = threadIdx.x - 64;
    uint32_t wcount = 0;
    for (int w = blockIdx.x; w < nwork; w += gridDim.x, ++wcount) {
      const WorkInfo wi = work_info(p, w);
      const int NQ = (wi.nqc + 15) & ~15;
      const int N = P * NQ;
      const uint32_t b = wcount & 1, r = wcount >> 1;
      mbar_wait(&empty_q[b], (r & 1) ^ 1);
      mbar_wait(&empty_m[b], (r & 1) ^ 1);
      int32_t* mp = m_pair(b);
      for (int i = tq; i < wi.nqc; i += 64) {
        const int pr = p.bq[wi.bstart + i];
        const int q = pr / p.npb;
        mp[i] = pr;
        m_qn(b)[i] = p.qnorm[q];
        m_qs(b)[i] = TYPE == MV_IVF_SQ8 ? p.qscale[q] : 1.0f;
        m_qa(b)[i] = TYPE == MV_IVF_SQ8 ? p.qa[q] : 0.0;
        m_lim(b)[i] = p.tau[q];
      }
      named_bar(2, 64);
      uint8_t* Qb = Qs + b * p.q_bytes;
      constexpr int PIECES = ATOM / 16;
      const int total = (p.dbg & 4) ? 0 : wi.nqc * P * nchunks * PIECES;
      for (int idx = tq; idx < total; idx += 64) {
        const int pc = idx % PIECES;
        int rest = idx / PIECES;
        const int c = rest % nchunks;
        rest /= nchunks;
        const int pl = rest % P;
        const int i = rest / P;
        const int q = mp[i] / p.npb;
        const int64_t prow = TYPE == MV_IVF_FLAT ? (int64_t)pl * p.nq + q : (int64_t)q * P + pl;
        cp_async16(Qb + c * N * ATOM + swz_off(pl * NQ + i, pc, ATOM), p.qplanes + prow * rowbytes + c * ATOM + pc * 16);
      }
      cp_async_wait_all();
      fence_proxy_async();
      mbar_arrive(&full_q[b]);
    }
  } else {
    // ------------------------------------------------------------------ epilogue (8 warps)
    const int ew = warp - 4;            // 0..7
    const int quarter = warp & 3;       // TMEM lane quarter this warp may access
    const int half = ew >> 2;           // which 16-column chunks of the accumulator it reads
    const int row = quarter * 32 + lane;
    const int et = threadIdx.x - 128;   // 0..255
    uint64_t* wscr = scratch + ew * 32;
    uint32_t titer = 0, wcount = 0;
    for (int w = blockIdx.x; w < nwork; w += gridDim.x, ++wcount) {
      const WorkInfo wi = work_info(p, w);
      const int NQ = (wi.nqc + 15) & ~15;
      const uint32_t b = wcount & 1;
      mbar_wait(&full_q[b], (wcount >> 1) & 1);
      const int32_t* mp = m_pair(b);
      const double* qn = m_qn(b);
      const float* qs = m_qs(b);
      const double* qa = m_qa(b);
      const uint64_t* lim = m_lim(b);
      const bool sel = (k <= kLocalSelectMaxK) && (wi.len > k);
      if (sel) {
        for (int i = et; i < wi.nqc * k; i += 32 * kEpiWarps) lists[i] = MV_KEY_PAD;
        if (k <= 32)
          for (int i = et; i < wi.nqc; i += 32 * kEpiWarps) {
            cnb[i] = 0;
            cbnd[i] = 0xffffffffu;
          }
      } else {
        for (int i = et; i < wi.nqc; i += 32 * kEpiWarps) ecnt[i] = 0;
      }
      named_bar(1, 32 * kEpiWarps);
      for (int t = 0; t < wi.ntiles; ++t, ++titer) {
        const uint32_t a = titer & 1;
        const uint32_t ts = titer % kNTS;
        const int vrow = t * 128 + row;
        const int row0 = (int)(wi.lstart + t * 128);
        // refresh the global per-query threshold tau once per tile (other work items of the same
        // query keep tightening it); the load latency overlaps the wait for the accumulator
        uint64_t tau_now = MV_KEY_PAD;
        if (et < wi.nqc) tau_now = *reinterpret_cast<volatile const uint64_t*>(p.tau + mp[et] / p.npb);
        mbar_wait(&full_t[ts], (titer / kNTS) & 1);
        const uint8_t* sd = side + ts * kSideBytes;
        const uint32_t* srank = reinterpret_cast<const uint32_t*>(sd + kSideRank) + (row0 & 3);
        bool valid = vrow < wi.len;
        if (valid && use_ids)
          valid = !bit_excluded(p.bitset, p.nbits, reinterpret_cast<const int64_t*>(sd + kSideIds)[(row0 & 1) + row]);
        const double xn = use_norms ? reinterpret_cast<const double*>(sd)[(row0 & 1) + row] : 0.0;
        mbar_wait(&tfull[a], (titer >> 1) & 1);
        if (et == 0) MV_TRACE(6, titer);
        tc_fence_after();
        const uint32_t tbase = tmem + a * p.ncol + ((uint32_t)(quarter * 32) << 16);
        for (int qc = half * 16; qc < ((p.dbg & 2) ? 0 : NQ); qc += 32) {
          uint32_t r[P][16];
#pragma unroll
          for (int pl = 0; pl < P; ++pl) tmem_ld16(tbase + pl * NQ + qc, r[pl]);
          tmem_wait_ld();
#pragma unroll
          for (int j = 0; j < 16; ++j) {
            const int i = qc + j;
            if (i < wi.nqc) {
              float dist;
              if (TYPE == MV_IVF_FLAT) {
                // exact for tf32-representable data (the only FLAT data this path accepts)
                const float dot = __uint_as_float(r[0][j]) + __uint_as_float(r[1 % P][j]);
                dist = use_norms ? ((float)qn[i] + (float)xn) - 2.0f * dot : dot;
              } else {
                // int32-exact digit partials; the L2 expansion is combined in fp64 (the norms are
                // ~400x the near-neighbour distances on SIFT-scale data)
                const double acc = (double)(int)r[0][j] + (double)(int)r[1 % P][j] * (1.0 / 128.0) +
                                   (double)(int)r[2 % P][j] * (1.0 / 16384.0) +
                                   (double)(int)r[3 % P][j] * (1.0 / 2097152.0);
                const double dot = fma((double)qs[i], acc, qa[i]);
                dist = use_norms ? (float)((qn[i] + xn) - 2.0 * dot) : (float)dot;
              }
              Dt[i * kDLD + row] = valid ? dist_key(dist, p.metric) : 0xffffffffu;
            }
          }
        }
        if (et < wi.nqc && tau_now < lim[et]) const_cast<uint64_t*>(lim)[et] = tau_now;
        if (et == 0) *selctr = 0;
        tc_fence_before();
        if (et == 0) MV_TRACE(4, titer);
        __syncwarp();
        if (lane == 0) mbar_arrive(&tempty[a]);
        named_bar(1, 32 * kEpiWarps);
        if (et == 0) MV_TRACE(5, titer);
        // ---- a6: filter against min(list k-th, running bound, global tau) + select (warp per query)
        if (sel && k <= 32) {
          constexpr int G = 4;
          // query slots are handed out G at a time through a shared counter, so a warp stuck in a
          // warm-up or flush does not hold the others at the end-of-tile barrier
          for (;;) {
            int i0 = 0;
            if (lane == 0) i0 = atomicAdd(selctr, G);
            i0 = __shfl_sync(MV_FULL, i0, 0);
            if (i0 >= ((p.dbg & 1) ? 0 : wi.nqc)) break;
            const int nvalid = min(G, wi.nqc - i0);
            warp_filter_group<G>(
                nvalid, k, [&](int g, int m) { return Dt[(i0 + g) * kDLD + m * 32 + lane]; },
                [&](int g, uint64_t*& L, uint64_t*& B, int*& nb, uint32_t*& bnd, uint64_t& li) {
                  const int i = i0 + g;
                  L = lists + (int64_t)i * k;
                  B = cbuf + i * 32;
                  nb = cnb + i;
                  bnd = cbnd + i;
                  li = lim[i];
                },
                [&](int, int v) { return srank[v]; },
                [&](int g, uint32_t t32) {
                  atomicMin(reinterpret_cast<unsigned long long*>(p.tau + mp[i0 + g] / p.npb),
                            ((unsigned long long)t32 << 32) | 0xffffffffull);
                },
                wscr, (p.prof && (p.dbg & 64)) ? p.prof + 8 * 1024 + 1000 : nullptr, !(p.dbg & 32));
          }
        } else {
          for (int i = ew; i < ((p.dbg & 1) ? 0 : wi.nqc); i += kEpiWarps) {
            const int pr = mp[i];
            const uint64_t li = lim[i];
            uint32_t k32[4];
#pragma unroll
            for (int m = 0; m < 4; ++m) k32[m] = Dt[i * kDLD + m * 32 + lane];
            if (!sel) {
#pragma unroll
              for (int m = 0; m < 4; ++m) {
                const uint64_t key = ((uint64_t)k32[m] << 32) | srank[m * 32 + lane];
                const bool pass = k32[m] != 0xffffffffu && key < li;
                const uint32_t msk = __ballot_sync(MV_FULL, pass);
                const int base = ecnt[i];
                if (pass) p.part[p.poff[pr] + base + __popc(msk & ((1u << lane) - 1))] = key;
                __syncwarp();
                if (lane == 0) ecnt[i] = base + __popc(msk);
                __syncwarp();
              }
              continue;
            }
            warp_select_tile(lists + (int64_t)i * k, k, li, k32, [&](int v) { return srank[v]; }, wscr);
          }
        }
        named_bar(1, 32 * kEpiWarps);
        if (et == 0) MV_TRACE(7, titer);
        if (lane == 0) mbar_arrive(&empty_t[ts]);
      }
      // ---- finalize this work item's (query, list) partial results
      for (int i = ew; i < wi.nqc; i += kEpiWarps) {
        const int pr = mp[i];
        if (sel && k <= 32) {
          // the sorted list (<= k) followed by the unsorted survivor buffer (<= 32): the final select
          // merges them exactly, so no end-of-pair sort is needed
          const uint64_t* L = lists + (int64_t)i * k;
          const uint64_t v = lane < k ? L[lane] : MV_KEY_PAD;
          const uint32_t lm = __ballot_sync(MV_FULL, v != MV_KEY_PAD);
          const int nl = __popc(lm), n = cnb[i];
          if (v != MV_KEY_PAD) p.part[p.poff[pr] + __popc(lm & ((1u << lane) - 1))] = v;
          if (lane < n) p.part[p.poff[pr] + nl + lane] = cbuf[i * 32 + lane];
          if (lane == 0) {
            p.pcnt[pr] = nl + n;
            if (L[k - 1] != MV_KEY_PAD)
              atomicMin(reinterpret_cast<unsigned long long*>(p.tau + pr / p.npb), (unsigned long long)L[k - 1]);
          }
        } else if (sel) {
          const uint64_t* L = lists + (int64_t)i * k;
          int c = 0;
          for (int j0 = 0; j0 < k; j0 += 32) {
            const int j = j0 + lane;
            const uint64_t v = j < k ? L[j] : MV_KEY_PAD;
            if (v != MV_KEY_PAD) p.part[p.poff[pr] + j] = v;
            c += __popc(__ballot_sync(MV_FULL, v != MV_KEY_PAD));
          }
          if (lane == 0) {
            p.pcnt[pr] = c;
            if (L[k - 1] != MV_KEY_PAD)
              atomicMin(reinterpret_cast<unsigned long long*>(p.tau + pr / p.npb), (unsigned long long)L[k - 1]);
          }
        } else if (lane == 0) {
          p.pcnt[pr] = ecnt[i];
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty_m[b]);
      named_bar(1, 32 * kEpiWarps);
    }
  }
  __syncthreads();
  if (p.prof && threadIdx.x == 0) {  // per-CTA start / end (ns) in rows 8.. of the debug buffer
    unsigned long long gt1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt1));
    int ntl = 0;
    for (int w = blockIdx.x; w < nwork; w += gridDim.x) ntl += work_info(p, w).ntiles;
    p.prof[8 * 1024 + blockIdx.x * 3 + 0] = gt0;
    p.prof[8 * 1024 + blockIdx.x * 3 + 1] = gt1;
    p.prof[8 * 1024 + blockIdx.x * 3 + 2] = ntl;
  }
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem, p.tmem_cols);
  }
}

// ----------------------------------------------------------------------------------------------
// a1 for the tensor-core path: query planes.
//   FLAT: [hi, lo] tf32 planes (hi = q with the 13 low mantissa bits cleared, lo = q - hi)
//   SQ8 : w_j = q_j * b_j, b_j = vdiff_j / 255, a_j = vmin_j + 0.5 b_j; qa = q.a;
//         s = max|w| / 127; four int8 digits of w / s (base 2^7); qscale = s
// ----------------------------------------------------------------------------------------------
__global__ void k_qplanes(int type, const float* __restrict__ qpad, int64_t nq, int dpad, const float* __restrict__ vmin,
                          const float* __restrict__ vdiff, uint8_t* __restrict__ out, float* __restrict__ qscale,
                          double* __restrict__ qa, double* __restrict__ qnorm) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t q = warp; q < nq; q += nwarps) {
    const float* x = qpad + q * dpad;
    double nn = 0.0;
    for (int j = lane; j < dpad; j += 32) nn = fma((double)x[j], (double)x[j], nn);
    for (int o = 16; o > 0; o >>= 1) nn += __shfl_xor_sync(MV_FULL, nn, o);
    if (lane == 0) qnorm[q] = nn;
    if (type == MV_IVF_FLAT) {
      // FLAT planes are the plane-major hi/lo split made by launch_hilo (shared with the coarse step)
    } else {
      // fp64: w_j = q_j b_j, b_j = vdiff_j / 255, a_j = vmin_j + b_j / 2 (mid-bin decode)
      double amax = 0.0, dot = 0.0;
      for (int j = lane; j < dpad; j += 32) {
        const double bj = (double)vdiff[j] / 255.0;
        const double aj = fma(0.5, bj, (double)vmin[j]);
        dot = fma((double)x[j], aj, dot);
        amax = fmax(amax, fabs((double)x[j] * bj));
      }
      for (int o = 16; o > 0; o >>= 1) {
        amax = fmax(amax, __shfl_xor_sync(MV_FULL, amax, o));
        dot += __shfl_xor_sync(MV_FULL, dot, o);
      }
      // the scale is rounded up to fp32 first, so the digits and the epilogue use the same exact s
      const double s = amax > 0.0 ? (double)__double2float_ru(amax / 127.0) : 1.0;
      int8_t* o = reinterpret_cast<int8_t*>(out) + q * 4 * dpad;
      for (int j = lane; j < dpad; j += 32) {
        double u = (double)x[j] * ((double)vdiff[j] / 255.0) / s;  // in [-127, 127]
#pragma unroll
        for (int dgt = 0; dgt < 4; ++dgt) {  // base-2^7 signed digits: u ~ d0 + d1/2^7 + d2/2^14 + d3/2^21
          const double dd = fmin(fmax(rint(u), -127.0), 127.0);
          o[dgt * dpad + j] = (int8_t)dd;
          u = (u - dd) * 128.0;
        }
      }
      if (lane == 0) {
        qscale[q] = (float)s;
        qa[q] = dot;
      }
    }
  }
}

cudaError_t launch_qplanes(int type, const float* qpad, int64_t nq, int dpad, const float* vmin, const float* vdiff,
                           uint8_t* out, float* qscale, double* qa, double* qnorm, cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  const int grid = (int)min64(kNumSMs * 16, (nq * 32 + 255) / 256);
  k_qplanes<<<grid, 256, 0, st>>>(type, qpad, nq, dpad, vmin, vdiff, out, qscale, qa, qnorm);
  return cudaGetLastError();
}

// any stored fp32 value with low mantissa bits set (not exactly representable in tf32)?
__global__ void k_tf32_check(const uint32_t* __restrict__ x, int64_t n, int* flag) {
  bool bad = false;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    bad |= (x[i] & 0x1fffu) != 0;
  if (__syncthreads_or(bad) && threadIdx.x == 0) atomicOr(flag, 1);
}

cudaError_t launch_tf32_check(const float* x, int64_t n, int* flag, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  const int grid = (int)min64(kNumSMs * 8, (n + 255) / 256);
  k_tf32_check<<<grid, 256, 0, st>>>(reinterpret_cast<const uint32_t*>(x), n, flag);
  return cudaGetLastError();
}

// ----------------------------------------------------------------------------------------------
bool tc_scan_plan(int type, int dpad, int k, TcScanParams& p) {
  const int esz = type == MV_IVF_FLAT ? 4 : 1;
  const int atom = type == MV_IVF_FLAT ? 128 : 32;
  const int P = type == MV_IVF_FLAT ? 2 : 4;
  const int qcmax = type == MV_IVF_FLAT ? 48 : 64;
  p.type = type;
  p.dpad = dpad;
  p.k = k;
  p.nchunks = dpad * esz / atom;
  int qc = qcmax;
  if (k <= kLocalSelectMaxK) qc = std::max(1, std::min(qcmax, 53248 / (8 * k)));
  p.qchunk = qc;
  const int qcp = (qc + 15) & ~15;
  p.ncol = P * qcp;
  int cols = 32;
  while (cols < 2 * p.ncol) cols <<= 1;
  if (cols > 512) return false;
  p.tmem_cols = cols;
  auto up = [](int x, int a) { return (x + a - 1) / a * a; };
  p.q_bytes = up(P * qcp * dpad * esz, 1024);
  const int dt_bytes = qc * 129 * 4;
  const int lists_bytes = k <= kLocalSelectMaxK ? qc * k * 8 : 0;
  p.meta_lim_off = up(8 * qc, 8);
  p.meta_bytes = up(p.meta_lim_off + 24 * qc, 16);
  const int misc_bytes = 256 + 32 * 8 * kEpiWarps + (k <= 32 ? qc * (32 * 8 + 8) : 0);
  const int side_bytes = kNTS * kSideBytes;
  const int stage = 128 * atom;
  const int fixed = 2 * p.q_bytes + up(dt_bytes, 16) + up(lists_bytes, 16) + 2 * p.meta_bytes + misc_bytes + side_bytes;
  const int budget = 227 * 1024 - 1024 - 512;  // alignment slack + barriers
  int ns = (budget - fixed) / stage;
  ns = std::min(ns, type == MV_IVF_FLAT ? 8 : 24);
  if (ns < 2) return false;
  p.nstage = ns;
  p.off_x = 0;
  p.off_q = ns * stage;
  p.off_dt = p.off_q + 2 * p.q_bytes;
  p.off_lists = p.off_dt + up(dt_bytes, 16);
  p.off_meta = p.off_lists + up(lists_bytes, 16);
  p.off_misc = p.off_meta + 2 * p.meta_bytes;
  p.off_ctr = p.off_misc + misc_bytes;
  p.off_side = up(p.off_ctr + 16, 128);
  p.off_bar = p.off_side + side_bytes;
  p.smem_total = p.off_bar + (2 * ns + 10 + 2 * kNTS) * 8 + 16 + 1024;
  return p.smem_total <= 227 * 1024;
}

cudaError_t launch_scan_tc(const CUtensorMap* xmap, const TcScanParams& p, cudaStream_t st) {
  auto kern = p.type == MV_IVF_FLAT ? k_scan_tc<MV_IVF_FLAT> : k_scan_tc<MV_IVF_SQ8>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_total);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = kNumSMs;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  kern<<<nsm, kThreads, p.smem_total, st>>>(*xmap, p);
  return cudaGetLastError();
}

}  // namespace mv
