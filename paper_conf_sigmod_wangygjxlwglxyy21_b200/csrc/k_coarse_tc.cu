// k_coarse_tc.cu -- §8 rows a2 + a3: the queries x centroids contraction on the tensor cores and
// the per-query top-nprobe.
//
// PAPER.md:523-529 (§3.1) step (1): "find the closest nprobe buckets based on the distance between
// q and the centroid of each bucket"; PAPER.md:838-843 (§3.4): this step "has a much higher
// computation-to-I/O ratio than step 2 ... all the queries compare against the same K centroids".
//
// k_coarse_gemm: CTA = one block of NQB queries (B operand: tf32 hi/lo planes, loaded once by TMA)
// x a range of centroid tiles (A operand: 128 centroids, tf32 hi and lo planes, TMA ring).  Per
// K-step, into one accumulator: C_hi Q_hi^T + C_lo Q_hi^T (+ C_hi Q_lo^T when some query needs its
// lo plane), so q.c to ~2^-22 relative.  The epilogue (two warps per TMEM lane quarter; a warp's
// lanes are 32 consecutive centroids) scores s(q, c) = ||c||^2 - 2 q.c (L2) or -q.c (IP) and
//   pass 0: writes the minimum score key of each (query, 32-centroid group) to G (redux.sync);
//   pass 1: stores key = (score key << 32 | centroid) when (score key, group) <= gbound[q], else
//           padding, to the group's slots of the query's list.
// k_group_bound (warp per query): gbound[q] = the nprobe-th smallest (G, group id) pair, by an
// MSB bisection over the u32 keys and a ballot walk over the tied groups.  Exactly nprobe groups
// are at or below it and each holds a centroid scoring at most its key, so the nprobe best
// centroids all pass, and only centroids of those nprobe groups can (a passing centroid's group
// minimum is at or below it): each selected group owns 32 fixed slots of the query's list
// (gslot), so pass 1 stores without atomics.  Ties among equal scores go to the smaller centroid
// id, as in the oracle.
// k_probe_final (warp per query): pass 1 keeps every lane's R smallest appended keys, whose
// nprobe-th smallest bounds the answer; pass 2 streams the keys at or below it through a 32-entry
// staging buffer into a sorted register list.
//
// (Round 1 fused the selection into the GEMM epilogue and was latency-bound on the per-tile folds;
// round 1's final form wrote the score matrix S -- 2.6 GB per search on configs[4] -- and
// selected from it.  Two passes of the GEMM cost flops, which are cheap here, instead of bytes.)
#include "mv_internal.cuh"
#include "sm100.cuh"

namespace mv {
using namespace sm100;

namespace {
constexpr int kCEpiMax = 16;
constexpr int kCThreads = 64 + 32 * kCEpiMax;  // warp 0 TMA, warp 1 MMA, warps 2..1+nepi epilogue
}  // namespace

__global__ void __launch_bounds__(kCThreads, 1)
    k_coarse_gemm(const __grid_constant__ CUtensorMap cmap, const __grid_constant__ CUtensorMap qmap,
                  const CoarseParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  constexpr int ATOM = 128;            // tf32: 32 fp32 per 128-B swizzle atom row
  constexpr int ABYTES = 128 * ATOM;   // one 128-centroid chunk of one plane
  const int NQB = p.nqb, BROWS = 2 * NQB;  // hi rows then lo rows
  const int nchunks = p.nchunks, nstage = p.nstage;
  const int ntiles_all = (p.nlist + 127) >> 7;
  const int qb = blockIdx.x / p.csplit, cs = blockIdx.x % p.csplit;
  const int t0 = (int)((int64_t)ntiles_all * cs / p.csplit), t1 = (int)((int64_t)ntiles_all * (cs + 1) / p.csplit);
  const int q0 = qb * NQB;
  // tf32-exact queries (device flag): no lo plane, so the B buffer holds the hi rows of 2 NQB
  // queries and every MMA is N = 2 NQB wide -- half the centroid stream per query; the odd query
  // blocks' CTAs have nothing to do
  const bool wide = p.qlo_any != nullptr && *p.qlo_any == 0;
  if (wide && (qb & 1)) return;
  const int NQW = wide ? 2 * NQB : NQB;  // queries of this CTA

  uint8_t* Bs = sm;                                       // nchunks x BROWS x 128 B
  uint8_t* As = Bs + nchunks * BROWS * ATOM;              // nstage x (hi chunk, lo chunk)
  uint64_t* bars = reinterpret_cast<uint64_t*>(As + nstage * 2 * ABYTES);
  uint64_t* full_a = bars;
  uint64_t* empty_a = bars + nstage;
  uint64_t* full_b = empty_a + nstage;
  uint64_t* tfull = full_b + 1;
  uint64_t* tempty = tfull + 4;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(tempty + 4);
  const int nacc = p.nacc;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < nstage; ++s) {
      mbar_init(&full_a[s], 1);
      mbar_init(&empty_a[s], 1);
    }
    mbar_init(full_b, 1);
    for (int b = 0; b < nacc; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], p.nepi);
    }
    fence_mbar_init();
  }
  if (warp == 1) {
    tmem_alloc(tslot, p.tmem_cols);
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
      // (wide: the hi rows of [q0, q0 + 2 NQB))
      mbar_expect_tx(full_b, nchunks * BROWS * ATOM);
      for (int c = 0; c < nchunks; ++c) {
        tma_load_2d(Bs + c * BROWS * ATOM, &qmap, full_b, c * 32, q0);
        tma_load_2d(Bs + c * BROWS * ATOM + NQB * ATOM, &qmap, full_b, c * 32, wide ? q0 + NQB : (int)p.nq + q0);
      }
      uint32_t it = 0;
      for (int t = t0; t < t1; ++t)
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
      const uint32_t id_q = idesc_tf32(NQW);
      const bool qlo = !wide;  // C_hi . Q_lo vanishes for tf32-exact queries
      uint32_t it = 0;
      for (int t = t0, tl = 0; t < t1; ++t, ++tl) {
        const uint32_t a = tl % nacc;
        mbar_wait(&tempty[a], ((tl / nacc) & 1) ^ 1);
        tc_fence_after();
        const uint32_t d = tmem + a * NQW;
        for (int c = 0; c < nchunks; ++c, ++it) {
          const uint32_t s = it % nstage;
          mbar_wait(&full_a[s], (it / nstage) & 1);
          tc_fence_after();
          const uint32_t ah = smem_u32(As + s * 2 * ABYTES), al = ah + ABYTES;
          const uint32_t bh = smem_u32(Bs + c * BROWS * ATOM), bl = bh + NQB * ATOM;
#pragma unroll
          for (int ks = 0; ks < 4; ++ks) {
            // D += C_hi . Q_hi^T + C_lo . Q_hi^T (+ C_hi . Q_lo^T): q.c to ~2^-22, one accumulator
            mma_tf32(d, kmajor_desc(ah + ks * 32, ATOM), kmajor_desc(bh + ks * 32, ATOM), id_q, (c | ks) != 0);
            mma_tf32(d, kmajor_desc(al + ks * 32, ATOM), kmajor_desc(bh + ks * 32, ATOM), id_q, 1);
            if (qlo) mma_tf32(d, kmajor_desc(ah + ks * 32, ATOM), kmajor_desc(bl + ks * 32, ATOM), id_q, 1);
          }
          mma_commit(&empty_a[s]);
        }
        mma_commit(&tfull[a]);
      }
    }
  } else {
    // ------------------------------------------------------------------ epilogue
    const int ew = warp - 2;             // 0..nepi-1
    const int quarter = warp & 3;        // TMEM lane quarter this warp may read
    const int sub = ew >> 2, nsub = p.nepi >> 2;
    const int row = quarter * 32 + lane;  // centroid within the tile
    const int nqv = (int)min64(NQW, p.nq - q0);
    uint32_t* G = p.G + (int64_t)q0 * p.ldg;
    const bool l2 = p.metric == MV_L2;
    const int ngr = (p.nlist + 31) / 32;
    for (int t = t0, tl = 0; t < t1; ++t, ++tl) {
      const uint32_t a = tl % nacc;
      const int cid = t * 128 + row;
      const uint32_t grp = (uint32_t)(t * 4 + quarter);
      const bool valid = cid < p.nlist;
      const float cn = (valid && l2) ? __ldg(p.cnorm + cid) : 0.0f;
      mbar_wait(&tfull[a], (tl / nacc) & 1);
      tc_fence_after();
      const uint32_t tb = tmem + a * NQW + ((uint32_t)(quarter * 32) << 16);
      for (int qc = sub * 16; qc < NQW; qc += 16 * nsub) {
        uint32_t rd[16];
        tmem_ld16(tb + qc, rd);
        tmem_wait_ld();
        const int jn = min(16, nqv - qc);
        if (p.mode == 0) {
          // lane j keeps group minimum j; the G row stores go out as one instruction per chunk
          uint32_t gmine = 0xffffffffu;
#pragma unroll
          for (int j = 0; j < 16; ++j) {
            const float dot = __uint_as_float(rd[j]);
            const float sc = l2 ? cn - 2.0f * dot : -dot;
            const uint32_t gm = __reduce_min_sync(MV_FULL, valid ? f2key(sc) : 0xffffffffu);
            if (lane == j) gmine = gm;
          }
          if (lane < jn) G[(int64_t)(qc + lane) * p.ldg + grp] = gmine;
        } else {
          // keys and the pass test for the 16 columns; a column with a passing centroid belongs to
          // one of the query's nprobe groups: lane j fetches column j's slot (one load per chunk)
          uint32_t key[16], m[16], any = 0;
#pragma unroll
          for (int j = 0; j < 16; ++j) {
            const float dot = __uint_as_float(rd[j]);
            key[j] = f2key(l2 ? cn - 2.0f * dot : -dot);
            const uint64_t b = j < jn ? __ldg(p.gbound + q0 + qc + j) : 0ull;  // (L1-resident)
            const uint32_t bk = (uint32_t)(b >> 32);
            const bool pass = valid && j < jn && (key[j] < bk || (key[j] == bk && grp <= (uint32_t)b));
            m[j] = __ballot_sync(MV_FULL, pass);
            any |= (m[j] != 0u) << j;
          }
          if (any) {
            int sl = -1;
            if (lane < 16 && ((any >> lane) & 1)) sl = (int)__ldg(p.gslot + (q0 + qc + lane) * (int64_t)ngr + grp);
#pragma unroll
            for (int j = 0; j < 16; ++j) {
              if (!((any >> j) & 1)) continue;  // warp-uniform
              const int slj = __shfl_sync(MV_FULL, sl, j);
              const bool pass = (m[j] >> lane) & 1;
              const int64_t qq = q0 + qc + j;  // passing keys compacted, their count in ccnt
              if (pass) p.cand[qq * p.ccap + slj * 32 + __popc(m[j] & ((1u << lane) - 1))] = ((uint64_t)key[j] << 32) | (uint32_t)cid;
              if (lane == 0) p.ccnt[qq * p.nprobe + slj] = (uint8_t)__popc(m[j]);
            }
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[a]);
    }
  }
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem, p.tmem_cols);
  }
}

// dpad <= 128: the same two passes with the QUERIES on the MMA's M side.  CTA = 128 queries (A
// operand: hi [+ lo] planes resident in shared memory) x a range of 128-centroid tiles (B operand:
// centroid hi and lo planes streamed by TMA, 32 dims per stage).  D[128 q x 128 c] += Q_hi C_hi^T
// + Q_hi C_lo^T (+ Q_lo C_hi^T): the same products as k_coarse_gemm, one accumulator.  The
// epilogue owns one query per thread and one 32-centroid group per warp (16 epilogue warps, four
// per TMEM lane quarter): a group minimum is a register fminf chain over the thread's 32 columns --
// no cross-lane reduction -- and pass 1 touches a group's keys only when that minimum passes the
// thread's own bound (held in a register).  The centroid norms of each tile come in by bulk copy.
constexpr int kQmEpi = 16;
constexpr int kQmThreads = 64 + 32 * kQmEpi;
constexpr int kQmAcc = 2;      // TMEM accumulators of 128 columns
constexpr int kQmMaxStage = 8;  // centroid ring stages (3 next to hi+lo query planes at dpad 128, 5 next to hi only)

__global__ void __launch_bounds__(kQmThreads, 1)
    k_coarse_qm(const __grid_constant__ CUtensorMap cmap, const __grid_constant__ CUtensorMap qmap,
                const CoarseParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  constexpr int ATOM = 128;
  constexpr int PBYTES = 128 * ATOM;  // one 32-dim chunk of 128 rows of one plane
  const int nchunks = p.nchunks;
  const int ntiles_all = (p.nlist + 127) >> 7;
  const int qb = blockIdx.x / p.csplit, cs = blockIdx.x % p.csplit;
  const int t0 = (int)((int64_t)ntiles_all * cs / p.csplit), t1 = (int)((int64_t)ntiles_all * (cs + 1) / p.csplit);
  const int q0 = qb * 128;
  const bool qlo = p.qlo_any == nullptr || *p.qlo_any != 0;

  // layout: centroid norms, barriers, then the query planes and the centroid ring; without a lo
  // plane (tf32-exact queries, device flag) the ring takes its room: more stages in flight
  float* cns = reinterpret_cast<float*>(sm);  // kQmAcc x 128 centroid norms (1 KB)
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + 1024);  // (<= 1 KB)
  uint8_t* Aq = sm + 2048;                      // [qlo ? 2 : 1 planes][nchunks][128 rows][128 B]
  uint8_t* Bs = Aq + (qlo ? 2 : 1) * nchunks * PBYTES;  // nstage x (hi chunk, lo chunk)
  // (p.smem_total includes 1 KB of alignment slack for the 1 KB-aligned base)
  const int nstage = min(kQmMaxStage, (p.smem_total - 1024 - 2048 - (qlo ? 2 : 1) * nchunks * PBYTES) / (2 * PBYTES));
  uint64_t* full_a = bars;
  uint64_t* full_b = full_a + 1;
  uint64_t* empty_b = full_b + kQmMaxStage;
  uint64_t* tfull = empty_b + kQmMaxStage;
  uint64_t* tempty = tfull + kQmAcc;
  uint64_t* full_c = tempty + kQmAcc;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(full_c + kQmAcc);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    mbar_init(full_a, 1);
    for (int s = 0; s < nstage; ++s) {
      mbar_init(&full_b[s], 1);
      mbar_init(&empty_b[s], 1);
    }
    for (int a = 0; a < kQmAcc; ++a) {
      mbar_init(&tfull[a], 1);
      mbar_init(&tempty[a], kQmEpi);
      mbar_init(&full_c[a], 1);
    }
    fence_mbar_init();
  }
  if (warp == 1) {
    tmem_alloc(tslot, 128 * kQmAcc);
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
      // the query block: hi rows [q0, q0+128) (and lo rows [nq + q0, ...)) of the plane-major matrix
      mbar_expect_tx(full_a, (qlo ? 2 : 1) * nchunks * PBYTES);
      for (int pl = 0; pl < (qlo ? 2 : 1); ++pl)
        for (int c = 0; c < nchunks; ++c)
          tma_load_2d(Aq + (pl * nchunks + c) * PBYTES, &qmap, full_a, c * 32, pl * (int)p.nq + q0);
      uint32_t s = 0, sph = 0, a = 0, aph = 0;
      for (int t = t0; t < t1; ++t) {
        // the tile's centroid norms, once the epilogue is done with the slot's previous tile
        mbar_wait(&tempty[a], aph ^ 1);
        mbar_expect_tx(&full_c[a], 512);
        bulk_g2s(cns + a * 128, p.cnorm + (int64_t)t * 128, 512, &full_c[a]);
        if (++a == (uint32_t)kQmAcc) {
          a = 0;
          aph ^= 1;
        }
        for (int c = 0; c < nchunks; ++c) {
          mbar_wait(&empty_b[s], sph ^ 1);
          mbar_expect_tx(&full_b[s], 2 * PBYTES);
          tma_load_2d(Bs + s * 2 * PBYTES, &cmap, &full_b[s], c * 32, t * 128);
          tma_load_2d(Bs + s * 2 * PBYTES + PBYTES, &cmap, &full_b[s], c * 32, p.nlist + t * 128);
          if (++s == (uint32_t)nstage) {
            s = 0;
            sph ^= 1;
          }
        }
      }
    }
  } else if (warp == 1) {
    // the whole warp runs the loop, one elected lane issues (k_scan_tc.cu: no per-MMA R2UR elect
    // loops, no divisions for the ring positions)
    {
      mbar_wait(full_a, 0);
      tc_fence_after();
      const uint32_t id = idesc_tf32(128);
      uint32_t s = 0, sph = 0, a = 0, aph = 0;
      for (int t = t0; t < t1; ++t) {
        mbar_wait(&tempty[a], aph ^ 1);
        tc_fence_after();
        const uint32_t d = tmem + a * 128;
        for (int c = 0; c < nchunks; ++c) {
          mbar_wait(&full_b[s], sph);
          tc_fence_after();
          const uint32_t qh = smem_u32(Aq + c * PBYTES), ql = smem_u32(Aq + (nchunks + c) * PBYTES);
          const uint32_t ch = smem_u32(Bs + s * 2 * PBYTES), cl = ch + PBYTES;
#pragma unroll
          for (int ks = 0; ks < 4; ++ks) {
            mma_tf32_elect(d, kmajor_desc(qh + ks * 32, ATOM), kmajor_desc(ch + ks * 32, ATOM), id, (c | ks) != 0);
            mma_tf32_elect(d, kmajor_desc(qh + ks * 32, ATOM), kmajor_desc(cl + ks * 32, ATOM), id, 1);
            if (qlo) mma_tf32_elect(d, kmajor_desc(ql + ks * 32, ATOM), kmajor_desc(ch + ks * 32, ATOM), id, 1);
          }
          mma_commit_elect(&empty_b[s]);
          if (++s == (uint32_t)nstage) {
            s = 0;
            sph ^= 1;
          }
        }
        mma_commit_elect(&tfull[a]);
        if (++a == (uint32_t)kQmAcc) {
          a = 0;
          aph ^= 1;
        }
      }
    }
  } else {
    // ------------------------------------------------------------------ epilogue
    const int ew = warp - 2;           // 0..15
    const int quarter = warp & 3;      // TMEM lane quarter: queries quarter*32 .. +31
    const int gsub = ew >> 2;          // this warp's group within the tile (columns 32 gsub .. +31)
    const int64_t q = q0 + quarter * 32 + lane;
    const bool vq = q < p.nq;
    const bool l2 = p.metric == MV_L2;
    const int ngr = (p.nlist + 31) / 32;
    const uint64_t bq = (p.mode == 1 && vq) ? __ldg(p.gbound + q) : 0ull;
    const uint32_t bk = (uint32_t)(bq >> 32), bg = (uint32_t)bq;
    for (int t = t0, tl = 0; t < t1; ++t, ++tl) {
      const uint32_t a = tl % kQmAcc;
      const uint32_t grp = (uint32_t)(t * 4 + gsub);
      const int c0 = t * 128 + gsub * 32;  // first centroid of the group
      mbar_wait(&full_c[a], (tl / kQmAcc) & 1);
      mbar_wait(&tfull[a], (tl / kQmAcc) & 1);
      tc_fence_after();
      uint32_t rd[32];
      tmem_ld32(tmem + a * 128 + gsub * 32 + ((uint32_t)(quarter * 32) << 16), rd);
      tmem_wait_ld();
      const float4* cn4 = reinterpret_cast<const float4*>(cns + a * 128 + gsub * 32);
      float sc[32];
      float mn = __int_as_float(0x7f800000);
#pragma unroll
      for (int v = 0; v < 8; ++v) {
        const float4 cv = cn4[v];
        const float cvv[4] = {cv.x, cv.y, cv.z, cv.w};
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int j = 4 * v + u;
          const float dot = __uint_as_float(rd[j]);
          sc[j] = c0 + j < p.nlist ? (l2 ? cvv[u] - 2.0f * dot : -dot) : __int_as_float(0x7f800000);
          mn = fminf(mn, sc[j]);
        }
      }
      const uint32_t kmin = f2key(mn);
      if (p.mode == 0) {
        if (vq && grp < (uint32_t)ngr) p.G[q * p.ldg + grp] = kmin;
      } else if (vq && grp < (uint32_t)ngr && (kmin < bk || (kmin == bk && grp <= bg))) {
        // one of the query's nprobe groups: its 32 keys (padding above the bound) to the group's slots
        // (compacted: the passing keys first, their count in ccnt)
        const int sl = (int)__ldg(p.gslot + q * (int64_t)ngr + grp);
        uint64_t* dst = p.cand + q * (int64_t)p.ccap + sl * 32;
        int n = 0;
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          const uint32_t kj = f2key(sc[j]);
          if (c0 + j < p.nlist && (kj < bk || (kj == bk && grp <= bg))) dst[n++] = ((uint64_t)kj << 32) | (uint32_t)(c0 + j);
        }
        p.ccnt[q * (int64_t)p.nprobe + sl] = (uint8_t)n;
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[a]);
    }
  }
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem, 128 * kQmAcc);
  }
}

// gbound[q] = the nprobe-th smallest (group minimum key, group id) of the query's G row, and
// gslot[q][g] = the rank (in group order) of group g among the nprobe groups at or below it, -1
// for the others: pass 1 writes a selected group's 32 keys to slots [32 rank, 32 rank + 32) of
// the query's candidate list -- no atomics.  One warp per query; a row of <= 32 kReg groups
// lives in registers (group i * 32 + lane in v[i]), longer rows are re-read from L1/L2.
constexpr int kReg = 64;

template <int NRT>  // values per lane held in registers (0: re-read from L1/L2)
__global__ void __launch_bounds__(256) k_group_bound(const uint32_t* __restrict__ G, int64_t ldg, int ng, int64_t nq,
                                                     int nprobe, uint64_t* __restrict__ gbound,
                                                     int16_t* __restrict__ gslot) {
  const int lane = threadIdx.x & 31;
  const int64_t q = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (q >= nq) return;
  const uint32_t* g = G + q * ldg;
  const uint32_t ltmask = (1u << lane) - 1;
  constexpr bool REG = NRT > 0;
  constexpr int NR = REG ? NRT : 1;
  uint32_t v[NR];
#pragma unroll
  for (int i = 0; i < NR; ++i) v[i] = (REG && i * 32 + lane < ng) ? g[i * 32 + lane] : 0xffffffffu;
  auto val = [&](int i) -> uint32_t {  // group i * 32 + lane (REG: i is a compile-time index)
    if (REG) {
      uint32_t x = 0xffffffffu;
#pragma unroll
      for (int j = 0; j < NR; ++j)
        if (j == i) x = v[j];
      return x;
    }
    return i * 32 + lane < ng ? __ldg(g + i * 32 + lane) : 0xffffffffu;
  };
  const int nrow = (ng + 31) / 32;
  auto count_below = [&](uint32_t trial) {  // groups with key < trial
    int c = 0;
    if (REG) {
#pragma unroll
      for (int i = 0; i < NR; ++i) c += v[i] < trial;
    } else {
      for (int i = 0; i < nrow; ++i) c += val(i) < trial;
    }
    return (int)__reduce_add_sync(MV_FULL, (uint32_t)c);
  };
  // the nprobe-th smallest key b: the largest b with count(< b) < nprobe.  The bisection starts
  // below the bits every group key shares (the row's min and max agree above them: b lies in
  // [min, max], so its higher bits are those of min)
  uint32_t mn = 0xffffffffu, mx = 0;
  if (REG) {
#pragma unroll
    for (int i = 0; i < NR; ++i)
      if (i * 32 + lane < ng) {
        mn = min(mn, v[i]);
        mx = max(mx, v[i]);
      }
  } else {
    for (int i = 0; i < nrow; ++i)
      if (i * 32 + lane < ng) {
        const uint32_t x = val(i);
        mn = min(mn, x);
        mx = max(mx, x);
      }
  }
  mn = __reduce_min_sync(MV_FULL, mn);
  mx = __reduce_max_sync(MV_FULL, mx);
  // (fewer groups than nprobe: every group is selected, b = the full 32-bit search's 0xffffffff)
  const int top = ng < nprobe ? 31 : (mn == mx ? -1 : 31 - __clz((int)(mn ^ mx)));  // highest differing bit
  uint32_t b = top >= 31 ? 0u : (mn >> (top + 1)) << (top + 1);
  for (int bit = top; bit >= 0; --bit) {
    const uint32_t trial = b | (1u << bit);
    if (count_below(trial) < nprobe) b = trial;
  }
  if (top < 0) b = mn;  // every group key equal (and ng >= nprobe)
  // among the groups with key == b (group order), the (nprobe - count(< b))-th; then the ranks
  int r = nprobe - count_below(b);
  uint32_t gsel = 0xffffffffu;
  int base = 0;
#pragma unroll
  for (int i = 0; i < (REG ? NR : 1); ++i) {
    for (int ii = REG ? i : 0; ii < (REG ? i + 1 : nrow); ++ii) {
      const uint32_t x = val(ii);
      const int gid = ii * 32 + lane;
      const uint32_t tie = __ballot_sync(MV_FULL, gid < ng && x == b);
      if (gsel == 0xffffffffu && tie) {
        const int c = __popc(tie);
        if (c >= r) {
          uint32_t mm = tie;
          for (int t = 1; t < r; ++t) mm &= mm - 1;
          gsel = (uint32_t)(ii * 32 + __ffs(mm) - 1);
        } else {
          r -= c;
        }
      }
      // selected: key < b, or key == b up to the chosen tied group (gsel is final once set, and
      // every tied group before it in group order has been seen)
      const bool sel = gid < ng && (x < b || (x == b && (gsel == 0xffffffffu || (uint32_t)gid <= gsel)));
      const uint32_t m = __ballot_sync(MV_FULL, sel);
      if (gid < ng) gslot[q * ng + gid] = sel ? (int16_t)(base + __popc(m & ltmask)) : (int16_t)-1;
      base += __popc(m);
    }
  }
  if (lane == 0) gbound[q] = ((uint64_t)b << 32) | gsel;
}

// per-query top-nprobe of the appended candidates (R = ceil(nprobe / 32)); see the file comment
template <int R>
__global__ void __launch_bounds__(256) k_probe_final(const uint64_t* __restrict__ cand, const uint8_t* __restrict__ ccnt,
                                                     int ccap, int64_t nq, int nprobe, int32_t* __restrict__ probes) {
  __shared__ uint64_t stage_all[8][64];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int64_t q = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (q >= nq) return;
  uint64_t* stage = stage_all[wib];
  const uint64_t* c = cand + q * ccap;
  const uint8_t* cn = ccnt + q * nprobe;
  // every key of the query: lane l walks slots l, l + 32, ... (each slot's keys are compacted)
  auto for_each_key = [&](auto&& f) {
    for (int s0 = 0; s0 < nprobe; s0 += 32) {
      const int sl = s0 + lane;
      const int n = sl < nprobe ? cn[sl] : 0;
      const int nmax = __reduce_max_sync(MV_FULL, (uint32_t)n);
      for (int i = 0; i < nmax; ++i) f(i < n ? c[sl * 32 + i] : MV_KEY_PAD);
    }
  };
  uint64_t t[R];
#pragma unroll
  for (int r = 0; r < R; ++r) t[r] = MV_KEY_PAD;
  for_each_key([&](uint64_t key) {
    if (key < t[R - 1]) {
      t[R - 1] = key;
#pragma unroll
      for (int r = R - 1; r > 0; --r)
        if (t[r] < t[r - 1]) {
          const uint64_t x = t[r];
          t[r] = t[r - 1];
          t[r - 1] = x;
        }
    }
  });
  warp_bitonic_sort<R>(t);
  uint64_t bsel = t[0];
#pragma unroll
  for (int r = 1; r < R; ++r)
    if (r == ((nprobe - 1) >> 5)) bsel = t[r];
  const uint64_t bound = shfl64(bsel, (nprobe - 1) & 31);
  uint64_t L[R];
#pragma unroll
  for (int r = 0; r < R; ++r) L[r] = MV_KEY_PAD;
  int ns = 0;
  auto flush32 = [&]() {
    uint64_t cc[R];
    uint64_t c1[1] = {lane < ns ? stage[lane] : MV_KEY_PAD};
    warp_bitonic_sort<1>(c1);
    cc[0] = c1[0];
#pragma unroll
    for (int r = 1; r < R; ++r) cc[r] = MV_KEY_PAD;
    warp_merge_smallest<R>(L, cc);
    const int rest = ns > 32 ? ns - 32 : 0;
    const uint64_t mv = lane < rest ? stage[32 + lane] : 0;
    __syncwarp();
    if (lane < rest) stage[lane] = mv;
    __syncwarp();
    ns = rest;
  };
  for_each_key([&](uint64_t key) {
    const bool ps = key != MV_KEY_PAD && key <= bound;
    const uint32_t bm = __ballot_sync(MV_FULL, ps);
    if (ps) stage[ns + __popc(bm & ((1u << lane) - 1))] = key;
    ns += __popc(bm);
    __syncwarp();
    if (ns >= 32) flush32();
  });
  if (ns > 0) flush32();
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const int i = r * 32 + lane;
    if (i < nprobe) probes[q * nprobe + i] = (int32_t)(uint32_t)(L[r] & 0xffffffffu);
  }
}

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

// Plan: the query-block size NQB (multiple of 16, <= 128) and centroid split that minimise
// (waves x per-CTA work) on nsm SMs, with >= 2 centroid stages in shared memory.
bool coarse_tc_plan(int dpad, int nprobe, int64_t nq, int nlist, int nsm, const Options& o, CoarseParams& p) {
  if (dpad % 32 != 0 || nprobe > 1024) return false;
  if (dpad <= 128 && o.coarse_nqb == 0) {
    // queries on the M side (k_coarse_qm): 128 queries per CTA; centroid splits fill the SMs
    p.qm = 1;
    p.nchunks = dpad / 32;
    p.nprobe = nprobe;
    p.nqb = 128;
    const int ntiles = (nlist + 127) / 128;
    const int64_t blocks = (nq + 127) / 128;
    // centroid splits: minimise waves x (tiles per CTA + the query block's load, ~2 tiles of time)
    int64_t best = -1;
    for (int cs = 1; cs <= std::min(ntiles, 64); ++cs) {
      const int64_t waves = (blocks * cs + nsm - 1) / nsm;
      const int64_t cost = waves * ((ntiles + cs - 1) / cs + 2);
      if (best < 0 || cost < best) {
        best = cost;
        p.csplit = cs;
      }
    }
    if (o.coarse_cs > 0) p.csplit = std::max(1, std::min(ntiles, o.coarse_cs));
    // shared memory: 1 KB of norms + barriers, 1 KB alignment slack, the query planes and the ring
    // (the kernel derives the ring depth from p.smem_total and its query-plane count)
    p.smem_total = 227 * 1024;
    p.nstage = (p.smem_total - 3072 - 2 * p.nchunks * 128 * 128) / (2 * 128 * 128);  // (hi + lo queries)
    p.nepi = 16;
    p.nacc = kQmAcc;
    p.tmem_cols = 128 * kQmAcc;
    return p.nstage >= 2 && p.smem_total <= 227 * 1024;
  }
  p.qm = 0;
  p.nchunks = dpad / 32;
  p.nprobe = nprobe;
  const int budget = 227 * 1024 - 1024 - 256;  // alignment slack, barriers
  const int stage = 2 * 128 * 128;
  const int ntiles = (nlist + 127) / 128;
  int64_t best_cost = -1;
  for (int nqb = 32; nqb <= 128; nqb += 16) {
    const int fixed = p.nchunks * 2 * nqb * 128;
    if ((budget - fixed) / stage < 2) continue;
    const int64_t blocks = (nq + nqb - 1) / nqb;
    for (int cs = 1; cs <= std::min(8, ntiles); ++cs) {
      const int64_t units = blocks * cs;
      const int64_t waves = (units + nsm - 1) / nsm;
      // per-CTA: the query block load + its share of centroid tiles x (MMA/epilogue ~ nqb + stream)
      const int64_t cost = waves * (4 * p.nchunks + (int64_t)((ntiles + cs - 1) / cs) * (nqb + 48));
      if (best_cost < 0 || cost < best_cost) {
        best_cost = cost;
        p.nqb = nqb;
        p.csplit = cs;
      }
    }
  }
  if (best_cost < 0) return false;
  // tuning options (mv_index_set_option): they change the launch shape, never the result
  if (o.coarse_nqb > 0) p.nqb = std::max(32, std::min(128, o.coarse_nqb / 16 * 16));
  if (o.coarse_cs > 0) p.csplit = std::max(1, std::min(ntiles, o.coarse_cs));
  const int fixed = p.nchunks * 2 * p.nqb * 128;
  p.nstage = std::min(6, (budget - fixed) / stage);
  p.smem_total = fixed + p.nstage * stage + 256 + 1024;
  p.nepi = 8;
  p.nacc = 2;
  if (o.coarse_epi > 0) p.nepi = std::max(4, std::min(kCEpiMax, o.coarse_epi / 4 * 4));
  if (o.coarse_nacc > 0) p.nacc = std::max(1, std::min(4, o.coarse_nacc));
  while (p.nacc > 1 && p.nacc * 2 * p.nqb > 512) --p.nacc;  // (wide mode: 2 nqb columns per accumulator)
  int cols = 32;
  while (cols < p.nacc * 2 * p.nqb) cols <<= 1;
  p.tmem_cols = cols;
  return p.smem_total <= 227 * 1024;
}

cudaError_t launch_coarse_tc(const CUtensorMap* cmap, const CUtensorMap* qmap, const CoarseParams& p0, int64_t nq,
                             cudaStream_t st) {
  const unsigned grid = (unsigned)(((nq + p0.nqb - 1) / p0.nqb) * p0.csplit);
  auto kern = p0.qm ? k_coarse_qm : k_coarse_gemm;
  const int nthr = p0.qm ? kQmThreads : 64 + 32 * p0.nepi;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, p0.smem_total);
  if (e != cudaSuccess) return e;
  CoarseParams p = p0;
  p.mode = 0;  // pass 0: group minima
  kern<<<grid, nthr, p.smem_total, st>>>(*cmap, *qmap, p);
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  const unsigned gw = (unsigned)((nq * 32 + 255) / 256);
  const int ng = (p.nlist + 31) / 32;
  if (ng <= 64) k_group_bound<2><<<gw, 256, 0, st>>>(p.G, p.ldg, ng, nq, p.nprobe, p.gbound, p.gslot);
  else if (ng <= 128) k_group_bound<4><<<gw, 256, 0, st>>>(p.G, p.ldg, ng, nq, p.nprobe, p.gbound, p.gslot);
  else if (ng <= 256) k_group_bound<8><<<gw, 256, 0, st>>>(p.G, p.ldg, ng, nq, p.nprobe, p.gbound, p.gslot);
  else if (ng <= 512) k_group_bound<16><<<gw, 256, 0, st>>>(p.G, p.ldg, ng, nq, p.nprobe, p.gbound, p.gslot);
  else if (ng <= 1024) k_group_bound<32><<<gw, 256, 0, st>>>(p.G, p.ldg, ng, nq, p.nprobe, p.gbound, p.gslot);
  else if (ng <= 2048) k_group_bound<64><<<gw, 256, 0, st>>>(p.G, p.ldg, ng, nq, p.nprobe, p.gbound, p.gslot);
  else k_group_bound<0><<<gw, 256, 0, st>>>(p.G, p.ldg, ng, nq, p.nprobe, p.gbound, p.gslot);
  // fewer groups than probes: every group is selected and the slots past them stay padding
  if (ng < p.nprobe && (e = cudaMemsetAsync(p.ccnt, 0, (size_t)nq * p.nprobe, st)) != cudaSuccess) return e;
  p.mode = 1;  // pass 1: the same scores, the selected groups' keys stored to their slots
  kern<<<grid, nthr, p.smem_total, st>>>(*cmap, *qmap, p);
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  const int R = (p.nprobe + 31) / 32;
  if (R <= 1) k_probe_final<1><<<gw, 256, 0, st>>>(p.cand, p.ccnt, p.ccap, nq, p.nprobe, p.probes);
  else if (R == 2) k_probe_final<2><<<gw, 256, 0, st>>>(p.cand, p.ccnt, p.ccap, nq, p.nprobe, p.probes);
  else if (R <= 4) k_probe_final<4><<<gw, 256, 0, st>>>(p.cand, p.ccnt, p.ccap, nq, p.nprobe, p.probes);
  else if (R <= 8) k_probe_final<8><<<gw, 256, 0, st>>>(p.cand, p.ccnt, p.ccap, nq, p.nprobe, p.probes);
  else if (R <= 16) k_probe_final<16><<<gw, 256, 0, st>>>(p.cand, p.ccnt, p.ccap, nq, p.nprobe, p.probes);
  else k_probe_final<32><<<gw, 256, 0, st>>>(p.cand, p.ccnt, p.ccap, nq, p.nprobe, p.probes);
  return cudaGetLastError();
}

}  // namespace mv
