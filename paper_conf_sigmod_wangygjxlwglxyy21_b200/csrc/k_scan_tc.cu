// k_scan_tc.cu -- §8 rows a5 + a6 on the 5th-generation tensor cores (sm_100a).
//
// PAPER.md:529-532 (§3.1) step (2): scan the nprobe probed buckets with the fine quantizer;
// PAPER.md:916-922 (§4.1 B): the bitmap is checked for every encountered vector before the
// top-k.  PAPER.md:569-575 (§3.2.1): the loaded data vectors are reused for many queries -- here
// one 128-vector list tile in shared memory meets every query of that list's bucket in one
// tensor-core contraction.  PAPER.md:590-596: per-worker partial results merged at the end.
//
// Work item = (list l, <= qchunk queries probing l).  Persistent CTA per SM, warp-specialised:
//   warp 0     TMA producer: list tiles (128 rows x one 128-B (FLAT; SQ8 with 128-multiple rows) or
//              32-B (other SQ8) swizzle atom per stage) and
//              the tiles' side data (norms, id ranks, ids) by bulk copy
//   warp 1     TMEM owner + single-thread tcgen05.mma issuer
//              D[128 vectors x N] (+)= X_tile[128 x K] . Qplanes[N x K]^T, N = P x roundup16(nq)
//   warps 2-3  query gatherer: the bucket's query planes -> swizzled K-major smem, and the
//              per-query metadata (threshold, output region) -- both double-buffered
//   warps 4-15 epilogue, three warps per TMEM lane quarter: every thread owns one vector row and
//              a share of the query columns; tcgen05.ld -> distance -> bitset -> threshold test ->
//              survivors are appended to the (query, list) pair's output region (a6).
//
// a6 is a filter, not a selection.  The search runs the scan twice:
//   phase A (p.phase 0) scans a prefix (p.rowcap rows) of each query's rA nearest lists and emits
//     every candidate; a
//     per-query select (k_select.cu) turns them into tau_q = the k-th best key so far -- an exact
//     upper bound of the query's final k-th best;
//   phase B (p.phase 1) scans every probed pair and emits only keys <= tau_q.
// The final select takes the exact top-k of everything emitted.  No per-pair selection state,
// no epilogue-wide barrier per tile: the epilogue warps run independently.
//
// FLAT (kind::tf32): X = fp32 payload used as tf32 -- exact when the stored values are
//   tf32-representable (integer SIFT data; the index checks this at add time); the query is
//   split into hi + lo tf32 planes (P = 2), so the query side is exact to ~2^-22.
// SQ8 (kind::i8): X = u8 codes straight from HBM; the query-side weights w_j = q_j * vdiff_j/255
//   are expanded into P = 4 signed 8-bit digit planes with a per-query scale, so
//   q.x_hat = q.a + s (D0 + D1/2^7 + D2/2^14 + D3/2^21) with int32-exact partials; no decode.
#include "mv_internal.cuh"
#include "sm100.cuh"

namespace mv {
using namespace sm100;

__device__ __forceinline__ void named_bar(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }
template <int W>
__device__ __forceinline__ void tmem_ld_w(uint32_t taddr, uint32_t (&r)[W]) {
  if constexpr (W == 16) sm100::tmem_ld16(taddr, r);
  else sm100::tmem_ld8(taddr, r);
}
// shared-memory accesses through explicit 32-bit shared addresses (the metadata pointers are
// generic: every generic access to them costs an address-window conversion)
__device__ __forceinline__ float4 lds_f4(uint32_t a) {
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(a));
  return v;
}
__device__ __forceinline__ int64_t lds_s64(uint32_t a) {
  int64_t v;
  asm volatile("ld.shared.s64 %0, [%1];" : "=l"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ int atoms_add(uint32_t a, int v) {
  int old;
  asm volatile("atom.shared.add.u32 %0, [%1], %2;" : "=r"(old) : "r"(a), "r"(v));
  return old;
}
// predicated 8-B global store (no divergent branch around the emission)
__device__ __forceinline__ void st_u64_if(uint32_t pred, uint64_t* a, uint64_t v) {
  asm volatile("{\n .reg .pred q;\n setp.ne.u32 q, %0, 0;\n @q st.global.u64 [%1], %2;\n}" ::"r"(pred), "l"(a), "l"(v));
}
// f2key (mv_internal.cuh) in two integer ops
__device__ __forceinline__ uint32_t f2key_fast(float f) {
  const uint32_t b = __float_as_uint(__fadd_rn(f, 0.0f));
  return b ^ ((uint32_t)((int32_t)b >> 31) | 0x80000000u);
}

// CTA-0 event timeline (row r holds up to 1024 clock64 stamps): a development build option
// (-DMV_SCAN_TRACE), compiled out of the product library
#ifdef MV_SCAN_TRACE
#define MV_TRACE(row, idx)                                                                      \
  do {                                                                                        \
    if (p.prof && blockIdx.x == 0 && (idx) < 1024) p.prof[(row) * 1024 + (idx)] = clock64();  \
  } while (0)
#else
#define MV_TRACE(row, idx) \
  do {                     \
  } while (0)
#endif

struct WorkInfo {
  int l, bstart, nqc, len, ntiles;
  int multi;  // the list has sibling items (kItemMulti): its tiles are kept in L2 for them
  int64_t lstart;
};
static_assert(sizeof(WorkInfo) == 32, "the metadata header holds one WorkInfo");

__device__ __forceinline__ WorkInfo work_info_of(const TcScanParams& p, int2 it, int qchunk) {
  WorkInfo wi;
  wi.multi = it.x & kItemMulti;
  it.x &= ~kItemMulti;
  wi.l = it.x >= p.nlist ? it.x - p.nlist : it.x;
  wi.bstart = it.y;
  wi.nqc = min(qchunk, p.boff[it.x + 1] - wi.bstart);
  wi.lstart = p.list_off[wi.l];
  wi.len = (int)min64(p.list_off[wi.l + 1] - wi.lstart, p.rowcap);
  wi.ntiles = (wi.len + 127) >> 7;
  return wi;
}
__device__ __forceinline__ WorkInfo work_info(const TcScanParams& p, int w, int qchunk) {
  return work_info_of(p, p.witems[w], qchunk);
}
// A work item's dependent loads are software-pipelined across items (producer and gatherer): the
// (list, bucket) entry of item i+3, then the bucket end and list range of item i+2 (ItemRaw), are
// loaded while item i runs, and nothing derived from a load is computed in the iteration that
// issues it -- so no global round trip sits between two items (short items: c3, c5).
struct ItemRaw {
  int2 it;
  int bend;
  int64_t lo0, lo1;
};
__device__ __forceinline__ ItemRaw item_raw(const TcScanParams& p, int2 it) {
  ItemRaw r;
  r.it = it;
  it.x &= ~kItemMulti;
  const int l = it.x >= p.nlist ? it.x - p.nlist : it.x;
  r.bend = p.boff[it.x + 1];
  r.lo0 = p.list_off[l];
  r.lo1 = p.list_off[l + 1];
  return r;
}
__device__ __forceinline__ WorkInfo work_info_raw(const TcScanParams& p, const ItemRaw& r, int qchunk) {
  WorkInfo wi;
  wi.multi = r.it.x & kItemMulti;
  const int v = r.it.x & ~kItemMulti;
  wi.l = v >= p.nlist ? v - p.nlist : v;
  wi.bstart = r.it.y;
  wi.nqc = min(qchunk, r.bend - wi.bstart);
  wi.lstart = r.lo0;
  wi.len = (int)min64(r.lo1 - r.lo0, p.rowcap);
  wi.ntiles = (wi.len + 127) >> 7;
  return wi;
}

constexpr int kMaxNTS = 16;      // per-tile side-data ring slots (p.nts <= kMaxNTS)
constexpr int kMaxAcc = 8;       // TMEM accumulator buffers (tiles in flight between MMA and epilogue)
constexpr int kRing = 16;        // item-position ring (gatherer -> producer)
constexpr int kLook = 12;        // the gatherer takes positions this many items ahead (<= kRing + 1)
// side slot: norms f64 [1152 B] | rank u32 [640 B] | ids i64 [1152 B]; each copied as the 16-B aligned
// superset of the tile's 128 rows (the arrays are padded at allocation so the copy stays in bounds)
// (p.side_bytes: 3072 with a bitset, else 1792 -- the ids are not copied)
constexpr int kSideRank = 1152, kSideIds = 1792;
// epilogue warps: three per TMEM lane quarter (<= 128 registers per thread: 512 threads fit the
// register file).  Measured: 8 -> 12 took configs[1]'s phase B from 289 to 256 us and configs[4]'s
// per-GPU scan from 9.4 to 8.9 ms; 16 was slower for FLAT (6 chunks of 16 columns over 4 warps)
// SQ8 with 128-code rows: four per quarter (640 threads, <= 102 registers; configs[4]'s phase B
// 3.98 -> 3.70 ms; configs[2]'s 96-code rows measured slower with four)
template <int TYPE, int ATOM>
constexpr int epi_warps() { return TYPE == MV_IVF_SQ8 && ATOM == 128 ? 16 : 12; }

// per-query metadata of one work item (QCP = roundup16(qchunk) entries per array)
struct Meta {
  WorkInfo* wi;    // the work item (written by the gatherer: the MMA and epilogue warps read it here)
  int32_t* qidx;   // query index
  int32_t* pair;   // (query, rank) pair id, q * npb + r
  int32_t* cnt;    // candidates emitted so far (smem atomics)
  float* thf;      // badness bound: a candidate can pass only if badness <= thf (NaN: padding column)
  float* qnf;      // (float)||q||^2
  float* qs;       // SQ8 digit scale
  float* qaf;      // SQ8 (float) q.a
  float* thc;      // SQ8 fp32-filter bound: thf + the column's share of the filter error bound
  uint64_t* tau;   // exact bound: emit only keys < tau
  int64_t* base;   // output region of the pair
  double* qn;      // ||q||^2 (fp64)
  double* qa;      // SQ8 q.a (fp64)
};
__device__ __forceinline__ Meta meta_at(uint8_t* m, int QCP) {
  Meta r;
  r.wi = reinterpret_cast<WorkInfo*>(m);
  r.qidx = reinterpret_cast<int32_t*>(m + 32);
  m += 32 + 4 * QCP;
  r.pair = reinterpret_cast<int32_t*>(m);
  r.cnt = r.pair + QCP;
  r.thf = reinterpret_cast<float*>(r.cnt + QCP);
  r.qnf = r.thf + QCP;
  r.qs = r.qnf + QCP;
  r.qaf = r.qs + QCP;
  r.thc = r.qaf + QCP;
  r.tau = reinterpret_cast<uint64_t*>(m + 28 * QCP);
  r.base = reinterpret_cast<int64_t*>(r.tau + QCP);
  r.qn = reinterpret_cast<double*>(r.base + QCP);
  r.qa = r.qn + QCP;
  return r;
}
constexpr int kMetaPerQuery = 64;  // bytes (+ a 32-B work-item header)

template <int TYPE, int ATOM, bool SMALLD>
__global__ void __launch_bounds__(128 + 32 * epi_warps<TYPE, ATOM>(), 1)
    k_scan_tc(const __grid_constant__ XMaps xm, const TcScanParams p) {
  constexpr int kEpiWarps = epi_warps<TYPE, ATOM>();
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  constexpr int ESZ = TYPE == MV_IVF_FLAT ? 4 : 1;
  constexpr int PMAX = 2;  // FLAT: hi/lo query planes; SQ8: kSq8Planes digit planes
  const int nstage = p.nstage, nchunks = p.nchunks;
  const int QCP = (p.qchunk + 15) & ~15;       // metadata capacity (the largest chunk)
  const int QC = p.cfg[0];                      // queries per work item in this search
  const int P = TYPE == MV_IVF_FLAT ? p.cfg[1] : kSq8Planes;  // query planes: FLAT 1 (tf32-exact queries) or 2
  const int rowbytes = p.dpad * ESZ;
  const bool use_norms = p.metric == MV_L2;
  const bool use_ids = p.bitset != nullptr;
  const bool phaseB = p.phase != 0;
  // phase A of a k > 256 search emits 4-byte distance keys (its tau select needs no id ranks)
  const bool key32 = !phaseB && p.key32;
  // filter mode: the tensor-core badness is an approximation with a rigorous error bound E_q
  // (SQ8 always; FLAT when the stored values or the queries are not tf32-exact); the keys are
  // re-scored exactly after the scan (k_select.cu k_rekey)
  const bool approx = TYPE == MV_IVF_SQ8 || p.approx_always || P == 2;
  // epilogue column chunk: 16 (FLAT), 8 (SQ8: few queries per list, so both warps of a lane quarter
  // get columns)
  constexpr int W = TYPE == MV_IVF_FLAT ? 16 : 8;
  // query columns per plane: a multiple of the epilogue chunk.  The MMA's N = P x NQ must be a
  // multiple of 16: SQ8's two digit planes allow 8-column granularity (c3 averages ~20 queries per
  // probed list, c5 ~10: 24 / 16 columns per plane instead of 32 / 16)
  constexpr int QG = W;
  static_assert(TYPE == MV_IVF_FLAT || (kSq8Planes * QG) % 16 == 0, "SQ8 MMA width must be a multiple of 16");

  uint8_t* Xs = sm + p.off_x;
  uint8_t* Qs = sm + p.off_q;
  uint8_t* metab = sm + p.off_meta;
  uint8_t* side = sm + p.off_side;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + p.off_bar);
  uint64_t* full_x = bars;
  uint64_t* empty_x = bars + nstage;
  uint64_t* full_q = empty_x + nstage;
  uint64_t* empty_q = full_q + 2;
  uint64_t* empty_m = empty_q + 2;
  const int NACC = p.nacc;  // TMEM accumulator buffers (4 for FLAT, 2 for SQ8's 4-plane tiles)
  uint64_t* tfull = empty_m + 2;
  uint64_t* tempty = tfull + kMaxAcc;
  uint64_t* full_t = tempty + kMaxAcc;
  uint64_t* empty_t = full_t + kMaxNTS;
  uint64_t* sfull = empty_t + kMaxNTS;   // item-position ring: filled by the gatherer ...
  uint64_t* sempty = sfull + kRing;      // ... drained by the producer
  int32_t* ring = reinterpret_cast<int32_t*>(sempty + kRing);
  uint32_t* tslot = reinterpret_cast<uint32_t*>(ring + kRing);
  const int NTS = p.nts, SIDEB = p.side_bytes;

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
    }
    for (int a = 0; a < kMaxAcc; ++a) {
      mbar_init(&tfull[a], 1);
      mbar_init(&tempty[a], 4);  // the tile's epilogue warp of each lane quarter
    }
    for (int s = 0; s < NTS; ++s) {
      mbar_init(&full_t[s], 1);
      mbar_init(&empty_t[s], 4);
    }
    for (int s = 0; s < kRing; ++s) {
      mbar_init(&sfull[s], 1);
      mbar_init(&sempty[s], 1);
    }
    fence_mbar_init();
  }
  if (warp == 1) {
    tmem_alloc(tslot, p.tmem_cols);
    tmem_relinquish();
  }
  if (warp == 0 && lane == 0)
    for (int i = 0; i < 4; ++i) tma_prefetch(&xm.m[i]);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tslot;
  const int nwork = *p.nwitems;
#ifdef MV_SCAN_TRACE
  auto gtimer = []() {
    uint64_t t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
  };
  if (p.prof && threadIdx.x == 0 && blockIdx.x < 148) p.prof[8 * 1024 + blockIdx.x * 3] = gtimer();
#endif
  // dynamic schedule over the longest-first item order: the gatherer takes the next position from
  // the launch's global counter kLook items ahead of its own iteration and hands the positions to
  // the producer through a shared-memory ring (the MMA and epilogue warps get each item from the
  // gatherer's metadata).  Items are taken in order by whichever CTA is free: a list's sibling items
  // (consecutive positions) run at the same time on several CTAs, so its tiles come from DRAM once
  // and from L2 for the siblings (round 2's static snake schedule read c4's lists 1.83x)
  const int wb = p.wbeg ? *p.wbeg : 0;

  if (warp == 0) {
    // ------------------------------------------------------------------ TMA producer
    // the whole warp runs the loop (warp-uniform values), one elected lane issues each copy; ring
    // positions advance without divisions (as the MMA warp)
    {
      uint32_t s = 0, sph = 0;    // X ring stage / phase
      uint32_t ts = 0, tph = 0;   // side-data slot / phase
#ifdef MV_SCAN_TRACE
      uint32_t it = 0;
#endif
      const uint32_t side_tx = 528 + (use_norms ? 1040 : 0) + (use_ids ? 1040 : 0);
      // list tiles stream through L2 evict-first, except a list with sibling items: its neighbours
      // in the schedule read the same tiles at about the same time
      const uint64_t pol_first = l2_evict_first_policy(), pol_normal = l2_evict_normal_policy();
      // the item positions, in the gatherer's order
      uint32_t rs = 0, rph = 0;
      auto take = [&]() {
        mbar_wait(&sfull[rs], rph);
        const int v = ring[rs];
        __syncwarp();
        mbar_arrive_elect(&sempty[rs]);
        if (++rs == (uint32_t)kRing) {
          rs = 0;
          rph ^= 1;
        }
        return v;
      };
      // three-deep load pipeline (ItemRaw): item i+1's work info is ready when item i starts
      int q0 = take(), q1 = take(), q2 = take();
      int2 it3 = q2 < nwork ? p.witems[q2] : make_int2(0, 0);
      ItemRaw r2{};
      if (q1 < nwork) r2 = item_raw(p, p.witems[q1]);
      WorkInfo wn = q0 < nwork ? work_info(p, q0, QC) : WorkInfo{};
      while (q0 < nwork) {
        const WorkInfo wi = wn;
        const int q3 = q2 < nwork ? take() : nwork;  // (positions only grow)
        if (q1 < nwork) wn = work_info_raw(p, r2, QC);
        if (q2 < nwork) r2 = item_raw(p, it3);
        if (q3 < nwork) it3 = p.witems[q3];
        q0 = q1;
        q1 = q2;
        q2 = q3;
        const uint64_t pol = wi.multi ? pol_normal : pol_first;
        for (int t = 0; t < wi.ntiles; ++t) {
          const int row0 = (int)(wi.lstart + t * 128);
          mbar_wait(&empty_t[ts], tph ^ 1);
#ifdef MV_EXP_NOSIDE  // timing experiment only (wrong results): no side data
          mbar_arrive_elect(&full_t[ts]);
          (void)side_tx;
#else
          mbar_expect_tx_elect(&full_t[ts], side_tx);
          uint8_t* sd = side + ts * SIDEB;
          bulk_g2s_elect(sd + kSideRank, p.rank + (row0 & ~3), 528, &full_t[ts]);
          if (use_norms) bulk_g2s_elect(sd, p.norms + (row0 & ~1), 1040, &full_t[ts]);
          if (use_ids) bulk_g2s_elect(sd + kSideIds, p.ids + (row0 & ~1), 1040, &full_t[ts]);
#endif
          if (++ts == (uint32_t)NTS) {
            ts = 0;
            tph ^= 1;
          }
          // a list's tail tile loads roundup16(rows) rows as 64/32/16-row boxes (< 16 rows past the
          // list end); its stale smem rows beyond are masked lanes of the MMA's M = 128
          const int rows = min(128, wi.len - t * 128);
          const int r16 = (rows + 15) & ~15;
          for (int c = 0; c < nchunks; ++c) {
            mbar_wait(&empty_x[s], sph ^ 1);
#ifdef MV_SCAN_TRACE
            if (lane == 0) MV_TRACE(0, it);
            ++it;
#endif
            uint8_t* dst = Xs + s * 128 * ATOM;
            if (rows > 112) {
              mbar_expect_tx_elect(&full_x[s], 128 * ATOM);
              tma_load_2d_hint_elect(dst, &xm.m[0], &full_x[s], c * ATOM / ESZ, row0, pol);
            } else {
              mbar_expect_tx_elect(&full_x[s], r16 * ATOM);
              int o = 0;
              if (r16 & 64) { tma_load_2d_hint_elect(dst, &xm.m[1], &full_x[s], c * ATOM / ESZ, row0, pol); o += 64; }
              if (r16 & 32) { tma_load_2d_hint_elect(dst + o * ATOM, &xm.m[2], &full_x[s], c * ATOM / ESZ, row0 + o, pol); o += 32; }
              if (r16 & 16) tma_load_2d_hint_elect(dst + o * ATOM, &xm.m[3], &full_x[s], c * ATOM / ESZ, row0 + o, pol);
            }
            if (++s == (uint32_t)nstage) {
              s = 0;
              sph ^= 1;
            }
          }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------------ MMA issuer
    // the whole warp runs the loop (warp-uniform values in uniform registers), one elected lane
    // issues each tcgen05 instruction; ring / accumulator positions advance without divisions
    {
      uint32_t s = 0, sph = 0;     // X ring stage and its phase
      uint32_t acc = 0, aph = 0;   // TMEM accumulator and its phase
#ifdef MV_SCAN_TRACE
      uint32_t it = 0;
#endif
      uint32_t titer = 0;
      for (uint32_t wcount = 0;; ++wcount) {
        const uint32_t b = wcount & 1;
        mbar_wait(&full_q[b], (wcount >> 1) & 1);
        if (lane == 0) MV_TRACE(1, wcount);
        tc_fence_after();
        const WorkInfo wi = *meta_at(metab + b * p.meta_bytes, QCP).wi;
        if (wi.ntiles < 0) break;  // the gatherer's end marker
        const int NQ = (wi.nqc + QG - 1) & ~(QG - 1);
        const int N = P * NQ;
        const uint32_t idesc = TYPE == MV_IVF_FLAT ? idesc_tf32(N) : idesc_u8s8(N);
        const uint32_t qbase = smem_u32(Qs + b * p.q_bytes);
        for (int t = 0; t < wi.ntiles; ++t, ++titer) {
          mbar_wait(&tempty[acc], aph ^ 1);
          if (lane == 0) MV_TRACE(2, titer);
          tc_fence_after();
          const uint32_t dcol = tmem + acc * p.ncol;
          for (int c = 0; c < nchunks; ++c) {
            mbar_wait(&full_x[s], sph);
#ifdef MV_SCAN_TRACE
            if (lane == 0) MV_TRACE(7, it);
            ++it;
#endif
            tc_fence_after();
            const uint32_t xb = smem_u32(Xs + s * 128 * ATOM);
            const uint32_t qb = qbase + c * N * ATOM;
#ifdef MV_EXP_NOMMA  // timing experiment only (wrong results): stages released without MMAs
            (void)xb; (void)qb; (void)dcol; (void)idesc;
            if (lane == 0) mbar_arrive(&empty_x[s]);
#else
#pragma unroll
            for (int ks = 0; ks < ATOM / 32; ++ks) {
              const uint64_t ad = kmajor_desc(xb + ks * 32, ATOM);
              const uint64_t bd = kmajor_desc(qb + ks * 32, ATOM);
              if (TYPE == MV_IVF_FLAT) mma_tf32_elect(dcol, ad, bd, idesc, (c | ks) != 0);
              else mma_i8_elect(dcol, ad, bd, idesc, (c | ks) != 0);
            }
            mma_commit_elect(&empty_x[s]);
#endif
            if (++s == (uint32_t)nstage) {
              s = 0;
              sph ^= 1;
            }
          }
#ifdef MV_EXP_NOMMA
          if (lane == 0) mbar_arrive(&tfull[acc]);
#else
          mma_commit_elect(&tfull[acc]);
#endif
          if (lane == 0) MV_TRACE(3, titer);
          if (++acc == (uint32_t)NACC) {
            acc = 0;
            aph ^= 1;
          }
        }
        mma_commit_elect(&empty_q[b]);
      }
#ifdef MV_SCAN_TRACE
      if (lane == 0 && p.prof && blockIdx.x < 148) {
        p.prof[8 * 1024 + blockIdx.x * 3 + 1] = gtimer();
        p.prof[8 * 1024 + blockIdx.x * 3 + 2] = titer;
      }
#endif
    }
  } else if (warp < 4) {
    // ------------------------------------------------------------------ query gatherer (64 thr)
    const int tq = threadIdx.x - 64;
    const int gw = tq >> 5;
    // the next item's list range and per-query metadata are loaded into registers before waiting
    // for its buffers, so only the plane copies sit on the critical path once a buffer frees
    struct Pref {
      WorkInfo wi;
      int pr[2], q[2];
      uint64_t tau[2];
      double qn[2], qa[2];
      float qs[2], qe[2];
      int64_t base[2];
    };
    // raw loads of the (list, bucket) level: the item's ranges and its queries' pair ids (bq
    // entries past the item are read but unused; nbq bounds the read)
    struct QRaw {
      ItemRaw r;
      int pr[2];
    };
    auto q_raw = [&](int2 it) {
      QRaw x;
      x.r = item_raw(p, it);
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        const int i = tq + 64 * u;
        const int64_t pos = (int64_t)it.y + i;
        x.pr[u] = (i < QC && pos < p.nbq) ? p.bq[pos] : 0;
      }
      return x;
    };
    // the per-query level (issued one item ahead; used when the item is processed)
    auto prefetch = [&](const QRaw& x) {
      Pref f;
      f.wi = work_info_raw(p, x.r, QC);
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        const int i = tq + 64 * u;
        if (i < f.wi.nqc) {
          f.pr[u] = x.pr[u];
          // phase-A entries carry pair id npairs + p (their own output regions)
          const int64_t npairs = p.nq * p.npb;
          f.q[u] = (int)((f.pr[u] >= npairs ? f.pr[u] - npairs : f.pr[u]) / p.npb);
          f.tau[u] = phaseB ? p.tau[f.q[u]] : MV_KEY_PAD;
          f.qn[u] = p.qnorm[f.q[u]];
          f.qs[u] = TYPE == MV_IVF_SQ8 ? p.qscale[f.q[u]] : 1.0f;
          f.qe[u] = approx ? p.qerr[f.q[u]] : 0.0f;
          f.qa[u] = TYPE == MV_IVF_SQ8 ? p.qa[f.q[u]] : 0.0;
          f.base[u] = p.poff[f.pr[u]];
        }
      }
      return f;
    };
    // item positions: thread tq == 0 takes them from the launch's counter kLook items ahead and
    // publishes them in the ring (for the producer, and for every gatherer thread after the
    // iteration's named barrier: position j is read at iteration j - 3 >= its publication + 1)
    int pend = 0;
    if (tq == 0) {
      for (int j = 0; j < kLook - 1; ++j) {
        ring[j] = wb + atomicAdd(p.counter, 1);
        mbar_arrive(&sfull[j]);
      }
      pend = wb + atomicAdd(p.counter, 1);  // position kLook - 1: published at iteration 0
    }
    named_bar(2, 64);
    auto pos = [&](uint32_t j) { return ring[j % kRing]; };
    Pref cur;
    if (pos(0) < nwork) cur = prefetch(q_raw(p.witems[pos(0)]));
    QRaw n2{};
    if (pos(1) < nwork) n2 = q_raw(p.witems[pos(1)]);
    int2 n1 = pos(2) < nwork ? p.witems[pos(2)] : make_int2(0, 0);
    uint32_t wcount = 0;
    // the epilogue never waits for its peers at the end of an item: the gatherer publishes an
    // item's candidate counts when its metadata buffer comes back (every epilogue warp has
    // arrived on empty_m), each thread for the query slots it is about to overwrite
    int prev_nqc[2] = {0, 0};
    auto publish = [&](uint32_t bb) {
      const Meta om = meta_at(metab + bb * p.meta_bytes, QCP);
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        const int i = tq + 64 * u;
        if (i < prev_nqc[bb]) p.pcnt[om.pair[i]] = om.cnt[i];
      }
      prev_nqc[bb] = 0;
    };
    for (uint32_t i = 0;; ++i, ++wcount) {
      const bool done = pos(i) >= nwork;  // positions only grow: every later one is past the end too
      Pref nxt;
      if (!done) {
        if (pos(i + 1) < nwork) nxt = prefetch(n2);
        if (pos(i + 2) < nwork) n2 = q_raw(n1);
        if (pos(i + 3) < nwork) n1 = p.witems[pos(i + 3)];
        if (tq == 0) {  // publish position i + kLook - 1, take position i + kLook
          const uint32_t j = i + kLook - 1, sl = j % kRing;
          mbar_wait(&sempty[sl], ((j / kRing) & 1) ^ 1);
          ring[sl] = pend;
          mbar_arrive(&sfull[sl]);
          pend = wb + atomicAdd(p.counter, 1);
        }
      }
      const WorkInfo wi = cur.wi;
      const int NQ = (wi.nqc + QG - 1) & ~(QG - 1);
      const int N = P * NQ;
      const uint32_t b = wcount & 1, r = wcount >> 1;
      mbar_wait(&empty_q[b], (r & 1) ^ 1);
      mbar_wait(&empty_m[b], (r & 1) ^ 1);
      publish(b);
      const Meta mt = meta_at(metab + b * p.meta_bytes, QCP);
      if (done) {  // end marker for the MMA and epilogue warps
        if (tq == 0) mt.wi->ntiles = -1;
        named_bar(2, 64);
        mbar_arrive(&full_q[b]);
        break;
      }
      prev_nqc[b] = wi.nqc;
      if (tq == 0) *mt.wi = wi;
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        const int i = tq + 64 * u;
        if (i < wi.nqc) {
          const uint64_t t = cur.tau[u];
          const uint32_t t32 = (uint32_t)(t >> 32);
          mt.qidx[i] = cur.q[u];
          mt.pair[i] = cur.pr[u];
          mt.cnt[i] = 0;
          mt.tau[i] = t;
          // filter mode: tau_q is the k-th best approximate key of phase A, so a candidate of the
          // exact top-k has an approximate badness <= tau_q + 2 E_q (DESIGN.md §5 "FLAT precision")
          mt.thf[i] = t32 >= 0xff800000u ? __int_as_float(0x7f800000)
                      : approx          ? __fadd_ru(key2f(t32), 2.0f * cur.qe[u])
                                        : key2f(t32);
          mt.qnf[i] = (float)cur.qn[u];
          mt.qn[i] = cur.qn[u];
          mt.qs[i] = cur.qs[u];
          mt.qa[i] = cur.qa[u];
          mt.qaf[i] = (float)cur.qa[u];
          mt.base[i] = cur.base[u];
        } else if (i < NQ) {  // padding column: no comparison passes
          mt.thf[i] = __int_as_float(0x7fffffff);
          mt.qnf[i] = 0.f;
          mt.qn[i] = 0.0;
          mt.qs[i] = 0.f;
          mt.qa[i] = 0.0;
          mt.qaf[i] = 0.f;
        }
      }
      named_bar(2, 64);
      // plane copies: one operand row (query i, plane pl) per warp iteration, the row's 16-B pieces
      // across the lanes (coalesced reads), swizzled into the K-major operand
      uint8_t* Qb = Qs + b * p.q_bytes;
      constexpr int PIECES = ATOM / 16;
      const int ppr = nchunks * PIECES;  // pieces per row
      const int nrows = wi.nqc * P;
      for (int u = gw; u < nrows; u += 2) {
        const int i = P == 1 ? u : (P == 2 ? u >> 1 : u >> 2);
        const int pl = u - i * P;
        const int q = mt.qidx[i];
        const int64_t prow = TYPE == MV_IVF_FLAT ? (int64_t)pl * p.nq + q : (int64_t)q * P + pl;
        const uint8_t* src = p.qplanes + prow * rowbytes;
        for (int e = lane; e < ppr; e += 32) {
          const int c = e / PIECES, pc = e % PIECES;  // PIECES is a power of two
#ifndef MV_EXP_NOGATHER  // timing experiment only (wrong results): no query-plane copies
          cp_async16(Qb + c * N * ATOM + swz_off(pl * NQ + i, pc, ATOM), src + e * 16);
#else
          (void)src; (void)c; (void)pc;
#endif
        }
      }
      cp_async_wait_all();
      fence_proxy_async();
      mbar_arrive(&full_q[b]);
      if (tq == 0) MV_TRACE(5, wcount);
      cur = nxt;
    }
    // the last item (the end marker's step published the one before): wait until the epilogue is
    // done with it, then publish
    {
      const uint32_t e = wcount + 1, b = e & 1, r = e >> 1;
      if (prev_nqc[b] != 0) {
        mbar_wait(&empty_m[b], (r & 1) ^ 1);
        publish(b);
      }
    }
  } else {
    // ------------------------------------------------------------------ epilogue (8 warps)
    const int ew = warp - 4;            // 0..7
    const int quarter = warp & 3;       // TMEM lane quarter this warp may access
    // the NPART warps of a lane quarter take the tiles in turn (tile titer: warp part titer % NPART),
    // each a whole tile's columns: one warp's per-tile latency chain (side data, TMEM loads, the
    // filter, the emission) overlaps its peers' tiles (measured: splitting every tile's columns
    // over the three warps left configs[4]'s 16-query tiles epilogue-bound at ~2300 cycles each)
    constexpr int NPART = kEpiWarps / 4;  // epilogue warps per lane quarter
    const int part = ew >> 2;
    const int row = quarter * 32 + lane;
    const int et = threadIdx.x - 128;   // 0..255
    const uint32_t ltmask = (1u << lane) - 1;
    uint32_t titer = 0;
    for (uint32_t wcount = 0;; ++wcount) {
      const uint32_t b = wcount & 1;
      mbar_wait(&full_q[b], (wcount >> 1) & 1);
      const Meta mt = meta_at(metab + b * p.meta_bytes, QCP);
      const WorkInfo wi = *mt.wi;
      if (wi.ntiles < 0) break;  // the gatherer's end marker
      const int NQ = (wi.nqc + QG - 1) & ~(QG - 1);
      const uint32_t s_qnf = smem_u32(mt.qnf), s_thf = smem_u32(mt.thf), s_qs = smem_u32(mt.qs),
                     s_qaf = smem_u32(mt.qaf), s_cnt = smem_u32(mt.cnt), s_base = smem_u32(mt.base);
      for (int t = 0; t < wi.ntiles; ++t, ++titer) {
        if ((int)(titer % NPART) != part) continue;
        const uint32_t a = titer % NACC;
        const uint32_t ts = titer % NTS;
        const int vrow = t * 128 + row;
        const int row0 = (int)(wi.lstart + t * 128);
        mbar_wait(&full_t[ts], (titer / NTS) & 1);
        const uint8_t* sd = side + ts * SIDEB;
#ifdef MV_EXP_NOSIDE
        const uint32_t rk = 0;
        const bool valid = vrow < wi.len;
        const double xn = 0.0;
        (void)sd;
#else
        const uint32_t rk = reinterpret_cast<const uint32_t*>(sd + kSideRank)[(row0 & 3) + row];
        bool valid = vrow < wi.len;
        if (valid && use_ids)
          valid = !bit_excluded(p.bitset, p.nbits, reinterpret_cast<const int64_t*>(sd + kSideIds)[(row0 & 1) + row]);
        const double xn = use_norms ? reinterpret_cast<const double*>(sd)[(row0 & 1) + row] : 0.0;
#endif
        const float xnf = (float)xn;
        mbar_wait(&tfull[a], (titer / NACC) & 1);
        if (et == 0) MV_TRACE(6, titer);
        tc_fence_after();
        const uint32_t tbase = tmem + a * p.ncol + ((uint32_t)(quarter * 32) << 16);
#ifdef MV_EXP_NOEPI  // timing experiment only (wrong results): no epilogue work
        for (int qc = 0; qc < 0; qc += W) {
#else
        for (int qc = 0; qc < NQ; qc += W) {
#endif
          uint32_t r[PMAX][W];
          tmem_ld_w<W>(tbase + qc, r[0]);
          if (TYPE == MV_IVF_SQ8 || P == 2) tmem_ld_w<W>(tbase + NQ + qc, r[1]);
          tmem_wait_ld();
          if (TYPE == MV_IVF_FLAT && P == 2) {  // hi + lo query planes
#pragma unroll
            for (int j = 0; j < W; ++j) r[0][j] = __float_as_uint(__uint_as_float(r[0][j]) + __uint_as_float(r[1][j]));
          }
          // the threshold filter, branch-free.  FLAT computes the fp32 distance (exact for
          // tf32-exact data and queries); SQ8 an fp32 approximation within E_q of the exact value
          float bad[W];
          uint32_t pm = 0;
#pragma unroll
          for (int v = 0; v < W / 4; ++v) {
            const float4 qn4 = lds_f4(s_qnf + 4 * (qc + 4 * v));
            const float4 th4 = lds_f4(s_thf + 4 * (qc + 4 * v));
            float4 qs4 = qn4, qa4 = qn4;
            if (TYPE == MV_IVF_SQ8) {
              qs4 = lds_f4(s_qs + 4 * (qc + 4 * v));
              qa4 = lds_f4(s_qaf + 4 * (qc + 4 * v));
            }
            const float qnv[4] = {qn4.x, qn4.y, qn4.z, qn4.w}, thv[4] = {th4.x, th4.y, th4.z, th4.w};
            const float qsv[4] = {qs4.x, qs4.y, qs4.z, qs4.w}, qav[4] = {qa4.x, qa4.y, qa4.z, qa4.w};
#pragma unroll
            for (int u = 0; u < 4; ++u) {
              const int j = 4 * v + u;
              if (TYPE == MV_IVF_FLAT) {
                // badness = L2 distance or -IP; exact for tf32-representable data (2 dot is exact,
                // so the fma rounds exactly like (|q|^2 + |x|^2) - 2 dot)
                const float dot = __uint_as_float(r[0][j]);
                bad[j] = use_norms ? fmaf(-2.0f, dot, qnv[u] + xnf) : -dot;
              } else {
                // digit partials converted exactly (magic number: |D| < 2^22 for rows of <= 128
                // codes), combined in fp32; the error is bounded by E_q (k_qplanes)
                float fd[kSq8Planes];
#pragma unroll
                for (int pl = 0; pl < kSq8Planes; ++pl)
                  fd[pl] = SMALLD ? __int_as_float(0x4B400000 + (int)r[pl][j]) - 12582912.0f
                                  : __int2float_rn((int)r[pl][j]);
                const float accf = fmaf(fd[1], 0.0078125f, fd[0]);  // D0 + D1 / 2^7
                const float dotf = fmaf(qsv[u], accf, qav[u]);
                bad[j] = use_norms ? fmaf(-2.0f, dotf, qnv[u] + xnf) : -dotf;
              }
              pm |= (bad[j] <= thv[u] ? 1u : 0u) << j;
            }
          }
          if (!valid) pm = 0;
          // (FLAT exact mode: an entry exactly at the bound's distance passes whatever its id rank
          // -- a few extra keys at tau_q's distance, never a missing one; the final select ranks them)
          if (__any_sync(MV_FULL, pm != 0)) {
            // ballot per column; lane j reserves column j's slots with one shared atomic and
            // broadcasts the column's output address (measured: a per-entry atomic path for sparse
            // chunks was slower on configs[1] and [2])
            uint32_t mj[W];
            int mine = 0;
#pragma unroll
            for (int j = 0; j < W; ++j) {
              mj[j] = __ballot_sync(MV_FULL, (pm >> j) & 1);
              if (lane == j) mine = __popc(mj[j]);
            }
            uint64_t cp = 0;  // lane j: the address of column j's first reserved slot
            if (key32) {  // seeding sample of a large-k search: the distance key alone (4 B)
              if (mine)
                cp = reinterpret_cast<uint64_t>(reinterpret_cast<uint32_t*>(p.part) + lds_s64(s_base + 8 * (qc + lane)) +
                                                atoms_add(s_cnt + 4 * (qc + lane), mine));
#pragma unroll
              for (int j = 0; j < W; ++j)
                if (mj[j]) {  // warp-uniform
                  uint32_t* dst = reinterpret_cast<uint32_t*>(__shfl_sync(MV_FULL, cp, j)) + __popc(mj[j] & ltmask);
                  if ((pm >> j) & 1) *dst = f2key_fast(bad[j]);
                }
              continue;
            }
            if (mine)
              cp = reinterpret_cast<uint64_t>(p.part + lds_s64(s_base + 8 * (qc + lane)) +
                                              atoms_add(s_cnt + 4 * (qc + lane), mine));
#pragma unroll
            for (int j = 0; j < W; ++j) {
              if (mj[j]) {  // warp-uniform
                uint64_t* dst = reinterpret_cast<uint64_t*>(__shfl_sync(MV_FULL, cp, j)) + __popc(mj[j] & ltmask);
                st_u64_if((pm >> j) & 1, dst, ((uint64_t)f2key_fast(bad[j]) << 32) | rk);
              }
            }
          }
        }
        tc_fence_before();
        if (et == 0) MV_TRACE(4, titer);
        __syncwarp();
        if (lane == 0) {
          mbar_arrive(&tempty[a]);
          mbar_arrive(&empty_t[ts]);
        }
      }
      // this warp is done with the work item (its slot reservations are in mt.cnt): free the
      // metadata; the gatherer publishes the counts once every epilogue warp has arrived
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty_m[b]);
    }
  }
  __syncthreads();
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
                          double* __restrict__ qa, double* __restrict__ qnorm, FlatErr fe, float* __restrict__ qerr) {
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
      // FLAT planes are the plane-major hi/lo split made by launch_hilo (shared with the coarse step).
      // Filter-mode bound E_q >= |approximate - exact badness| for every stored x:
      // the MMA sees x (1 + ex) and q (1 + eq) per element, so |q~.x~ - q.x| <= (ex + eq + ex eq) S
      // with S = sum |q_j x_j| <= ||q|| X; the fp32 accumulation of dpad exact tf32 products adds
      // <= dpad 2^-24 S per rounding chain (taken as (dpad + 4) 2^-23: 2x slack for the
      // accumulator's internal order, + the hi/lo column sum); 5% on top.  L2 doubles the dot's
      // error and adds the fp32 expansion (||q||^2 + ||x||^2) - 2 dot: <= 2^-22 (||q||^2 + X^2).
      if (qerr && lane == 0) {
        const double S = sqrt(nn) * sqrt(fe.xmax2);
        const double cdot = 1.05 * (fe.ex + fe.eq + fe.ex * fe.eq + (dpad + 4) * 0x1p-23);
        const double E = fe.metric == MV_L2 ? 2.0 * cdot * S + 0x1p-21 * (nn + fe.xmax2) : cdot * S + 0x1p-23 * S;
        qerr[q] = __double2float_ru(E);
      }
    } else {
      // fp64: w_j = q_j b_j, b_j = vdiff_j / 255, a_j = vmin_j + b_j / 2 (mid-bin decode)
      double amax = 0.0, dot = 0.0, qdec = 0.0;
      for (int j = lane; j < dpad; j += 32) {
        const double bj = (double)vdiff[j] / 255.0;
        const double aj = fma(0.5, bj, (double)vmin[j]);
        dot = fma((double)x[j], aj, dot);
        amax = fmax(amax, fabs((double)x[j] * bj));
        qdec = fma(fabs((double)x[j]), 2.0 * (double)vdiff[j] + fabs((double)vmin[j]), qdec);
      }
      for (int o = 16; o > 0; o >>= 1) {
        amax = fmax(amax, __shfl_xor_sync(MV_FULL, amax, o));
        dot += __shfl_xor_sync(MV_FULL, dot, o);
        qdec += __shfl_xor_sync(MV_FULL, qdec, o);
      }
      // the scale is rounded up to fp32 first, so the digits and the epilogue use the same exact s
      const double s = amax > 0.0 ? (double)__double2float_ru(amax / 127.0) : 1.0;
      int8_t* o = reinterpret_cast<int8_t*>(out) + q * kSq8Planes * dpad;
      // the digits' residual r_j = w_j / s - (d0 + d1 / 2^7 + ...), summed by sign: the filter's
      // error from the digits is s sum_j r_j c_j with codes c_j in [0, 255], at most
      // 255 s max(sum r+, sum r-) -- the actual residuals of this query, not the worst case
      double rp = 0.0, rn = 0.0;
      for (int j = lane; j < dpad; j += 32) {
        double u = (double)x[j] * ((double)vdiff[j] / 255.0) / s;  // in [-127, 127]
        double scale = 1.0;
#pragma unroll
        for (int dgt = 0; dgt < kSq8Planes; ++dgt) {  // base-2^7 signed digits: u ~ d0 + d1/2^7
          const double dd = fmin(fmax(rint(u), -127.0), 127.0);
          o[dgt * dpad + j] = (int8_t)dd;
          u = (u - dd) * 128.0;
          scale *= 1.0 / 128.0;
        }
        const double r = u * scale;  // (the last digit's remainder, in units of s)
        rp += fmax(r, 0.0);
        rn += fmax(-r, 0.0);
      }
      for (int o2 = 16; o2 > 0; o2 >>= 1) {
        rp += __shfl_xor_sync(MV_FULL, rp, o2);
        rn += __shfl_xor_sync(MV_FULL, rn, o2);
      }
      if (lane == 0) {
        qscale[q] = (float)s;
        qa[q] = dot;
        // Filter-mode bound E_q >= |fp32 filter badness - the oracle's badness|:
        //   the fp32 conversions, three FMAs and the expansion: 2^-21 (||q||^2 + X^2 + 2 (s Amax + |q.a|)),
        //   Amax = the largest |digit-weighted partial| (127 * 255 * dpad * (1 + 2^-7 + ...));
        //   the digits' residual: 255 s max(sum r+, sum r-) over this query's remainders r_j;
        //   the oracle's fp32 decode vmin + ((c + 0.5)/255) vdiff vs the exact affine map:
        //   2^-22 sum |q_j| (2 vdiff_j + |vmin_j|);  L2 doubles the dot's share;  + 2^-22 (||q||^2 + X^2)
        //   for the roundings of the result.
        if (qerr) {
          const double amx = 127.0 * 255.0 * dpad * 1.0079;
          const double mc = 0x1p-21 * (nn + fe.xmax2 + 2.0 * (s * amx + fabs(dot)));
          // (x 1.001 + a 2^-40 floor for the fp64 rounding of the residual sums)
          const double dd = (255.0 * s * fmax(rp, rn) * 1.001 + 0x1p-40 * s * dpad) + 0x1p-22 * qdec;
          const double E = mc + (fe.metric == MV_L2 ? 2.0 : 1.0) * dd + 0x1p-22 * (nn + fe.xmax2);
          qerr[q] = __double2float_ru(1.05 * E);
        }
      }
    }
  }
}

cudaError_t launch_qplanes(int type, const float* qpad, int64_t nq, int dpad, const float* vmin, const float* vdiff,
                           uint8_t* out, float* qscale, double* qa, double* qnorm, const FlatErr* fe, float* qerr,
                           cudaStream_t st) {
  if (nq == 0) return cudaSuccess;
  const int grid = (int)min64(kNumSMs * 16, (nq * 32 + 255) / 256);
  const FlatErr f = fe ? *fe : FlatErr{0.0, 0.0, 0.0, 0};
  k_qplanes<<<grid, 256, 0, st>>>(type, qpad, nq, dpad, vmin, vdiff, out, qscale, qa, qnorm, f, fe ? qerr : nullptr);
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
// Shared-memory plan: X ring + double-buffered query planes + double-buffered per-query metadata
// + the side-data ring; the deepest X ring (<= the type's cap) that fits in 227 KB.
static bool tc_scan_layout(int type, int dpad, int qc, int ns, bool ids, TcScanParams& p) {
  const int esz = type == MV_IVF_FLAT ? 4 : 1;
  // swizzle-atom row: 128 B (FLAT: 32 fp32; SQ8 rows of a multiple of 128 codes), else 32 B (SQ8)
  const int atom = (type == MV_IVF_FLAT || dpad % 128 == 0) ? 128 : 32;
  p.atom = atom;
  // FLAT: qc queries of one plane (tf32-exact queries) or qc/2 queries of two (hi/lo) in the same
  // operand rows; SQ8: four digit planes
  const int rows_per_q = type == MV_IVF_FLAT ? 1 : kSq8Planes;
  auto up = [](int x, int a) { return (x + a - 1) / a * a; };
  p.type = type;
  p.dpad = dpad;
  p.nchunks = dpad * esz / atom;
  p.qchunk = qc;
  p.qchunk_split = type == MV_IVF_FLAT ? qc / 2 : qc;
  const int qcp = (qc + 15) & ~15;
  // FLAT two-plane items hold qc/2 queries: N = 2 roundup16(qc/2) columns, which exceeds qcp for
  // qc = 16, 48, 80 -- the operand and the accumulators are sized for the wider of the two shapes
  p.ncol = type == MV_IVF_FLAT ? std::max(qcp, 2 * ((qc / 2 + 15) & ~15)) : rows_per_q * qcp;
  // FLAT: 4 accumulators of <= 96 columns; SQ8: as many 4-plane accumulators as TMEM holds (2 of
  // 256 columns for 64-query items, 4 for 32, 8 for 16): the epilogue's latency per tile is
  // hidden by the tiles in flight
  p.nacc = type == MV_IVF_FLAT ? 4 : std::max(2, std::min(kMaxAcc, 512 / p.ncol));
  int cols = 32;
  while (cols < p.nacc * p.ncol) cols <<= 1;
  if (cols > 512) return false;
  p.tmem_cols = cols;
  p.q_bytes = up(p.ncol * dpad * esz, 1024);
  p.meta_bytes = up(32 + kMetaPerQuery * qcp, 16);
  const int stage = 128 * atom;
  p.nstage = ns;
  p.off_x = 0;
  p.off_q = ns * stage;
  p.off_meta = p.off_q + 2 * p.q_bytes;
  p.off_side = up(p.off_meta + 2 * p.meta_bytes, 128);
  // side-data slots: every tile in the X ring, in the accumulators and in the epilogue holds one
  // (with too few the producer stalls on them and the ring never fills: 4 slots capped configs[4]'s
  // one-stage SQ8 tiles at 4 tiles in flight)
  p.side_bytes = ids ? 3072 : 1792;
  p.nts = std::max(4, std::min(kMaxNTS, ns / p.nchunks + p.nacc + 1));
  p.off_bar = p.off_side + p.nts * p.side_bytes;
  p.smem_total = p.off_bar + (2 * ns + 6 + 2 * kMaxAcc + 2 * kMaxNTS + 2 * kRing) * 8 + 4 * kRing + 16 +
                 1024;  // + 1 KB alignment slack
  return p.smem_total <= 227 * 1024;
}

bool tc_scan_plan(int type, int dpad, int k, double qpl, bool ids, const Options& o, TcScanParams& p) {
  const bool wide = type == MV_IVF_FLAT || dpad % 128 == 0;  // 16-KB stages
  // SQ8 items: 64 queries.  (Measured on configs[4], ~10 queries per probed list: 32-query items
  // with 4 TMEM accumulators in flight 0.76M qps, 16 with 8 0.61M, 64 with 2 0.87M; qpl, the
  // expected queries per probed list, is kept for the plan but does not change it.)
  (void)qpl;
  int qcmax = type == MV_IVF_FLAT ? 96 : 64;
  // tuning options (mv_index_set_option "sq8_qc" / "flat_qc"): launch shape only, never the result
  if (o.sq8_qc > 0 && type == MV_IVF_SQ8) qcmax = std::max(16, std::min(64, o.sq8_qc / 16 * 16));
  if (o.flat_qc > 0 && type == MV_IVF_FLAT) qcmax = std::max(16, std::min(128, o.flat_qc / 16 * 16));
  const int nscap = wide ? 12 : 36;
  const int nsmin = wide ? 4 : 6;  // >= 64 KB (16-KB stages) / 24 KB (4-KB stages) of list tiles in flight
  p.k = k;
  for (int qc = qcmax; qc >= 16; qc -= 16)
    for (int ns = nscap; ns >= nsmin; --ns)
      if (tc_scan_layout(type, dpad, qc, ns, ids, p)) return true;
  return false;
}

cudaError_t launch_scan_tc(const XMaps& xm, const TcScanParams& p, cudaStream_t st) {
  // SMALLD: SQ8 rows of <= 128 codes, whose digit partials stay below 2^22 in magnitude
  const bool sd = p.dpad <= 128;
  auto kern = p.type == MV_IVF_FLAT ? k_scan_tc<MV_IVF_FLAT, 128, true>
              : p.atom == 128       ? (sd ? k_scan_tc<MV_IVF_SQ8, 128, true> : k_scan_tc<MV_IVF_SQ8, 128, false>)
                                    : (sd ? k_scan_tc<MV_IVF_SQ8, 32, true> : k_scan_tc<MV_IVF_SQ8, 32, false>);
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_total);
  if (e != cudaSuccess) return e;
  int dev = 0, nsm = kNumSMs;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  const int nepi = p.type == MV_IVF_FLAT ? epi_warps<MV_IVF_FLAT, 128>()
                   : p.atom == 128       ? epi_warps<MV_IVF_SQ8, 128>()
                                         : epi_warps<MV_IVF_SQ8, 32>();
  kern<<<nsm, 128 + 32 * nepi, p.smem_total,
         st>>>(xm, p);
  return cudaGetLastError();
}

}  // namespace mv
