/*
 * mv.h -- C ABI of the B200-native batched IVF k-NN hot path (Milvus, SIGMOD'21).
 *
 * Problem (§3.2.1): given a batch of m queries and n data vectors, find for
 * each query its top-k most similar vectors; results are (int64 id, float distance) pairs
 * (Eq. (1) sizes heap entries as sizeof(int64)+sizeof(float)).
 * Indexes: IVF_FLAT and IVF_SQ8 (§2.2, 510-520 §3.1) and IVF_PQ (PAPER.md:519-521,
 * SURVEY §8(f) f3), metrics squared L2 and inner product (§2.1).  Also on the
 * device: k-means training of the coarse codebook (mv_kmeans, f1), strategy E's range bitmap
 * (mv_attr_bitset) and multi-vector fusion (mv_fuse_rows, f4).  Query processing is the two-step IVF procedure of
 * PAPER.md:523-532 (§3.1): find the nprobe closest buckets, then scan them.  k <= 16384
 * (§3.3).  A bitmap of entity ids is checked whenever a vector is
 * encountered, before the top-k (strategy B, §4.1).
 *
 * Conventions (all entry points):
 *   - Every call returns mv_status (MV_OK = 0).  No exception or abort crosses the ABI.  On a
 *     non-OK status, mv_last_error() returns a thread-local message.
 *   - Pointers are device pointers on the index's device, OR host pointers: host buffers are
 *     detected (cudaPointerGetAttributes), staged through device memory, and the call then
 *     completes synchronously before returning.
 *   - `stream` is a cudaStream_t (NULL = the legacy default stream).  With device pointers the
 *     work is enqueued on `stream` and the call returns without synchronising (cudaMemcpyAsync
 *     semantics): inputs must stay valid and outputs must not be read until the stream reaches
 *     the work.  Exceptions that synchronise are documented per call.
 *   - Argument errors return MV_EINVAL synchronously, before any work is enqueued.
 *     Asynchronous CUDA faults surface as MV_ECUDA from a later call.
 *   - The index owns all of its device storage; `add` copies.  Inputs and outputs are owned by
 *     the caller; outputs are caller-allocated.
 *   - State machine: create -> set_centroids -> (SQ8 only: train_sq8 | set_sq8) -> add* ->
 *     search*.  Out-of-order calls return MV_ESTATE.  `add` and `search` on one index must not
 *     overlap (the caller serialises); concurrent searches on different streams are allowed
 *     (read-only index, per-call workspace).
 */
#ifndef MV_H
#define MV_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define MV_API __attribute__((visibility("default")))
#else
#define MV_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct mv_index mv_index; /* opaque; owned by the library */

typedef enum {
  MV_L2 = 0, /* squared Euclidean distance; smaller is better */
  MV_IP = 1  /* inner product; larger is better */
} mv_metric;

typedef enum {
  MV_IVF_FLAT = 0, /* fine quantizer keeps the fp32 vector */
  MV_IVF_SQ8 = 1,  /* fine quantizer keeps one byte per dimension */
  MV_IVF_PQ = 2    /* product quantization: M one-byte sub-codes */
} mv_type;

/* Device-memory allocator supplied by the caller.  alloc(bytes, stream, ctx)
 * returns device memory on the index's device usable in stream order on `stream` (NULL on
 * failure -> MV_ENOMEM); free(ptr, stream, ctx) releases it, stream-ordered after the work the
 * library enqueued on `stream`.  The Python binding routes both to torch's caching allocator.
 * The index storage is taken from it too (freed by mv_index_destroy).  Per-search scratch is
 * requested in blocks of >= 16 MB (a few callbacks per search). */
typedef struct {
  void* (*alloc)(size_t bytes, void* stream, void* ctx);
  void (*free)(void* ptr, void* stream, void* ctx);
  void* ctx;
} mv_allocator;

typedef enum {
  MV_OK = 0,
  MV_EINVAL = -1, /* bad argument (range, null pointer, reserved id -1 in add, ...) */
  MV_ESTATE = -2, /* call out of order for the index state machine */
  MV_ENOMEM = -3, /* device allocation failed */
  MV_ECUDA = -4,  /* a CUDA runtime/driver error (possibly from earlier asynchronous work) */
  MV_ENCCL = -5   /* reserved for collective failures reported by the sharding layer */
} mv_status;

/* Create an empty index on CUDA device `device`.
 *   d      1 <= d <= 512 (rows are stored zero-padded to a multiple of 32 elements, which changes
 *             neither L2 nor IP; the tensor-core kernels stage a query operand of <= 512 dims in
 *             shared memory); nlist >= 1 buckets (K-means buckets, K=16384
 *             default).
 *   alloc  nullable: every device allocation of the index goes through it (else cudaMalloc for
 *             the storage and the device's stream-ordered pool for scratch).  Copied.
 * Synchronous.  *out receives the handle (destroy with mv_index_destroy). */
MV_API mv_status mv_index_create(int32_t d, mv_metric metric, mv_type type, int32_t nlist, int32_t device,
                                 const mv_allocator* alloc, mv_index** out);

/* Tuning options.  None changes a result (tested): they pick launch shapes, the seeding sample and
 * the scratch budget.  Names: "seeding" (0/1), "need" (seeding sample, candidates), "capa" (rows
 * per list of the sample), "sq8_qc" / "flat_qc" (queries per scan work item), "coarse_nqb",
 * "coarse_cs", "coarse_epi", "coarse_nacc" (coarse GEMM shape), "large_k_select" (k > 256: 0 = the
 * seeding sample as 4-byte keys + the staged radix select, 1 = the sample-threshold select, 2 =
 * 8-byte seeding keys + the staged radix select, 3 = the streaming select for the seeding bound,
 * 4 = 4-byte seeding keys + the streaming final select (k <= 4096, staged fallback)), "big_ctas" / "big_cap" (the staged
 * select's first launch: CTAs per SM, 1..4, and candidates staged per query; queries past it are
 * redone with all of shared memory), "async_host" (1: a search whose host buffers are all page-locked
 * enqueues its copies on `stream` and returns without synchronising -- the caller synchronises
 * `stream` before reading the results; pageable host buffers still complete synchronously),
 * "workspace_bytes" (per-search
 * scratch budget: larger batches run as several query chunks; 0 = half of the device memory that was
 * free after the last create/add).
 * value 0 = automatic.  MV_EINVAL for an unknown name or a negative value. */
MV_API mv_status mv_index_set_option(mv_index* index, const char* name, int64_t value);

/* Supply the coarse codebook C (§3.1): nlist x d fp32, row-major.  The
 * north star consumes supplied centroids; training them (k-means) is outside the library.
 * Synchronous (the centroid array is copied before return). */
MV_API mv_status mv_index_set_centroids(mv_index* index, const float* centroids);

/* SQ8 only.  Per-dimension range from a training sample (n x d fp32, n >= 1):
 *   vmin_j = min_i x_ij, vdiff_j = max_i x_ij - vmin_j  (fp32).  (the exact
 * formula is reading O3 of DESIGN.md §2.)  Synchronous. */
MV_API mv_status mv_index_train_sq8(mv_index* index, const float* sample, int64_t n);

/* SQ8 only.  Supply the quantizer parameters directly (d floats each, host or device).
 * vdiff_j >= 0; vdiff_j == 0 encodes every value of dimension j as code 0.  Synchronous. */
MV_API mv_status mv_index_set_sq8(mv_index* index, const float* vmin, const float* vdiff);

/* Insert n vectors (n x d fp32, row-major) with caller ids (n int64, any values except the
 * reserved -1; duplicates allowed); an index holds < 2^31 vectors.  Each vector goes to bucket I(v) = its closest centroid
 * (L2: argmin ||v-c||^2, IP: argmax <v,c>; ties -> smaller bucket id);
 * SQ8 codes are code = floor(255*clamp((x-vmin)/vdiff,0,1)) in fp32 with one rounding per
 * operation (bit-exact with the oracle).  Storage is list-major, each list in insertion order.
 * Synchronous (returns after the index is updated; re-allocates list storage). */
MV_API mv_status mv_index_add(mv_index* index, const float* vectors, const int64_t* ids, int64_t n, void* stream);

/* Batched k-NN search (§3.1, 537-546 §3.2.1).
 *   queries   nq x d fp32 row-major; nq >= 0 (nq == 0 is a no-op)
 *   k         1 <= k <= 16384
 *   nprobe    >= 1; values > nlist are clamped to nlist
 *   bitset    nullable; bit i = (bitset[i>>3] >> (i&7)) & 1, indexed by ID; 1 = EXCLUDED
 *             (deleted / failing the attribute filter; reading of PAPER.md:916-922).  ids >= nbits
 *             are never excluded.  Applied inside the scan, before selection.
 *   distances nq x k fp32 (out), ids nq x k int64 (out), row-major, best-first: ascending L2 /
 *             descending IP; exact ties ordered by smaller id, then storage position.  Slots
 *             beyond the number of candidates hold id -1 and distance +inf (L2) / -inf (IP).
 * Results are deterministic and independent of the rest of the batch (the batch runs as query
 * chunks when its scratch would exceed the "workspace_bytes" budget).  Asynchronous on `stream`
 * for device pointers.
 * Precision: IVF_SQ8 distances come from int32-exact digit partials combined in fp64.  IVF_FLAT
 * is exact on the tensor cores when the stored values and the queries are tf32-representable
 * (integer-valued data); otherwise the scan runs as a filter whose fp32 badness carries a
 * rigorous per-query error bound, and every candidate that can still reach the top-k is
 * re-scored in fp64 from the fp32 vectors: returned distances are the fp64 values
 * rounded to fp32 and the ids are those of the exact top-k. */
MV_API mv_status mv_search(mv_index* index, const float* queries, int64_t nq, int32_t k, int32_t nprobe,
                    const uint8_t* bitset, int64_t nbits, float* distances, int64_t* ids, void* stream);

/* Step (1) only: the nprobe closest buckets per query, best-first by
 * (centroid score, bucket id) -> probes nq x nprobe' int32 where nprobe' = min(nprobe, nlist).
 * When nprobe >= nlist every bucket is probed and they are listed in id order.  Parity hook for
 * the conditional-oracle protocol; same kernels as mv_search.  Asynchronous like mv_search. */
MV_API mv_status mv_search_probes(mv_index* index, const float* queries, int64_t nq, int32_t nprobe, int32_t* probes,
                           void* stream);

/* Steps (2)-(3) with caller-supplied probes (§3.1): probes nq x nprobe' int32
 * (nprobe' = min(nprobe, nlist)), each row the query's buckets best-first (as mv_search_probes
 * returns them; ids in [0, nlist), no duplicates -- not checked on the device).  Used by the
 * multi-GPU query-split coarse step: each rank computes the probes of a slice of the batch and
 * the slices are all-gathered.  Results equal mv_search's when the probes equal
 * mv_search_probes'.  Other arguments, errors and asynchrony as mv_search; host probes are staged. */
MV_API mv_status mv_search_with_probes(mv_index* index, const float* queries, int64_t nq, int32_t k, int32_t nprobe,
                                       const int32_t* probes, const uint8_t* bitset, int64_t nbits, float* distances,
                                       int64_t* ids, void* stream);

/* Merge nsrc per-shard top-k results (segments, §3.3; heap merge,
 * PAPER.md:590-596): dists nsrc x nq x k fp32, ids nsrc x nq x k int64, each row best-first
 * with -1 padding -> out_d / out_i nq x k, ordered by (distance, id, source, position).  Device
 * pointers (or host; staged).  Asynchronous on `stream` for device pointers. */
MV_API mv_status mv_merge_topk(mv_metric metric, const float* dists, const int64_t* ids, int32_t nsrc, int64_t nq,
                        int32_t k, float* out_d, int64_t* out_i, void* stream);

/* IVF_PQ fine quantizer ("splits each vector into multiple
 * sub-vectors and applies k-means for each sub-space"; reading R19): M sub-spaces of d / M
 * consecutive dimensions (d % M == 0, M % 4 == 0, M <= 64), 256 sub-centroids each.
 * set_pq: codebooks [M][256][d/M] fp32 (host or device), copied.  train_pq: per sub-space
 * mv_kmeans (L2, niter iterations, initial sub-centroids = the first 256 rows) over the
 * sample's sub-vectors (device [n][d] fp32, n >= 256).  Both synchronous; only before the first
 * add, on an MV_IVF_PQ index (else MV_ESTATE).  A search on an IVF_PQ index returns the
 * asymmetric distance from each query to the decoded vector (fp32 sums of fp32 table entries). */
MV_API mv_status mv_index_set_pq(mv_index* index, int32_t M, const float* codebooks);
MV_API mv_status mv_index_train_pq(mv_index* index, int32_t M, const float* sample, int64_t n, int32_t niter);
/* Parity hook: the PQ codebooks ([M][256][d/M] fp32, host or device) and M.  Synchronous. */
MV_API mv_status mv_index_get_pq(const mv_index* index, int32_t* M, float* codebooks);

/* Lloyd k-means training of the coarse codebook on the device (PAPER.md:503-514
 * §3.1: the buckets are K-means clusters).  x: device [n][d] fp32 training rows; centroids: device
 * [nlist][d] fp32 -- in: the initial centroids (e.g. nlist seeded training rows), out: after niter
 * iterations.  Each iteration assigns every row to its closest centroid under `metric` with the
 * index's tensor-core coarse step (the assignment mv_index_add makes: exact to the oracle up to
 * ties) and sets each centroid to the mean of its rows (fp64 sums, one rounding to fp32; spherical
 * != 0 normalises it); a centroid without rows keeps its position.  Synchronous; the scratch comes
 * from cudaMallocAsync.  MV_EINVAL: null pointers, nlist < 1, n < nlist, niter < 0, host pointers. */
MV_API mv_status mv_kmeans(const float* x, int64_t n, int32_t d, mv_metric metric, int32_t nlist, int32_t niter,
                           int32_t spherical, float* centroids, int32_t device, void* stream);

/* Strategy E's per-partition bitmap (§4.1 with strategy B's
 * bitmap): writes the whole bitset -- ceil(nbits/32) 32-bit words, LSB-first,
 * bit = 1 means excluded (the polarity mv_search takes) -- with bit ids[i] set for every i < n
 * whose attr[i] is outside [lo, hi].  ids / attr: n int64 each (the partition's entity ids and
 * attribute values, device); bitset: device, 4-byte aligned, caller-owned; ids outside
 * [0, nbits) are ignored (size nbits above the largest id).  Asynchronous on `stream`.
 * MV_EINVAL for n < 0, nbits < 0, lo > hi is allowed (everything excluded), null pointers with n > 0. */
MV_API mv_status mv_attr_bitset(const int64_t* ids, const int64_t* attr, int64_t n, int64_t lo, int64_t hi,
                                uint8_t* bitset, int64_t nbits, void* stream);

/* Vector fusion (§4.2): out[r] = [w_0 parts[0][r] | ... |
 * w_{m-1} parts[m-1][r]] for r < n -- the concatenated entity vectors (weights 1) or the
 * aggregated query (weights = the weighted-sum aggregation's w_i), so that one MV_IP search
 * returns the top-k by sum_i w_i (q.v_i . e.v_i).  parts: host array of m device pointers, part i
 * row-major [n][dims[i]] fp32; dims, weights: host arrays of m (weights NULL = all 1);
 * out: device [n][sum dims] fp32.  1 <= m <= 16.  Asynchronous on `stream`. */
MV_API mv_status mv_fuse_rows(const float* const* parts, const int32_t* dims, const float* weights, int32_t m,
                              int64_t n, float* out, void* stream);

/* Number of stored vectors. */
MV_API int64_t mv_index_ntotal(const mv_index* index);

/* Parity hook: copy the list-major storage description.  list_off: nlist+1 int64 (may be
 * NULL); ids: ntotal int64 in storage order (may be NULL); codes: ntotal x d uint8 (SQ8,
 * unpadded) or ntotal x M uint8 (IVF_PQ), may be NULL.  Host or device pointers.  Synchronous. */
MV_API mv_status mv_index_storage(const mv_index* index, int64_t* list_off, int64_t* ids, uint8_t* codes);

/* Parity hook: SQ8 parameters (d floats each). Synchronous. */
MV_API mv_status mv_index_get_sq8(const mv_index* index, float* vmin, float* vdiff);

/* Stage profiling (measurement, §8(d)).  When enabled, mv_search records CUDA events on its
 * stream around each stage:  0 = query staging + coarse (a1-a3), 1 = bucketing (a4),
 * 2 = list scan phase A (a5-a6: the seeding lists, every candidate emitted; the whole scan when
 * there is no seeding), 3 = seed select (tau_q = k-th best key of phase A), 4 = list scan phase B
 * (a5-a6: candidates below tau_q), 5 = final select (a7).
 * mv_profile_read synchronises on the recorded events and returns, per stage, the summed
 * milliseconds since the last reset (ms[6]); *searches = profiled mv_search calls; *launches =
 * kernels libmv launched in them.  `reset` != 0 clears the accumulators after reading. */
MV_API mv_status mv_profile_enable(mv_index* index, int on);
/* Emission counters of the profiled searches (measurement, §8(d)): out[0] = queries, out[1] =
 * candidates the seeding phase emitted, out[2] = candidates the main scan emitted (what the
 * selects read).  Synchronises the device.  `reset` != 0 clears them. */
MV_API mv_status mv_profile_counters(mv_index* index, int64_t* out, int reset);
MV_API mv_status mv_profile_read(mv_index* index, double* ms, int64_t* searches, int64_t* launches, int reset);

/* Human-readable index state (JSON object): d, nlist, ntotal, max list length, whether the
 * tensor-core scan is available and which scan implementation the last search used.  Writes at
 * most `len` bytes including the terminating NUL. */
MV_API mv_status mv_index_describe(const mv_index* index, char* buf, size_t len);

/* Release the index and all of its device storage (NULL is a no-op). */
MV_API void mv_index_destroy(mv_index* index);

/* Thread-local message for the last non-OK status on this thread ("" if none). */
MV_API const char* mv_last_error(void);

/* Library build string (compile target and version). */
MV_API const char* mv_version(void);

#ifdef __cplusplus
}
#endif
#endif /* MV_H */
