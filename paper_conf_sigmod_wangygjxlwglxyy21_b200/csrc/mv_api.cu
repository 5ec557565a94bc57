// mv_api.cu -- the C ABI of include/mv.h: index state, validation, memory (caller allocator or
// stream-ordered CUDA pools), host-pointer staging, and the search pipeline
// a1 -> a2/a3 -> a4 -> a5/a6 -> (FLAT filter mode: exact re-scoring) -> a7, enqueued on the
// caller's stream in query chunks that fit the workspace budget.
#include <cub/device/device_radix_sort.cuh>

#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <functional>
#include <string>
#include <vector>

#include "mv_internal.cuh"
#include "tmap.h"

using namespace mv;

struct mv_index {
  int d = 0, dpad = 0, metric = 0, type = 0, nlist = 0, device = 0;
  bool has_centroids = false, has_sq8 = false, has_pq = false;
  int pq_m = 0, pq_dsub = 0;    // IVF_PQ: sub-spaces and their dimension
  float* pq_cb = nullptr;       // IVF_PQ: [M][256][dsub] sub-centroids
  mv_allocator alloc{};         // caller allocator (alloc.alloc == NULL: CUDA's own)
  Options opt;
  float* cpad = nullptr;    // nlist x dpad
  float* cnorm = nullptr;   // nlist
  float* chl = nullptr;     // [2][nlist][dpad] tf32 hi / lo planes of the centroids (tcgen05 coarse)
  CUtensorMap cmap;
  float* vmin = nullptr;    // dpad (zero padded)
  float* vdiff = nullptr;   // dpad (zero padded)
  float* sq8_t = nullptr;   // 256: (c + 0.5f) / 255.f
  int64_t ntotal = 0;
  int64_t* list_off = nullptr;  // nlist + 1 (device)
  std::vector<int64_t> h_list_off;
  std::vector<int64_t> top_len_prefix;  // [j] = total length of the j longest lists (j = 0..nlist)
  int64_t maxlen = 0;
  void* payload = nullptr;      // ntotal x dpad (fp32 or u8)
  double* norms = nullptr;      // ntotal (+pad): ||x||^2 / ||x_hat||^2 in fp64
  int64_t* ids = nullptr;       // ntotal, storage order
  uint32_t* rank = nullptr;     // ntotal: position of (id, row) in sorted order
  int64_t* sorted_ids = nullptr;  // ntotal: ids in (id, row) order
  bool ids_identity = false;      // sorted_ids[r] == r (ids exactly 0..ntotal-1): no id gather
  uint32_t* row_of_rank = nullptr;  // storage row of each rank (the filter mode's exact re-scoring)
  double xmax2 = 0.0;           // max ||x||^2 (SQ8: ||x_hat||^2) over the stored rows (filter-mode bound)
  XMaps xm;                     // payload tensor maps: 128/64/32/16-row boxes (rebuilt by every add)
  bool tf32_exact = true;       // FLAT: every stored value exactly representable in tf32
  const char* last_scan = "none";
  const char* last_coarse = "none";
  int64_t last_chunks = 0;      // query chunks of the last search (workspace budget)
  int64_t auto_budget = 0;      // half of the free device memory, sampled at create and after each add
                                // (cudaMemGetInfo is a driver call that can stall behind NVML
                                // queries, so it is kept off the search path)
  // profiling
  bool prof = false;
  std::vector<cudaEvent_t> ev;   // kProfStages + 1 events per profiled search chunk
  int64_t prof_searches = 0, launches = 0;
  unsigned long long* d_count = nullptr;  // profiled: [queries, phase-A emissions, phase-B emissions]
};

// ------------------------------------------------------------------------------------------
namespace {
thread_local std::string g_err;

mv_status fail(mv_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return s;
}

mv_status from_cuda(cudaError_t e, const char* what) {
  cudaGetLastError();
  return fail(e == cudaErrorMemoryAllocation ? MV_ENOMEM : MV_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

#define CK(x)                                         \
  do {                                                \
    cudaError_t _e = (x);                             \
    if (_e != cudaSuccess) return from_cuda(_e, #x);  \
  } while (0)

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (dev >= 0 && prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

// page-locked host memory (cudaHostAlloc / cudaHostRegister): stream-ordered copies need no sync
bool is_pinned_ptr(const void* p) {
  if (p == nullptr) return true;
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return at.type == cudaMemoryTypeHost || at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

bool is_host_ptr(const void* p) {
  if (p == nullptr) return false;
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return true;
  }
  return at.type == cudaMemoryTypeHost || at.type == cudaMemoryTypeUnregistered;
}

// Long-lived index storage: the caller's allocator, else cudaMalloc.
void* mem_alloc(const mv_index* ix, size_t bytes, cudaStream_t st) {
  if (ix->alloc.alloc) return ix->alloc.alloc(bytes, st, ix->alloc.ctx);
  void* p = nullptr;
  if (cudaMalloc(&p, bytes) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return p;
}
void mem_free(const mv_index* ix, void* p, cudaStream_t st) {
  if (!p) return;
  if (ix->alloc.alloc) ix->alloc.free(p, st, ix->alloc.ctx);
  else cudaFree(p);
}

// Per-call scratch, released (stream-ordered) at scope exit.  With a caller allocator it is an
// arena of >= 16 MB blocks taken from the allocator on the call's stream (a handful of callbacks
// per search); otherwise stream-ordered cudaMallocAsync from the device pool.
struct Scratch {
  const mv_index* ix;
  cudaStream_t st;
  std::vector<void*> ptrs;
  char* cur = nullptr;
  size_t left = 0;
  Scratch(const mv_index* i, cudaStream_t s) : ix(i), st(s) {}
  ~Scratch() {
    for (void* p : ptrs) {
      if (ix && ix->alloc.alloc) ix->alloc.free(p, st, ix->alloc.ctx);
      else cudaFreeAsync(p, st);
    }
  }
  template <typename T>
  cudaError_t alloc(T** p, size_t n) {
    *p = nullptr;
    size_t bytes = (std::max<size_t>(n, 1) * sizeof(T) + 255) & ~(size_t)255;
    if (ix && ix->alloc.alloc) {
      if (bytes > left) {
        const size_t c = std::max<size_t>(bytes, (size_t)16 << 20);
        void* q = ix->alloc.alloc(c, st, ix->alloc.ctx);
        if (!q) return cudaErrorMemoryAllocation;
        ptrs.push_back(q);
        cur = static_cast<char*>(q);
        left = c;
      }
      *p = reinterpret_cast<T*>(cur);
      cur += bytes;
      left -= bytes;
      return cudaSuccess;
    }
    cudaError_t e = cudaMallocAsync(reinterpret_cast<void**>(p), bytes, st);
    if (e == cudaSuccess) ptrs.push_back(*p);
    return e;
  }
};

// Device view of a caller buffer: device pointers pass through; host buffers are staged.
template <typename T>
cudaError_t stage_in(Scratch& s, const T* p, size_t n, const T** out, bool* staged) {
  *staged = is_host_ptr(p);
  if (!*staged) {
    *out = p;
    return cudaSuccess;
  }
  T* d = nullptr;
  cudaError_t e = s.alloc(&d, n);
  if (e != cudaSuccess) return e;
  e = cudaMemcpyAsync(d, p, n * sizeof(T), cudaMemcpyHostToDevice, s.st);
  *out = d;
  return e;
}

void set_pool_threshold(int dev) {
  static bool done[64] = {false};
  if (dev < 0 || dev >= 64 || done[dev]) return;
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  done[dev] = true;
}

void prof_mark(mv_index* ix, cudaStream_t st) {
  if (!ix->prof) return;
  cudaEvent_t e;
  if (cudaEventCreate(&e) != cudaSuccess) return;
  cudaEventRecord(e, st);
  ix->ev.push_back(e);
}

void free_storage(mv_index* ix) {
  mem_free(ix, ix->payload, nullptr);
  mem_free(ix, ix->norms, nullptr);
  mem_free(ix, ix->ids, nullptr);
  mem_free(ix, ix->rank, nullptr);
  mem_free(ix, ix->sorted_ids, nullptr);
  mem_free(ix, ix->row_of_rank, nullptr);
  ix->payload = nullptr;
  ix->norms = nullptr;
  ix->ids = nullptr;
  ix->rank = nullptr;
  ix->sorted_ids = nullptr;
  ix->row_of_rank = nullptr;
}

int device_sms() {
  int dev = 0, nsm = kNumSMs;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  return nsm;
}
}  // namespace

// a2 + a3: tcgen05 coarse GEMM + per-query top-nprobe; every bucket (id order) when npb >= nlist
static cudaError_t run_coarse(mv_index* ix, const float* qhl, const int* qlo_any, int64_t nq, int npb, int32_t* P,
                              Scratch& s, cudaStream_t st) {
  if (npb >= ix->nlist) {
    ix->last_coarse = "all-lists";
    return launch_all_lists(nq, ix->nlist, P, st);
  }
  CoarseParams cp;
  if (!coarse_tc_plan(ix->dpad, npb, nq, ix->nlist, device_sms(), ix->opt, cp)) return cudaErrorInvalidConfiguration;
  CUtensorMap qmap;
  if (!make_tmap_2d(&qmap, qhl, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, (uint64_t)ix->dpad, 2 * (uint64_t)nq,
                    (uint64_t)ix->dpad * 4, 32, (uint32_t)cp.nqb, CU_TENSOR_MAP_SWIZZLE_128B))
    return cudaErrorInvalidValue;
  cp.nq = nq;
  cp.nlist = ix->nlist;
  cp.metric = ix->metric;
  cp.cnorm = ix->cnorm;
  cp.probes = P;
  cp.ldg = ((ix->nlist + 127) / 128) * 4;
  cp.ccap = 32 * npb;
  cp.qlo_any = qlo_any;
  cudaError_t e = s.alloc(&cp.G, (size_t)nq * cp.ldg);
  if (e == cudaSuccess) e = s.alloc(&cp.gbound, (size_t)nq);
  if (e == cudaSuccess) e = s.alloc(&cp.cand, (size_t)nq * cp.ccap);
  if (e == cudaSuccess) e = s.alloc(&cp.gslot, (size_t)nq * ((ix->nlist + 31) / 32));
  if (e == cudaSuccess) e = s.alloc(&cp.ccnt, (size_t)nq * npb);
  if (e != cudaSuccess) return e;
  ix->last_coarse = "tcgen05.tf32";
  return launch_coarse_tc(&ix->cmap, &qmap, cp, nq, st);
}

// Scratch bytes per query of one search chunk (an upper bound used to size the chunks)
static int64_t search_bytes_per_query(const mv_index* ix, int npb, int k) {
  const int64_t cand = ix->top_len_prefix[std::min<size_t>(npb, ix->top_len_prefix.size() - 1)];
  const int64_t need = std::max<int64_t>(2 * (int64_t)k, k + 32);
  const int64_t seed = std::min<int64_t>(65536, std::max<int64_t>(need, 4096)) + 4096;
  const int64_t coarse = npb < ix->nlist ? (int64_t)ix->nlist / 8 + 256 * (int64_t)npb + 16 : 0;
  return 8 * (cand + seed) + coarse + 48 * (int64_t)npb + 32 * (int64_t)ix->dpad + 64;
}

// ------------------------------------------------------------------------------------------
extern "C" {

const char* mv_last_error(void) { return g_err.c_str(); }

const char* mv_version(void) { return "libmv 0.2 (sm_100a; IVF_FLAT/IVF_SQ8/IVF_PQ; L2/IP)"; }

int64_t mv_index_ntotal(const mv_index* ix) { return ix ? ix->ntotal : 0; }

mv_status mv_index_create(int32_t d, mv_metric metric, mv_type type, int32_t nlist, int32_t device,
                          const mv_allocator* alloc, mv_index** out) {
  if (!out) return fail(MV_EINVAL, "out is NULL");
  *out = nullptr;
  if (d < 1 || d > kMaxD) return fail(MV_EINVAL, "d must be in [1, %d] (got %d)", kMaxD, d);
  if (metric != MV_L2 && metric != MV_IP) return fail(MV_EINVAL, "unknown metric %d", (int)metric);
  if (type != MV_IVF_FLAT && type != MV_IVF_SQ8 && type != MV_IVF_PQ)
    return fail(MV_EINVAL, "unknown index type %d", (int)type);
  if (nlist < 1) return fail(MV_EINVAL, "nlist must be >= 1 (got %d)", nlist);
  if (alloc && (alloc->alloc == nullptr) != (alloc->free == nullptr))
    return fail(MV_EINVAL, "allocator: alloc and free must both be set");
  int ndev = 0;
  CK(cudaGetDeviceCount(&ndev));
  if (device < 0 || device >= ndev) return fail(MV_EINVAL, "device %d out of range (%d devices)", device, ndev);
  DeviceGuard g(device);
  set_pool_threshold(device);
  mv_index* ix = new mv_index();
  if (alloc) ix->alloc = *alloc;
  ix->d = d;
  ix->dpad = (d + 31) / 32 * 32;
  ix->metric = metric;
  ix->type = type;
  ix->nlist = nlist;
  ix->device = device;
  ix->h_list_off.assign(nlist + 1, 0);
  ix->top_len_prefix.assign(nlist + 1, 0);
  bool ok = (ix->list_off = (int64_t*)mem_alloc(ix, sizeof(int64_t) * (nlist + 1), nullptr)) &&
            (ix->cpad = (float*)mem_alloc(ix, sizeof(float) * (size_t)nlist * ix->dpad, nullptr)) &&
            (ix->cnorm = (float*)mem_alloc(ix, sizeof(float) * ((size_t)(nlist + 127) / 128 * 128), nullptr)) &&
            (ix->chl = (float*)mem_alloc(ix, sizeof(float) * 2 * (size_t)nlist * ix->dpad, nullptr)) &&
            (ix->vmin = (float*)mem_alloc(ix, sizeof(float) * ix->dpad, nullptr)) &&
            (ix->vdiff = (float*)mem_alloc(ix, sizeof(float) * ix->dpad, nullptr)) &&
            (ix->sq8_t = (float*)mem_alloc(ix, sizeof(float) * 256, nullptr));
  cudaError_t e = ok ? cudaSuccess : cudaErrorMemoryAllocation;
  if (e == cudaSuccess) e = cudaMemset(ix->list_off, 0, sizeof(int64_t) * (nlist + 1));
  if (e == cudaSuccess) e = cudaMemset(ix->cnorm, 0, sizeof(float) * ((size_t)(nlist + 127) / 128 * 128));
  if (e == cudaSuccess) {
    float t[256];
    for (int c = 0; c < 256; ++c) t[c] = ((float)c + 0.5f) / 255.0f;  // oracle.sq8_decode's first two ops
    e = cudaMemcpy(ix->sq8_t, t, sizeof t, cudaMemcpyHostToDevice);
  }
  if (e == cudaSuccess) e = cudaMemset(ix->vmin, 0, sizeof(float) * ix->dpad);
  if (e == cudaSuccess) e = cudaMemset(ix->vdiff, 0, sizeof(float) * ix->dpad);
  if (e != cudaSuccess) {
    mv_index_destroy(ix);
    return from_cuda(e, "create");
  }
  size_t fr = 0, tot = 0;
  if (cudaMemGetInfo(&fr, &tot) == cudaSuccess) ix->auto_budget = (int64_t)(fr / 2);
  *out = ix;
  return MV_OK;
}

mv_status mv_index_set_option(mv_index* ix, const char* name, int64_t value) {
  if (!ix || !name) return fail(MV_EINVAL, "null argument");
  if (value < 0) return fail(MV_EINVAL, "option %s: value must be >= 0", name);
  Options& o = ix->opt;
  const std::string n(name);
  if (n == "seeding") o.seeding = value != 0;
  else if (n == "need") o.need = value;
  else if (n == "capa") o.capa = value;
  else if (n == "sq8_qc") o.sq8_qc = (int)std::min<int64_t>(value, 64);
  else if (n == "flat_qc") o.flat_qc = (int)std::min<int64_t>(value, 128);
  else if (n == "coarse_nqb") o.coarse_nqb = (int)std::min<int64_t>(value, 128);
  else if (n == "coarse_cs") o.coarse_cs = (int)std::min<int64_t>(value, 64);
  else if (n == "coarse_epi") o.coarse_epi = (int)std::min<int64_t>(value, 16);
  else if (n == "coarse_nacc") o.coarse_nacc = (int)std::min<int64_t>(value, 4);
  else if (n == "workspace_bytes") o.workspace = value;
  else if (n == "scan_trace") o.scan_trace = value;  // development builds only (-DMV_SCAN_TRACE)
  else if (n == "async_host") o.async_host = value != 0;
  else if (n == "large_k_select") o.large_k_select = (int)std::min<int64_t>(std::max<int64_t>(value, 0), 4);
  else if (n == "big_cap") o.big_cap = std::max<int64_t>(value, 0);
  else if (n == "big_ctas") o.big_ctas = (int)std::min<int64_t>(std::max<int64_t>(value, 0), 4);
  else return fail(MV_EINVAL, "unknown option '%s'", name);
  return MV_OK;
}

void mv_index_destroy(mv_index* ix) {
  if (!ix) return;
  DeviceGuard g(ix->device);
  cudaDeviceSynchronize();
  free_storage(ix);
  for (cudaEvent_t e : ix->ev) cudaEventDestroy(e);
  mem_free(ix, ix->list_off, nullptr);
  mem_free(ix, ix->cpad, nullptr);
  mem_free(ix, ix->cnorm, nullptr);
  mem_free(ix, ix->chl, nullptr);
  mem_free(ix, ix->vmin, nullptr);
  mem_free(ix, ix->vdiff, nullptr);
  mem_free(ix, ix->sq8_t, nullptr);
  mem_free(ix, ix->pq_cb, nullptr);
  cudaFree(ix->d_count);
  delete ix;
}

mv_status mv_index_set_centroids(mv_index* ix, const float* centroids) {
  if (!ix || !centroids) return fail(MV_EINVAL, "null argument");
  if (ix->ntotal > 0) return fail(MV_ESTATE, "centroids cannot change after vectors were added");
  DeviceGuard g(ix->device);
  cudaStream_t st = 0;
  Scratch s(ix, st);
  bool staged;
  const float* c;
  CK(stage_in(s, centroids, (size_t)ix->nlist * ix->d, &c, &staged));
  CK(launch_centroid_prep(c, ix->nlist, ix->d, ix->dpad, ix->cpad, ix->cnorm, st));
  CK(launch_hilo(c, ix->nlist, ix->d, ix->dpad, ix->chl, nullptr, st));
  CK(cudaStreamSynchronize(st));
  if (!make_tmap_2d(&ix->cmap, ix->chl, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, (uint64_t)ix->dpad, 2 * (uint64_t)ix->nlist,
                    (uint64_t)ix->dpad * 4, 32, 128, CU_TENSOR_MAP_SWIZZLE_128B))
    return fail(MV_ECUDA, "set_centroids: cannot encode the centroid tensor map");
  ix->has_centroids = true;
  return MV_OK;
}

mv_status mv_index_train_sq8(mv_index* ix, const float* sample, int64_t n) {
  if (!ix || !sample) return fail(MV_EINVAL, "null argument");
  if (ix->type != MV_IVF_SQ8) return fail(MV_ESTATE, "train_sq8 on a non-SQ8 index");
  if (n < 1) return fail(MV_EINVAL, "train_sq8 needs n >= 1");
  if (ix->ntotal > 0) return fail(MV_ESTATE, "SQ8 parameters cannot change after vectors were added");
  DeviceGuard g(ix->device);
  cudaStream_t st = 0;
  Scratch s(ix, st);
  bool staged;
  const float* x;
  CK(stage_in(s, sample, (size_t)n * ix->d, &x, &staged));
  CK(launch_sq8_minmax(x, n, ix->d, ix->vmin, ix->vdiff, st));
  CK(cudaStreamSynchronize(st));
  ix->has_sq8 = true;
  return MV_OK;
}

static mv_status pq_check(const mv_index* ix, int32_t M) {
  if (!ix) return fail(MV_EINVAL, "null index");
  if (ix->type != MV_IVF_PQ) return fail(MV_ESTATE, "PQ parameters on a non-IVF_PQ index");
  if (ix->ntotal > 0) return fail(MV_ESTATE, "PQ parameters cannot change after vectors were added");
  if (M < 4 || M > 64 || M % 4 || ix->d % M) return fail(MV_EINVAL, "M must divide d, be a multiple of 4 and <= 64");
  return MV_OK;
}

mv_status mv_index_set_pq(mv_index* ix, int32_t M, const float* codebooks) {
  mv_status v = pq_check(ix, M);
  if (v != MV_OK) return v;
  if (!codebooks) return fail(MV_EINVAL, "null codebooks");
  DeviceGuard g(ix->device);
  const size_t bytes = sizeof(float) * 256 * (size_t)ix->d;
  if (!ix->pq_cb && !(ix->pq_cb = (float*)mem_alloc(ix, bytes, nullptr)))
    return fail(MV_ENOMEM, "set_pq: cannot allocate the codebooks");
  CK(cudaMemcpy(ix->pq_cb, codebooks, bytes, cudaMemcpyDefault));
  ix->pq_m = M;
  ix->pq_dsub = ix->d / M;
  ix->has_pq = true;
  return MV_OK;
}

mv_status mv_index_get_pq(const mv_index* ix, int32_t* M, float* codebooks) {
  if (!ix) return fail(MV_EINVAL, "null index");
  if (ix->type != MV_IVF_PQ || !ix->has_pq) return fail(MV_ESTATE, "no PQ parameters");
  DeviceGuard g(ix->device);
  if (M) *M = ix->pq_m;
  if (codebooks) CK(cudaMemcpy(codebooks, ix->pq_cb, sizeof(float) * 256 * (size_t)ix->d, cudaMemcpyDefault));
  return MV_OK;
}

mv_status mv_index_train_pq(mv_index* ix, int32_t M, const float* sample, int64_t n, int32_t niter) {
  mv_status v = pq_check(ix, M);
  if (v != MV_OK) return v;
  if (!sample || n < 256) return fail(MV_EINVAL, "train_pq needs >= 256 sample rows");
  if (is_host_ptr(sample)) return fail(MV_EINVAL, "train_pq: device sample only");
  DeviceGuard g(ix->device);
  const int dsub = ix->d / M;
  float *sub = nullptr, *cb = nullptr;
  CK(cudaMalloc(&sub, sizeof(float) * (size_t)n * dsub));
  struct F {
    float** a;
    float** b;
    ~F() { cudaFree(*a); cudaFree(*b); }
  } f{&sub, &cb};
  CK(cudaMalloc(&cb, sizeof(float) * 256 * (size_t)ix->d));
  for (int m = 0; m < M; ++m) {  // k-means of each sub-space, 256 sub-centroids
    CK(cudaMemcpy2D(sub, sizeof(float) * dsub, sample + m * dsub, sizeof(float) * ix->d, sizeof(float) * dsub, n,
                    cudaMemcpyDeviceToDevice));
    float* cbm = cb + (size_t)m * 256 * dsub;
    CK(cudaMemcpy(cbm, sub, sizeof(float) * 256 * dsub, cudaMemcpyDeviceToDevice));
    v = mv_kmeans(sub, n, dsub, MV_L2, 256, niter, 0, cbm, ix->device, nullptr);
    if (v != MV_OK) return v;
  }
  return mv_index_set_pq(ix, M, cb);
}

mv_status mv_index_set_sq8(mv_index* ix, const float* vmin, const float* vdiff) {
  if (!ix || !vmin || !vdiff) return fail(MV_EINVAL, "null argument");
  if (ix->type != MV_IVF_SQ8) return fail(MV_ESTATE, "set_sq8 on a non-SQ8 index");
  if (ix->ntotal > 0) return fail(MV_ESTATE, "SQ8 parameters cannot change after vectors were added");
  DeviceGuard g(ix->device);
  std::vector<float> hv(ix->d), hd(ix->d);
  CK(cudaMemcpy(hv.data(), vmin, sizeof(float) * ix->d, cudaMemcpyDefault));
  CK(cudaMemcpy(hd.data(), vdiff, sizeof(float) * ix->d, cudaMemcpyDefault));
  for (int j = 0; j < ix->d; ++j)
    if (!(hd[j] >= 0.0f)) return fail(MV_EINVAL, "vdiff[%d] must be >= 0", j);
  CK(cudaMemcpy(ix->vmin, hv.data(), sizeof(float) * ix->d, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(ix->vdiff, hd.data(), sizeof(float) * ix->d, cudaMemcpyHostToDevice));
  ix->has_sq8 = true;
  return MV_OK;
}

mv_status mv_index_get_sq8(const mv_index* ix, float* vmin, float* vdiff) {
  if (!ix) return fail(MV_EINVAL, "null index");
  if (ix->type != MV_IVF_SQ8 || !ix->has_sq8) return fail(MV_ESTATE, "no SQ8 parameters");
  DeviceGuard g(ix->device);
  if (vmin) CK(cudaMemcpy(vmin, ix->vmin, sizeof(float) * ix->d, cudaMemcpyDefault));
  if (vdiff) CK(cudaMemcpy(vdiff, ix->vdiff, sizeof(float) * ix->d, cudaMemcpyDefault));
  return MV_OK;
}

mv_status mv_index_add(mv_index* ix, const float* vectors, const int64_t* ids, int64_t n, void* stream) {
  if (!ix) return fail(MV_EINVAL, "null index");
  if (n < 0) return fail(MV_EINVAL, "n must be >= 0");
  if (n == 0) return MV_OK;
  if (!vectors || !ids) return fail(MV_EINVAL, "null vectors/ids");
  if (!ix->has_centroids) return fail(MV_ESTATE, "add before set_centroids");
  if (ix->type == MV_IVF_SQ8 && !ix->has_sq8) return fail(MV_ESTATE, "add on SQ8 index before train_sq8/set_sq8");
  if (ix->type == MV_IVF_PQ && !ix->has_pq) return fail(MV_ESTATE, "add on IVF_PQ index before train_pq/set_pq");
  if (n > 0x7fffffffLL) return fail(MV_EINVAL, "one add call takes at most 2^31-1 vectors");
  if (ix->ntotal + n > 0x7fffffffLL) return fail(MV_EINVAL, "an index holds at most 2^31-1 vectors");
  DeviceGuard g(ix->device);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  Scratch s(ix, st);
  bool sv, si;
  const float* x;
  const int64_t* idv;
  CK(stage_in(s, vectors, (size_t)n * ix->d, &x, &sv));
  CK(stage_in(s, ids, (size_t)n, &idv, &si));
  int* flag;
  CK(s.alloc(&flag, 1));
  CK(cudaMemsetAsync(flag, 0, sizeof(int), st));
  CK(launch_check_ids(idv, n, flag, st));
  int hflag = 0;
  CK(cudaMemcpyAsync(&hflag, flag, sizeof(int), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (hflag) return fail(MV_EINVAL, "id -1 is reserved (padding)");

  const int nlist = ix->nlist, dpad = ix->dpad;
  float *xpad, *xnorm;
  int32_t *lists, *cnt, *addoff, *idx, *sidx, *slist;
  int64_t *sizes, *new_off;
  CK(s.alloc(&xpad, (size_t)n * dpad));
  CK(s.alloc(&xnorm, (size_t)n));
  CK(s.alloc(&lists, (size_t)n));
  CK(s.alloc(&cnt, nlist));
  CK(s.alloc(&addoff, nlist + 1));
  CK(s.alloc(&idx, (size_t)n));
  CK(s.alloc(&sidx, (size_t)n));
  CK(s.alloc(&slist, (size_t)n));
  CK(s.alloc(&sizes, nlist));
  CK(s.alloc(&new_off, nlist + 1));
  // a0: assignment I(v) = closest centroid -- the tensor-core coarse step with nprobe = 1, in row
  // blocks whose group-minimum matrix stays <= 512 MB
  CK(launch_query_prep(x, n, ix->d, dpad, xpad, xnorm, st));
  {
    const int64_t ldg = ((nlist + 127) / 128) * 4;
    const int64_t sub = std::min<int64_t>(n, std::max<int64_t>(4096, (int64_t(1) << 27) / ldg));
    float* qhl;
    int* lo_any;  // the rows' lo planes vanish (integer data): the GEMM's wide mode
    CK(s.alloc(&qhl, (size_t)2 * sub * dpad));
    CK(s.alloc(&lo_any, 1));
    for (int64_t r0 = 0; r0 < n; r0 += sub) {
      const int64_t m = std::min(sub, n - r0);
      Scratch sb(ix, st);  // the block's coarse scratch, freed (stream-ordered) before the next block
      CK(cudaMemsetAsync(lo_any, 0, sizeof(int), st));
      CK(launch_hilo(x + r0 * ix->d, m, ix->d, dpad, qhl, lo_any, st));
      CK(run_coarse(ix, qhl, lo_any, m, 1, lists + r0, sb, st));
    }
  }
  CK(cudaMemsetAsync(cnt, 0, sizeof(int32_t) * nlist, st));
  CK(launch_count_lists(lists, n, cnt, st));
  CK(launch_scan_i32(cnt, nlist, addoff, st));
  // stable order of the new rows by list (radix sort is stable; values = input order)
  CK(launch_iota_i32(idx, n, st));
  int endbit = 1;
  while ((1 << endbit) < nlist && endbit < 31) ++endbit;
  size_t tmp_bytes = 0;
  CK(cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, (const uint32_t*)lists, (uint32_t*)slist, idx, sidx, (int)n, 0,
                                     endbit, st));
  uint8_t* tmp;
  CK(s.alloc(&tmp, tmp_bytes));
  CK(cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, (const uint32_t*)lists, (uint32_t*)slist, idx, sidx, (int)n, 0,
                                     endbit, st));
  CK(launch_new_sizes(cnt, nlist, ix->list_off, sizes, st));
  CK(launch_scan_i64(sizes, nlist, new_off, st));

  const int64_t ntot = ix->ntotal + n;
  const bool pq = ix->type == MV_IVF_PQ;
  const size_t esize = ix->type == MV_IVF_FLAT ? 4 : 1;
  const int prow = pq ? ix->pq_m : dpad;  // payload elements per row (PQ: M sub-codes)
  // per-row side arrays carry kSidePad zeroed tail elements: the scan bulk-copies 16-B aligned
  // supersets of 128-row tiles
  constexpr int64_t kSidePad = 256;
  mv_index nx;  // the new storage (only the pointers are used)
  nx.alloc = ix->alloc;
  nx.payload = mem_alloc(ix, (size_t)ntot * prow * esize + 16, st);
  nx.norms = (double*)mem_alloc(ix, sizeof(double) * (ntot + kSidePad), st);
  nx.ids = (int64_t*)mem_alloc(ix, sizeof(int64_t) * (ntot + kSidePad), st);
  nx.rank = (uint32_t*)mem_alloc(ix, sizeof(uint32_t) * (ntot + kSidePad), st);
  nx.sorted_ids = (int64_t*)mem_alloc(ix, sizeof(int64_t) * ntot, st);
  nx.row_of_rank = (uint32_t*)mem_alloc(ix, sizeof(uint32_t) * ntot, st);
  if (!nx.payload || !nx.norms || !nx.ids || !nx.rank || !nx.sorted_ids || !nx.row_of_rank) {
    free_storage(&nx);
    return fail(MV_ENOMEM, "add: cannot allocate storage for %lld vectors", (long long)ntot);
  }
  CK(cudaMemsetAsync(nx.norms + ntot, 0, sizeof(double) * kSidePad, st));
  CK(cudaMemsetAsync(nx.ids + ntot, 0, sizeof(int64_t) * kSidePad, st));
  CK(cudaMemsetAsync(nx.rank + ntot, 0, sizeof(uint32_t) * kSidePad, st));
  CK(launch_move_old(pq ? MV_IVF_SQ8 : ix->type, prow, nlist, ix->list_off, new_off, ix->payload, ix->norms, ix->ids,
                     ix->ntotal, nx.payload, nx.norms, nx.ids, st));
  if (pq)
    CK(launch_pq_encode(xpad, idv, sidx, slist, n, dpad, ix->pq_m, ix->pq_dsub, ix->pq_cb, new_off, ix->list_off, addoff,
                        reinterpret_cast<uint8_t*>(nx.payload), nx.norms, nx.ids, st));
  else
    CK(launch_store_rows(ix->type, ix->metric, xpad, idv, sidx, slist, n, dpad, new_off, ix->list_off, addoff,
                         nx.payload, nx.norms, nx.ids, ix->vmin, ix->vdiff, ix->sq8_t, st));
  // id ranks: stable radix sort of (id) over storage rows -> (id, row) order
  uint64_t *keys, *skeys;
  uint32_t *vals, *svals;
  CK(s.alloc(&keys, (size_t)ntot));
  CK(s.alloc(&skeys, (size_t)ntot));
  CK(s.alloc(&vals, (size_t)ntot));
  CK(s.alloc(&svals, (size_t)ntot));
  CK(launch_id_keys(nx.ids, ntot, keys, vals, st));
  size_t tmp2 = 0;
  CK(cub::DeviceRadixSort::SortPairs(nullptr, tmp2, keys, skeys, vals, svals, (int64_t)ntot, 0, 64, st));
  uint8_t* t2;
  CK(s.alloc(&t2, tmp2));
  CK(cub::DeviceRadixSort::SortPairs(t2, tmp2, keys, skeys, vals, svals, (int64_t)ntot, 0, 64, st));
  CK(launch_rank_scatter(skeys, svals, ntot, nx.rank, nx.sorted_ids, nx.row_of_rank, st));
  int* idflag;
  CK(s.alloc(&idflag, 1));
  CK(cudaMemsetAsync(idflag, 0, sizeof(int), st));
  CK(launch_check_identity(nx.sorted_ids, ntot, idflag, st));
  int hid = 1;
  CK(cudaMemcpyAsync(&hid, idflag, sizeof(int), cudaMemcpyDeviceToHost, st));
  unsigned long long* xm;
  CK(s.alloc(&xm, 1));
  unsigned long long hxm = 0;
  if (ix->type == MV_IVF_FLAT) {
    CK(cudaMemsetAsync(flag, 0, sizeof(int), st));
    CK(launch_tf32_check(xpad, (int64_t)n * dpad, flag, st));
    CK(cudaMemcpyAsync(&hflag, flag, sizeof(int), cudaMemcpyDeviceToHost, st));
  }
  CK(cudaMemsetAsync(xm, 0, sizeof(unsigned long long), st));
  CK(launch_max_f64(nx.norms, ntot, xm, st));
  CK(cudaMemcpyAsync(&hxm, xm, sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
  CK(cudaMemcpyAsync(ix->list_off, new_off, sizeof(int64_t) * (nlist + 1), cudaMemcpyDeviceToDevice, st));
  CK(cudaMemcpyAsync(ix->h_list_off.data(), new_off, sizeof(int64_t) * (nlist + 1), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  free_storage(ix);
  ix->payload = nx.payload;
  ix->norms = nx.norms;
  ix->ids = nx.ids;
  ix->rank = nx.rank;
  ix->sorted_ids = nx.sorted_ids;
  ix->row_of_rank = nx.row_of_rank;
  nx.payload = nx.norms = nullptr;
  nx.ids = nx.sorted_ids = nullptr;
  nx.rank = nx.row_of_rank = nullptr;
  ix->ntotal = ntot;
  ix->ids_identity = hid == 0;
  if (ix->type == MV_IVF_FLAT && hflag) ix->tf32_exact = false;
  double xm2;
  memcpy(&xm2, &hxm, sizeof xm2);
  ix->xmax2 = xm2;
  // one swizzle atom per box row: 128 B (FLAT: 32 fp32; SQ8 when dpad is a multiple of 128), else 32 B
  const bool wide = ix->type == MV_IVF_FLAT || dpad % 128 == 0;
  for (int i = 0; i < 4 && !pq; ++i)
    if (!make_tmap_2d(&ix->xm.m[i], ix->payload,
                      ix->type == MV_IVF_FLAT ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_UINT8,
                      (uint64_t)dpad, (uint64_t)ntot, (uint64_t)dpad * esize, ix->type == MV_IVF_FLAT ? 32 : (wide ? 128 : 32),
                      128 >> i, wide ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_32B))
      return fail(MV_ECUDA, "add: cannot encode the payload tensor map");
  ix->maxlen = 0;
  std::vector<int64_t> lens(nlist);
  for (int l = 0; l < nlist; ++l) {
    lens[l] = ix->h_list_off[l + 1] - ix->h_list_off[l];
    ix->maxlen = std::max(ix->maxlen, lens[l]);
  }
  std::sort(lens.begin(), lens.end(), std::greater<int64_t>());
  ix->top_len_prefix.assign(nlist + 1, 0);
  for (int l = 0; l < nlist; ++l) ix->top_len_prefix[l + 1] = ix->top_len_prefix[l] + lens[l];
  size_t fr = 0, tot = 0;
  if (cudaMemGetInfo(&fr, &tot) == cudaSuccess) ix->auto_budget = (int64_t)(fr / 2);
  return MV_OK;
}

static mv_status validate_search(const mv_index* ix, const float* q, int64_t nq, int32_t k, int32_t nprobe,
                                 const void* d, const void* i) {
  if (!ix) return fail(MV_EINVAL, "null index");
  if (nq < 0) return fail(MV_EINVAL, "nq must be >= 0");
  if (k < 1 || k > kMaxK) return fail(MV_EINVAL, "k must be in [1, %d] (got %d)", kMaxK, k);
  if (nprobe < 1) return fail(MV_EINVAL, "nprobe must be >= 1 (got %d)", nprobe);
  const int npb = std::min(nprobe, ix->nlist);
  if (npb < ix->nlist && npb > kMaxNprobe)
    return fail(MV_EINVAL, "nprobe must be <= %d or >= nlist (got %d)", kMaxNprobe, nprobe);
  if (nq > 0 && (!q || !d || !i)) return fail(MV_EINVAL, "null queries/outputs");
  if (!ix->has_centroids) return fail(MV_ESTATE, "search before set_centroids");
  return MV_OK;
}

mv_status mv_search_probes(mv_index* ix, const float* queries, int64_t nq, int32_t nprobe, int32_t* probes,
                           void* stream) {
  mv_status v = validate_search(ix, queries, nq, 1, nprobe, probes, probes);
  if (v != MV_OK) return v;
  if (nq == 0) return MV_OK;
  DeviceGuard g(ix->device);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  const int npb = std::min(nprobe, ix->nlist);
  bool sq;
  Scratch s0(ix, st);
  const float* q;
  CK(stage_in(s0, queries, (size_t)nq * ix->d, &q, &sq));
  const bool sp = is_host_ptr(probes);
  // chunks of queries whose coarse scratch stays <= 1 GB
  const int64_t per = (int64_t)ix->nlist / 8 + 256 * (int64_t)npb + 8 * (int64_t)ix->dpad + 64;
  const int64_t chunk = std::max<int64_t>(1, std::min<int64_t>(nq, (int64_t(1) << 30) / per));
  for (int64_t q0 = 0; q0 < nq; q0 += chunk) {
    const int64_t m = std::min(chunk, nq - q0);
    Scratch s(ix, st);
    int32_t* P = probes + q0 * npb;
    if (sp) CK(s.alloc(&P, (size_t)m * npb));
    float* qhl;
    int* lo_any;
    CK(s.alloc(&qhl, (size_t)2 * m * ix->dpad));
    CK(s.alloc(&lo_any, 1));
    CK(cudaMemsetAsync(lo_any, 0, sizeof(int), st));
    CK(launch_hilo(q + q0 * ix->d, m, ix->d, ix->dpad, qhl, lo_any, st));
    CK(run_coarse(ix, qhl, lo_any, m, npb, P, s, st));
    if (sp) CK(cudaMemcpyAsync(probes + q0 * npb, P, sizeof(int32_t) * m * npb, cudaMemcpyDeviceToHost, st));
  }
  if (sp || sq) CK(cudaStreamSynchronize(st));
  return MV_OK;
}

// One chunk of queries through the whole pipeline (a1 .. a7).  q: device queries [nq][d];
// P_in: caller probes [nq][npb] (device) or nullptr; bs: device bitset or nullptr.
static mv_status search_chunk(mv_index* ix, const float* q, int64_t nq, int32_t k, int npb, const int32_t* P_in,
                              const uint8_t* bs, int64_t nbits, float* D, int64_t* I, cudaStream_t st) {
  Scratch s(ix, st);
  const int nlist = ix->nlist, dpad = ix->dpad;
  const bool flat = ix->type == MV_IVF_FLAT;
  const bool pq = ix->type == MV_IVF_PQ;  // the query-major ADC scan (k_pq.cu) instead of k_scan_tc
  const int64_t* idmap = ix->ids_identity ? nullptr : ix->sorted_ids;  // rank -> id (nullptr: identity)
  // a1 + a2/a3
  prof_mark(ix, st);
  float *qpad, *qnorm;
  int32_t* P;
  CK(s.alloc(&qpad, (size_t)nq * dpad));
  CK(s.alloc(&qnorm, (size_t)nq));
  if (P_in) P = const_cast<int32_t*>(P_in);
  else CK(s.alloc(&P, (size_t)nq * npb));
  CK(launch_query_prep(q, nq, ix->d, dpad, qpad, qnorm, st));
  float* qhl;  // plane-major tf32 hi/lo query planes: coarse B operand and the FLAT scan's query planes
  CK(s.alloc(&qhl, (size_t)2 * nq * dpad));
  int* qlo_any;  // does any query need its lo plane (not tf32-exact)?  Decides the FLAT scan shape
  CK(s.alloc(&qlo_any, 1));
  CK(cudaMemsetAsync(qlo_any, 0, sizeof(int), st));
  CK(launch_hilo(q, nq, ix->d, dpad, qhl, qlo_any, st));
  if (!P_in) CK(run_coarse(ix, qhl, qlo_any, nq, npb, P, s, st));
  prof_mark(ix, st);
  // a4 (the work-item shape follows the scan's shared-memory plan)
  TcScanParams tp;
  // (IVF_PQ: the planner's pair regions and seeding lists are used, its work items are not)
  if (!tc_scan_plan(pq ? (int)MV_IVF_SQ8 : ix->type, dpad, k, (double)nq * npb / std::max(1, nlist), bs != nullptr,
                    ix->opt, tp))
    return fail(MV_EINVAL, "search: no tensor-core scan plan fits d = %d", ix->d);
  const int qchunk = tp.qchunk;
  const int qchunk_min = tp.qchunk_split;  // FLAT two-plane items
  int32_t* qcfg;
  CK(s.alloc(&qcfg, 2));
  const int64_t npairs = nq * npb;
  // Seeding (nprobe >= 2): phase A scans the first capA rows of each query's ra[q] nearest lists --
  // the fewest holding >= need such rows -- and emits all of them; their k-th best key tau_q bounds
  // the query's final k-th best (k distinct candidates are at or below it), so phase B scans every
  // probed list and emits only keys <= tau_q.
  const bool split = npb >= 2 && ix->opt.seeding;
  int32_t* ra = nullptr;
  if (split) CK(s.alloc(&ra, (size_t)nq));
  const int nv = split ? 2 * nlist : nlist;
  Bucketing b;
  CK(s.alloc(&b.lcount, nv));
  CK(s.alloc(&b.boff, nv + 1));
  CK(s.alloc(&b.bfill, nv));
  const int64_t nent = split ? 2 * npairs : npairs;  // bucket entries (phase-A entries with seeding)
  CK(s.alloc(&b.bq, (size_t)nent));
  CK(s.alloc(&b.wcount, nv));
  CK(s.alloc(&b.woff, nv + 1));
  CK(s.alloc(&b.witems, (size_t)(nv + nent / qchunk_min + 1)));
  CK(s.alloc(&b.qtot, (size_t)(2 * (nq + 1))));
  CK(s.alloc(&b.poff, (size_t)nent));
  CK(s.alloc(&b.pcnt, (size_t)nent));
  CK(s.alloc(&b.counter, 2));
  CK(s.alloc(&b.whist, (size_t)kPlanCostBins));
  CK(s.alloc(&b.bsum, (size_t)(2 * kPlanMaxBlocks)));
  PlanArgs pa;
  pa.probes = P; pa.nq = nq; pa.npb = npb; pa.nlist = nlist; pa.k = k;
  pa.split = split ? 1 : 0; pa.need = std::max<int64_t>(2 * (int64_t)k, k + 32);
  // Sample size of the seeding phase.  tau_q = the k-th best of `need` candidates is about the
  // (k N / need)-th best of the query's N candidates, so phase B emits ~k N / need keys.  Phase A
  // costs ~need rows of payload, an emission ~a fixed number of bytes (the key store, the final
  // select's reads); balancing the two gives need ~ sqrt(k N c / rowbytes).  c is measured
  // (DESIGN.md §5): 96 B for k <= 256 (round-2 sweep on the current kernels: configs[2] need 1200
  // vs 806 2.13 vs 2.20 ms, configs[4] 1000 vs 552 5.86 vs 5.94 ms; round 1 measured 32 B); the
  // CTA-per-query select for k > 256 costs ~26x more per candidate, c = 832 B.
  {
    const double ncand = (double)ix->ntotal * npb / std::max(1, nlist);
    const double rowb = pq ? (double)ix->pq_m : (double)dpad * (flat ? 4 : 1);
    const double c = k > 256 ? 832.0 : (pq ? 32.0 : 96.0);  // (IVF_PQ's query-major scan: 32 B, c3pq 4.10 vs 4.25 ms)
    const int64_t bal = (int64_t)std::sqrt((double)k * ncand * c / rowb);
    pa.need = std::max<int64_t>(pa.need, std::min<int64_t>(bal, 65536));
  }
  if (ix->opt.need > 0) pa.need = std::max<int64_t>(2 * (int64_t)k, ix->opt.need);
  // Rows per list of the sample: ~sqrt(f need), i.e. the sample spreads over ~sqrt(need / f)
  // nearest lists, at least 128 rows.  f = 64 (configs[3]: capA 1024 best of 128..1024;
  // configs[2], k = 100: 240 rows, 464 measured 5% slower); f = 256 for k <= 32 (round-2 sweep:
  // configs[4] capA 384 vs 192: 7.68 vs 7.90 ms; configs[1] unchanged: its sample is 128 rows)
  const double capf = k <= 32 ? 256.0 : 64.0;
  pa.capA = std::max<int64_t>(128, std::min<int64_t>((pa.need + 15) & ~(int64_t)15,
                                                     ((int64_t)std::sqrt(capf * pa.need) + 15) & ~(int64_t)15));
  if (ix->opt.capa > 0) pa.capA = std::max<int64_t>(16, (ix->opt.capa + 15) & ~15ll);
  pa.list_off = ix->list_off;
  // FLAT with tf32-exact stored values: two-plane (hi/lo) items when some query needs its lo plane;
  // other FLAT data always take one-plane items (the stored side's tf32 error dominates)
  pa.qlo_any = (flat && ix->tf32_exact) ? qlo_any : nullptr;
  pa.qc_exact = qchunk; pa.p_exact = flat ? 1 : kSq8Planes;
  pa.qc_split = qchunk_min; pa.p_split = flat ? 2 : kSq8Planes;
  pa.qcfg = qcfg; pa.ra = ra; pa.b = b;
  CK(launch_plan(pa, st));
  prof_mark(ix, st);
  // candidate regions: the worst case without a device round trip, nq x (the npb longest lists)
  // (+ the phase-A prefixes: < need + capA rows per query); the chunking bounds it
  const int64_t tmax = ix->top_len_prefix[std::min<size_t>(npb, ix->top_len_prefix.size() - 1)];
  int64_t cap = nq * tmax;
  if (split) cap += nq * std::min<int64_t>(tmax, pa.need + pa.capA);
  uint8_t* over = nullptr;
  uint64_t* kmin = nullptr;  // k > 256 with seeding: each query's smallest phase-A key (streaming select)
  if (k > 256) CK(s.alloc(&over, (size_t)2 * nq));
  if (k > 256 && split) {
    CK(s.alloc(&kmin, (size_t)nq));
    CK(cudaMemsetAsync(kmin, 0, sizeof(uint64_t) * nq, st));  // (a query the seeding select skips: bins from 0)
  }
  uint64_t* part;
  CK(s.alloc(&part, (size_t)max64(cap, 1)));
  // a5/a6 on the tensor cores
  uint8_t* qplanes;
  float *qscale, *qerr = nullptr;
  double *qa, *qn64;
  uint64_t* tau;
  if (!flat && !pq) CK(s.alloc(&qplanes, (size_t)nq * kSq8Planes * dpad));
  else qplanes = reinterpret_cast<uint8_t*>(qhl);
  CK(s.alloc(&qscale, (size_t)nq));
  CK(s.alloc(&qa, (size_t)nq));
  CK(s.alloc(&qn64, (size_t)nq));
  CK(s.alloc(&tau, (size_t)nq));
  CK(cudaMemsetAsync(tau, 0xff, sizeof(uint64_t) * nq, st));
  // filter mode: the tensor-core badness carries a rigorous error bound E_q -- SQ8
  // always, FLAT when the stored values (always) or the queries (device flag) are not tf32-exact;
  // the keys are then re-scored exactly before the final select
  const bool approx_always = !flat || !ix->tf32_exact;
  const int* gate = approx_always ? nullptr : qlo_any;
  FlatErr fe{ix->tf32_exact ? 0.0 : 0x1p-10, ix->tf32_exact ? 0x1p-21 : 0x1p-11, ix->xmax2, ix->metric};
  CK(s.alloc(&qerr, (size_t)nq));
  if (!pq)
    CK(launch_qplanes(ix->type, qpad, nq, dpad, ix->vmin, ix->vdiff, flat ? nullptr : qplanes, qscale, qa, qn64, &fe,
                      qerr, st));
  PqScanParams pp{};
  if (pq) {
    pp.metric = ix->metric; pp.dpad = dpad; pp.M = ix->pq_m; pp.dsub = ix->pq_dsub; pp.npb = npb; pp.nq = nq;
    pp.qpad = qpad; pp.codebooks = ix->pq_cb; pp.probes = P; pp.ra = ra; pp.tau = tau; pp.list_off = ix->list_off;
    pp.codes = reinterpret_cast<const uint8_t*>(ix->payload); pp.rank = ix->rank; pp.ids = ix->ids;
    pp.bitset = bs; pp.nbits = bs ? nbits : 0; pp.poff = b.poff; pp.pcnt = b.pcnt; pp.part = part;
  }
  tp.metric = ix->metric; tp.npb = npb; tp.nq = nq;
  tp.list_off = ix->list_off; tp.norms = ix->norms; tp.ids = ix->ids; tp.rank = ix->rank;
  tp.bitset = bs; tp.nbits = bs ? nbits : 0;
  tp.qplanes = qplanes; tp.qnorm = qn64; tp.qscale = qscale; tp.qa = qa;
  tp.bq = b.bq; tp.nbq = nent; tp.boff = b.boff; tp.witems = b.witems; tp.nlist = nlist; tp.cfg = qcfg;
  tp.poff = b.poff; tp.pcnt = b.pcnt; tp.part = part; tp.tau = tau;
  tp.approx_always = approx_always ? 1 : 0; tp.qerr = qerr;
  // k > 256 with seeding: phase A emits 4-byte distance keys and k_tau32 takes the bound from them
  // (half the sample's bytes written and read; large_k_select = 2 keeps the 8-byte keys)
  const bool key32 = k > 256 && split && !pq && (ix->opt.large_k_select == 0 || ix->opt.large_k_select == 4);
  tp.key32 = key32 ? 1 : 0;
  tp.prof = nullptr;
  // phase A (or, without seeding, the whole scan emitting every candidate) ...
  tp.phase = 0;
  tp.rowcap = split ? (int)pa.capA : 0x7fffffff;
  tp.wbeg = nullptr;
  tp.nwitems = b.woff + nlist;
  tp.counter = b.counter;
  if (pq) {
    pp.phase = split ? 0 : 1;  // without seeding: one pass over every pair, everything emitted (tau = pad)
    pp.rowcap = split ? (int)pa.capA : 0x7fffffff;
    CK(launch_pq_scan(pp, st));
  } else {
    CK(launch_scan_tc(ix->xm, tp, st));
  }
  prof_mark(ix, st);
  if (split) {
    // ... tau_q = k-th best key of phase A (phase A emits < need + capA candidates per query) ...
    if (key32)
      CK(launch_tau32(b.poff + npairs, b.pcnt + npairs, part, nq, npb, ra, k, tau, kmin,
                      std::min<int64_t>(tmax, pa.need + pa.capA), st));
    else
    CK(launch_tau_select(b.poff + npairs, b.pcnt + npairs, part, nq, npb, ra, k, tau,
                         std::min<int64_t>(tmax, pa.need + pa.capA), over, nullptr,
                         BigSel{ix->opt.large_k_select, ix->opt.big_ctas, ix->opt.big_cap, std::min<int64_t>(tmax, pa.need),
                                kmin, nullptr},
                         st));
    prof_mark(ix, st);
    // ... phase B over every probed pair, emitting keys <= tau_q
    tp.phase = 1;
    tp.prof = reinterpret_cast<unsigned long long*>(ix->opt.scan_trace);
    tp.rowcap = 0x7fffffff;
    tp.wbeg = b.woff + nlist;
    tp.nwitems = b.woff + 2 * nlist;
    tp.counter = b.counter + 1;
    if (pq) {
      pp.phase = 1;
      pp.rowcap = 0x7fffffff;
      CK(launch_pq_scan(pp, st));
    } else {
      CK(launch_scan_tc(ix->xm, tp, st));
    }
  } else {
    prof_mark(ix, st);
  }
  prof_mark(ix, st);
  if (ix->prof) {  // emission counters (mv_profile_counters): what the selects have to read
    if (!ix->d_count) {
      CK(cudaMalloc(&ix->d_count, 4 * sizeof(unsigned long long)));
      CK(cudaMemset(ix->d_count, 0, 4 * sizeof(unsigned long long)));
    }
    CK(launch_count_add(nq, ix->d_count, st));
    if (split) CK(launch_sum_i32(b.pcnt + npairs, npairs, npb, ra, ix->d_count + 1, st));
    CK(launch_sum_i32(b.pcnt, npairs, npb, nullptr, ix->d_count + 2, st));
  }
  if (pq) {
    // IVF_PQ: the keys are the asymmetric distances themselves -- the plain exact select
    CK(launch_final_select(b.poff, b.pcnt, part, nq, npb, k, ix->metric, idmap, D, I, tmax, over,
                           BigSel{ix->opt.large_k_select, ix->opt.big_ctas, ix->opt.big_cap, 0, kmin, tau}, st));
  } else if (k <= 256) {
    // a7 with the filter mode's exact re-scoring fused in (a plain exact select when the search is
    // exact: FLAT with tf32-exact data and queries, gate = qlo_any == 0 on the device)
    uint64_t* tau2;
    int* notgate;
    CK(s.alloc(&tau2, (size_t)nq));
    CK(s.alloc(&notgate, 1));
    CK(launch_final_refine(ix->type, b.poff, b.pcnt, part, nq, npb, k, ix->metric, idmap, D, I, qerr, qpad,
                           dpad, ix->payload, ix->row_of_rank, ix->vmin, ix->vdiff, ix->sq8_t, gate, tau2, notgate, st));
  } else {
    // filter mode: t~_q = the k-th best approximate key, exact re-scoring in place of the keys within
    // 2 E_q of it (both skipped on the device when the search is exact), then a7
    uint64_t* tau2;
    CK(s.alloc(&tau2, (size_t)nq));
    CK(cudaMemsetAsync(tau2, 0xff, sizeof(uint64_t) * nq, st));
    CK(launch_tau_select(b.poff, b.pcnt, part, nq, npb, nullptr, k, tau2, tmax, over, gate,
                         BigSel{ix->opt.large_k_select, ix->opt.big_ctas, ix->opt.big_cap, 0}, st));
    CK(launch_rekey(ix->type, b.poff, b.pcnt, part, nq, npb, tau2, qerr, ix->metric, qpad, dpad, ix->payload,
                    ix->row_of_rank, ix->vmin, ix->vdiff, ix->sq8_t, gate, st));
    ix->launches += 2;
    CK(launch_final_select(b.poff, b.pcnt, part, nq, npb, k, ix->metric, idmap, D, I, tmax, over,
                           BigSel{ix->opt.large_k_select, ix->opt.big_ctas, ix->opt.big_cap, 0, kmin, tau}, st));
  }
  prof_mark(ix, st);
  ix->last_scan = pq ? "simt.pq_adc" : (flat ? "tcgen05.tf32" : "tcgen05.i8");
  // prep, hilo, coarse (GEMM pass 0, group bound, GEMM pass 1, top-nprobe | all lists), plan, qplanes,
  // scan A (+ seed select, scan B), final select
  ix->launches += 5 + (P_in ? 0 : (npb >= nlist ? 1 : 4)) + (split ? 2 : 0) + 1;
  return MV_OK;
}

static mv_status search_impl(mv_index* ix, const float* queries, int64_t nq, int32_t k, int32_t nprobe,
                             const int32_t* probes_in, const uint8_t* bitset, int64_t nbits, float* distances,
                             int64_t* out_ids, void* stream) {
  mv_status v = validate_search(ix, queries, nq, k, nprobe, distances, out_ids);
  if (v != MV_OK) return v;
  if (nbits < 0) return fail(MV_EINVAL, "nbits must be >= 0");
  if (nq == 0) return MV_OK;
  if (bitset == nullptr) nbits = 0;
  DeviceGuard g(ix->device);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  Scratch s(ix, st);
  const int npb = std::min(nprobe, ix->nlist);
  bool sq = false, sb = false, sp = false;
  const float* q;
  const uint8_t* bs = nullptr;
  const int32_t* P = nullptr;
  CK(stage_in(s, queries, (size_t)nq * ix->d, &q, &sq));
  if (bitset && nbits > 0) CK(stage_in(s, bitset, (size_t)((nbits + 7) / 8), &bs, &sb));
  if (probes_in) CK(stage_in(s, probes_in, (size_t)nq * npb, &P, &sp));
  const bool host_out = is_host_ptr(distances) || is_host_ptr(out_ids);
  float* D = distances;
  int64_t* I = out_ids;
  if (host_out) {
    CK(s.alloc(&D, (size_t)nq * k));
    CK(s.alloc(&I, (size_t)nq * k));
  }
  if (ix->ntotal == 0) {
    CK(launch_fill_pad((int64_t)nq * k, ix->metric, D, I, st));
  } else {
    // query chunks: each one's scratch (candidate regions, score matrix, ...) within the budget,
    // and < 2^29 (query, list) pairs (int32 pair ids with the seeding phase's second copy)
    int64_t budget = ix->opt.workspace > 0 ? ix->opt.workspace : std::max<int64_t>(ix->auto_budget, 1 << 30);
    const int64_t per = search_bytes_per_query(ix, npb, k);
    int64_t chunk = std::min<int64_t>(nq, std::max<int64_t>(1, budget / std::max<int64_t>(per, 1)));
    chunk = std::min<int64_t>(chunk, std::max<int64_t>(1, (int64_t(1) << 29) / npb));
    ix->last_chunks = 0;
    for (int64_t q0 = 0; q0 < nq; q0 += chunk) {
      const int64_t m = std::min(chunk, nq - q0);
      mv_status r = search_chunk(ix, q + q0 * ix->d, m, k, npb, P ? P + q0 * npb : nullptr, bs, nbits,
                                 D + q0 * k, I + q0 * k, st);
      if (r != MV_OK) return r;
      ix->last_chunks++;
    }
    if (ix->prof) ix->prof_searches++;
  }
  if (host_out) {
    CK(cudaMemcpyAsync(distances, D, sizeof(float) * nq * k, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(out_ids, I, sizeof(int64_t) * nq * k, cudaMemcpyDeviceToHost, st));
  }
  // host inputs/outputs: the call completes before returning (mv.h) -- unless the caller asked for
  // stream-ordered host I/O (option "async_host") and every host buffer is page-locked: then the
  // copies are ordered on `stream` like the kernels (a serving loop overlaps one batch's copies
  // with another batch's search on a second stream)
  const bool async_io = ix->opt.async_host && is_pinned_ptr(queries) && is_pinned_ptr(distances) &&
                        is_pinned_ptr(out_ids) && (!bitset || is_pinned_ptr(bitset)) &&
                        (!probes_in || is_pinned_ptr(probes_in));
  if ((host_out || sq || sb || sp) && !async_io) CK(cudaStreamSynchronize(st));
  return MV_OK;
}

mv_status mv_search(mv_index* ix, const float* queries, int64_t nq, int32_t k, int32_t nprobe, const uint8_t* bitset,
                    int64_t nbits, float* distances, int64_t* out_ids, void* stream) {
  return search_impl(ix, queries, nq, k, nprobe, nullptr, bitset, nbits, distances, out_ids, stream);
}

mv_status mv_search_with_probes(mv_index* ix, const float* queries, int64_t nq, int32_t k, int32_t nprobe,
                                const int32_t* probes, const uint8_t* bitset, int64_t nbits, float* distances,
                                int64_t* out_ids, void* stream) {
  if (probes == nullptr && nq > 0) return fail(MV_EINVAL, "probes is NULL");
  return search_impl(ix, queries, nq, k, nprobe, probes, bitset, nbits, distances, out_ids, stream);
}

mv_status mv_kmeans(const float* x, int64_t n, int32_t d, mv_metric metric, int32_t nlist, int32_t niter,
                    int32_t spherical, float* centroids, int32_t device, void* stream) {
  if (!x || !centroids) return fail(MV_EINVAL, "null argument");
  if (n < nlist || nlist < 1) return fail(MV_EINVAL, "k-means needs 1 <= nlist <= n (n = %lld, nlist = %d)",
                                          (long long)n, nlist);
  if (niter < 0) return fail(MV_EINVAL, "niter must be >= 0");
  if (n > 0x7fffffffLL) return fail(MV_EINVAL, "at most 2^31-1 training rows");
  if (is_host_ptr(x) || is_host_ptr(centroids)) return fail(MV_EINVAL, "device pointers only");
  mv_index* ix = nullptr;
  mv_status v = mv_index_create(d, metric, MV_IVF_FLAT, nlist, device, nullptr, &ix);
  if (v != MV_OK) return v;
  struct Closer {
    mv_index* p;
    ~Closer() { mv_index_destroy(p); }
  } closer{ix};
  DeviceGuard g(device);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  const int dpad = ix->dpad;
  Scratch s(ix, st);
  int32_t* lists;
  double* sums;
  unsigned long long* cnt;
  CK(s.alloc(&lists, (size_t)n));
  CK(s.alloc(&sums, (size_t)nlist * d));
  CK(s.alloc(&cnt, (size_t)nlist));
  const int64_t ldg = ((nlist + 127) / 128) * 4;
  const int64_t sub = std::min<int64_t>(n, std::max<int64_t>(4096, (int64_t(1) << 27) / ldg));
  float* qhl;
  int* lo_any;
  CK(s.alloc(&qhl, (size_t)2 * sub * dpad));
  CK(s.alloc(&lo_any, 1));
  for (int it = 0; it < niter; ++it) {
    CK(cudaStreamSynchronize(st));  // set_centroids works on the legacy stream
    v = mv_index_set_centroids(ix, centroids);
    if (v != MV_OK) return v;
    // assignment: the tensor-core coarse step with nprobe = 1 (as mv_index_add)
    for (int64_t r0 = 0; r0 < n; r0 += sub) {
      const int64_t m = std::min(sub, n - r0);
      Scratch sb(ix, st);
      CK(cudaMemsetAsync(lo_any, 0, sizeof(int), st));
      CK(launch_hilo(x + r0 * d, m, d, dpad, qhl, lo_any, st));
      CK(run_coarse(ix, qhl, lo_any, m, 1, lists + r0, sb, st));
    }
    CK(cudaMemsetAsync(sums, 0, sizeof(double) * (size_t)nlist * d, st));
    CK(cudaMemsetAsync(cnt, 0, sizeof(unsigned long long) * nlist, st));
    CK(launch_kmeans_accum(x, n, d, lists, sums, cnt, st));
    CK(launch_kmeans_update(sums, cnt, nlist, d, spherical, centroids, st));
  }
  CK(cudaStreamSynchronize(st));
  return MV_OK;
}

mv_status mv_attr_bitset(const int64_t* ids, const int64_t* attr, int64_t n, int64_t lo, int64_t hi,
                         uint8_t* bitset, int64_t nbits, void* stream) {
  if (n < 0 || nbits < 0) return fail(MV_EINVAL, "n and nbits must be >= 0");
  if ((n > 0 && (!ids || !attr)) || (nbits > 0 && !bitset)) return fail(MV_EINVAL, "null argument");
  if (nbits == 0) return MV_OK;
  if (reinterpret_cast<uintptr_t>(bitset) % 4) return fail(MV_EINVAL, "bitset must be 4-byte aligned");
  if (is_host_ptr(ids) || is_host_ptr(attr) || is_host_ptr(bitset)) return fail(MV_EINVAL, "device pointers only");
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, bitset) != cudaSuccess) return from_cuda(cudaGetLastError(), "bitset");
  DeviceGuard g(at.device);
  CK(launch_attr_bitset(ids, attr, n, lo, hi, bitset, nbits, reinterpret_cast<cudaStream_t>(stream)));
  return MV_OK;
}

mv_status mv_fuse_rows(const float* const* parts, const int32_t* dims, const float* weights, int32_t m, int64_t n,
                       float* out, void* stream) {
  if (m < 1 || m > kMaxFuse) return fail(MV_EINVAL, "m must be in [1, %d]", kMaxFuse);
  if (n < 0) return fail(MV_EINVAL, "n must be >= 0");
  if (!parts || !dims || (n > 0 && !out)) return fail(MV_EINVAL, "null argument");
  FuseArgs a{};
  a.m = m;
  int64_t tot = 0;
  for (int i = 0; i < m; ++i) {
    if (dims[i] < 1 || (n > 0 && !parts[i])) return fail(MV_EINVAL, "part %d: bad dims or null pointer", i);
    a.part[i] = parts[i];
    a.dim[i] = dims[i];
    a.off[i] = (int)tot;
    a.w[i] = weights ? weights[i] : 1.0f;
    tot += dims[i];
  }
  if (tot > (1 << 20)) return fail(MV_EINVAL, "fused dimension too large");
  a.dtot = (int)tot;
  if (n == 0) return MV_OK;
  if (is_host_ptr(out)) return fail(MV_EINVAL, "device pointers only");
  for (int i = 0; i < m; ++i)
    if (is_host_ptr(parts[i])) return fail(MV_EINVAL, "device pointers only");
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, out) != cudaSuccess) return from_cuda(cudaGetLastError(), "out");
  DeviceGuard g(at.device);
  CK(launch_fuse_rows(a, n, out, reinterpret_cast<cudaStream_t>(stream)));
  return MV_OK;
}

mv_status mv_merge_topk(mv_metric metric, const float* dists, const int64_t* ids, int32_t nsrc, int64_t nq, int32_t k,
                        float* out_d, int64_t* out_i, void* stream) {
  if (metric != MV_L2 && metric != MV_IP) return fail(MV_EINVAL, "unknown metric");
  if (nsrc < 1 || k < 1 || k > kMaxK || nq < 0) return fail(MV_EINVAL, "bad nsrc/k/nq");
  if (nq == 0) return MV_OK;
  if (!dists || !ids || !out_d || !out_i) return fail(MV_EINVAL, "null argument");
  // the device of the (first) device buffer, else the current one: scratch goes there
  int dev = -1;
  for (const void* p : {(const void*)out_d, (const void*)dists}) {
    cudaPointerAttributes at;
    if (dev < 0 && cudaPointerGetAttributes(&at, p) == cudaSuccess && at.type == cudaMemoryTypeDevice) dev = at.device;
    cudaGetLastError();
  }
  DeviceGuard g(dev);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  Scratch s(nullptr, st);
  const size_t per = (size_t)nq * k;
  bool sd, si;
  const float* D;
  const int64_t* I;
  CK(stage_in(s, dists, per * nsrc, &D, &sd));
  CK(stage_in(s, ids, per * nsrc, &I, &si));
  const bool host_out = is_host_ptr(out_d) || is_host_ptr(out_i);
  std::vector<const float*> cd;
  std::vector<const int64_t*> ci;
  for (int i = 0; i < nsrc; ++i) {
    cd.push_back(D + per * i);
    ci.push_back(I + per * i);
  }
  while (cd.size() > 1) {
    std::vector<const float*> nd;
    std::vector<const int64_t*> ni;
    for (size_t i = 0; i + 1 < cd.size(); i += 2) {
      float* od;
      int64_t* oi;
      CK(s.alloc(&od, per));
      CK(s.alloc(&oi, per));
      CK(launch_merge2(metric, cd[i], ci[i], cd[i + 1], ci[i + 1], nq, k, od, oi, st));
      nd.push_back(od);
      ni.push_back(oi);
    }
    if (cd.size() & 1) {
      nd.push_back(cd.back());
      ni.push_back(ci.back());
    }
    cd.swap(nd);
    ci.swap(ni);
  }
  CK(cudaMemcpyAsync(out_d, cd[0], per * sizeof(float), cudaMemcpyDefault, st));
  CK(cudaMemcpyAsync(out_i, ci[0], per * sizeof(int64_t), cudaMemcpyDefault, st));
  if (host_out || sd || si) CK(cudaStreamSynchronize(st));
  return MV_OK;
}

mv_status mv_index_describe(const mv_index* ix, char* buf, size_t len) {
  if (!ix || !buf || len == 0) return fail(MV_EINVAL, "null argument");
  const char* refine = ix->type != MV_IVF_FLAT ? "always (SQ8 digit-plane filter)"
                       : ix->tf32_exact        ? "when a query is not tf32-exact"
                                               : "always (stored values not tf32-exact)";
  snprintf(buf, len,
           "{\"d\": %d, \"dpad\": %d, \"nlist\": %d, \"ntotal\": %lld, \"maxlen\": %lld, \"type\": \"%s\", "
           "\"metric\": \"%s\", \"tf32_exact\": %s, \"flat_refine\": \"%s\", \"xmax2\": %.17g, "
           "\"allocator\": \"%s\", \"last_scan\": \"%s\", \"last_coarse\": \"%s\", \"last_chunks\": %lld}",
           ix->d, ix->dpad, ix->nlist, (long long)ix->ntotal, (long long)ix->maxlen,
           ix->type == MV_IVF_FLAT ? "IVF_FLAT" : (ix->type == MV_IVF_SQ8 ? "IVF_SQ8" : "IVF_PQ"),
           ix->metric == MV_L2 ? "L2" : "IP",
           ix->tf32_exact ? "true" : "false", refine, ix->xmax2, ix->alloc.alloc ? "caller" : "cuda-pool",
           ix->last_scan, ix->last_coarse, (long long)ix->last_chunks);
  return MV_OK;
}

mv_status mv_profile_enable(mv_index* ix, int on) {
  if (!ix) return fail(MV_EINVAL, "null index");
  ix->prof = on != 0;
  return MV_OK;
}

mv_status mv_profile_read(mv_index* ix, double* ms, int64_t* searches, int64_t* launches, int reset) {
  if (!ix) return fail(MV_EINVAL, "null index");
  DeviceGuard g(ix->device);
  constexpr int NS = kProfStages;
  double acc[NS] = {0};
  for (size_t i = 0; i + NS + 1 <= ix->ev.size(); i += NS + 1) {
    CK(cudaEventSynchronize(ix->ev[i + NS]));
    for (int s = 0; s < NS; ++s) {
      float t = 0.f;
      CK(cudaEventElapsedTime(&t, ix->ev[i + s], ix->ev[i + s + 1]));
      acc[s] += t;
    }
  }
  if (ms)
    for (int s = 0; s < NS; ++s) ms[s] = acc[s];
  if (searches) *searches = ix->prof_searches;
  if (launches) *launches = ix->launches;
  if (reset) {
    for (cudaEvent_t e : ix->ev) cudaEventDestroy(e);
    ix->ev.clear();
    ix->prof_searches = 0;
    ix->launches = 0;
  }
  return MV_OK;
}

mv_status mv_profile_counters(mv_index* ix, int64_t* out, int reset) {
  if (!ix || !out) return fail(MV_EINVAL, "null argument");
  DeviceGuard g(ix->device);
  unsigned long long h[4] = {0, 0, 0, 0};
  if (ix->d_count) {
    CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(h, ix->d_count, sizeof h, cudaMemcpyDeviceToHost));
    if (reset) CK(cudaMemset(ix->d_count, 0, sizeof h));
  }
  for (int i = 0; i < 3; ++i) out[i] = (int64_t)h[i];
  return MV_OK;
}

mv_status mv_index_storage(const mv_index* ix, int64_t* list_off, int64_t* ids, uint8_t* codes) {
  if (!ix) return fail(MV_EINVAL, "null index");
  DeviceGuard g(ix->device);
  if (list_off) CK(cudaMemcpy(list_off, ix->list_off, sizeof(int64_t) * (ix->nlist + 1), cudaMemcpyDefault));
  if (ids && ix->ntotal) CK(cudaMemcpy(ids, ix->ids, sizeof(int64_t) * ix->ntotal, cudaMemcpyDefault));
  if (codes && ix->ntotal) {
    if (ix->type == MV_IVF_PQ) {
      CK(cudaMemcpy(codes, ix->payload, (size_t)ix->ntotal * ix->pq_m, cudaMemcpyDefault));
      return MV_OK;
    }
    if (ix->type != MV_IVF_SQ8) return fail(MV_ESTATE, "codes requested from a FLAT index");
    CK(cudaMemcpy2D(codes, ix->d, ix->payload, ix->dpad, ix->d, ix->ntotal, cudaMemcpyDefault));
  }
  return MV_OK;
}

}  // extern "C"
