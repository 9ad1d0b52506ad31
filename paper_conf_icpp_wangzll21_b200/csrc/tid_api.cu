// tid_api.cu — C-ABI implementation (include/tid.h): index lifecycle, reference arena
// (HBM level-1 + pinned-host level-2, §6.1), host-tier streaming with a
// double-buffered copy stream (§6.2), query batching, shard merge over NCCL.
#include <cuda.h>
#include <cuda_runtime.h>
#include <nccl.h>

#include <dlfcn.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/tid.h"
#include "tid_kernels.cuh"

using namespace tid;

namespace {

thread_local std::string g_err;

tid_status fail(tid_status st, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return st;
}

#define CU(call)                                                                                  \
  do {                                                                                            \
    cudaError_t e__ = (call);                                                                     \
    if (e__ != cudaSuccess)                                                                       \
      return fail(TID_ECUDA, "%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(e__)); \
  } while (0)

// NCCL is resolved at run time (dlopen) so that the library never forces its own NCCL
// build into a process that already loaded another one (e.g. PyTorch's): an already
// loaded libnccl.so.2 is preferred, then $TID_NCCL_LIBRARY, then the system library.
struct NcclApi {
  bool ok = false;
  std::string err;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  ncclResult_t (*CommCount)(const ncclComm_t, int*) = nullptr;
};

const NcclApi& nccl() {
  static NcclApi api;
  static bool tried = false;
  if (tried) return api;
  tried = true;
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
  if (!h) {
    const char* env = getenv("TID_NCCL_LIBRARY");
    if (env && *env) h = dlopen(env, RTLD_NOW | RTLD_LOCAL);
  }
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_LOCAL);
  if (!h) {
    api.err = std::string("cannot load libnccl.so.2: ") + dlerror();
    return api;
  }
  api.GetUniqueId = reinterpret_cast<decltype(api.GetUniqueId)>(dlsym(h, "ncclGetUniqueId"));
  api.CommInitRank = reinterpret_cast<decltype(api.CommInitRank)>(dlsym(h, "ncclCommInitRank"));
  api.CommDestroy = reinterpret_cast<decltype(api.CommDestroy)>(dlsym(h, "ncclCommDestroy"));
  api.AllGather = reinterpret_cast<decltype(api.AllGather)>(dlsym(h, "ncclAllGather"));
  api.GetErrorString = reinterpret_cast<decltype(api.GetErrorString)>(dlsym(h, "ncclGetErrorString"));
  api.AllReduce = reinterpret_cast<decltype(api.AllReduce)>(dlsym(h, "ncclAllReduce"));
  api.CommCount = reinterpret_cast<decltype(api.CommCount)>(dlsym(h, "ncclCommCount"));
  api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.AllGather && api.AllReduce &&
           api.GetErrorString;
  if (!api.ok) api.err = "libnccl.so.2 lacks a required symbol";
  return api;
}

#define NC(call)                                                                                          \
  do {                                                                                                    \
    if (!nccl().ok) return fail(TID_ENCCL, "%s", nccl().err.c_str());                                    \
    ncclResult_t r__ = (call);                                                                            \
    if (r__ != ncclSuccess)                                                                               \
      return fail(TID_ENCCL, "%s:%d %s: %s", __FILE__, __LINE__, #call, nccl().GetErrorString(r__));     \
  } while (0)

#define TRY(x)                    \
  do {                            \
    tid_status s__ = (x);         \
    if (s__ != TID_OK) return s__; \
  } while (0)

// ---------------------------------------------------------------- growable device buffer
struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
  tid_status ensure(size_t need, const char* what) {
    if (need <= bytes) return TID_OK;
    if (p) cudaFree(p);
    p = nullptr;
    bytes = 0;
    size_t want = std::max(need, static_cast<size_t>(1) << 20);
    cudaError_t e = cudaMalloc(&p, want);
    if (e != cudaSuccess) {
      cudaGetLastError();
      p = nullptr;
      return fail(TID_ENOMEM, "cudaMalloc(%zu) for %s: %s", want, what, cudaGetErrorString(e));
    }
    bytes = want;
    return TID_OK;
  }
  void release() {
    if (p) cudaFree(p);
    p = nullptr;
    bytes = 0;
  }
  template <class T> T* as() const { return static_cast<T*>(p); }
};

// ---------------------------------------------------------------- tensor maps (driver entry point)
typedef CUresult (*PFN_encodeTiled_t)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                      const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                      CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

PFN_encodeTiled_t encode_fn() {
  static PFN_encodeTiled_t fn = nullptr;
  if (!fn) {
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_encodeTiled_t>(ptr);
  }
  return fn;
}

// Encoded maps depend only on (address, geometry), so repeated searches reuse them: a small
// per-thread cache (encoding costs host microseconds, which bound small-search latency).
struct MapKey {
  int kind;
  const void* base;
  int64_t count, rows;
  int box;
  bool operator==(const MapKey& o) const {
    return kind == o.kind && base == o.base && count == o.count && rows == o.rows && box == o.box;
  }
};
bool map_cache_get(const MapKey& k, CUtensorMap* map);
void map_cache_put(const MapKey& k, const CUtensorMap& map);
struct MapCache {
  static constexpr int kN = 16;
  MapKey key[kN];
  CUtensorMap map[kN];
  int used = 0, next = 0;
};
thread_local MapCache g_maps;
bool map_cache_get(const MapKey& k, CUtensorMap* map) {
  for (int i = 0; i < g_maps.used; ++i)
    if (g_maps.key[i] == k) {
      *map = g_maps.map[i];
      return true;
    }
  return false;
}
void map_cache_put(const MapKey& k, const CUtensorMap& map) {
  const int i = g_maps.next;
  g_maps.key[i] = k;
  g_maps.map[i] = map;
  g_maps.next = (i + 1) % MapCache::kN;
  g_maps.used = std::min(g_maps.used + 1, MapCache::kN);
}

// u8 tensor [count][rows][128] -> 3-D map with box {128 B, box_rows, 1}, SWIZZLE_128B,
// out-of-bounds rows zero-filled (this is how ragged n / m are padded to the tile).
tid_status make_map(CUtensorMap* map, const void* base, int64_t count, int64_t rows, int box_rows) {
  const MapKey key{0, base, count, rows, box_rows};
  if (map_cache_get(key, map)) return TID_OK;
  PFN_encodeTiled_t fn = encode_fn();
  if (!fn) return fail(TID_ECUDA, "cuTensorMapEncodeTiled entry point unavailable");
  if (reinterpret_cast<uintptr_t>(base) % 16) return fail(TID_EINVAL, "descriptor buffer must be 16-byte aligned");
  cuuint64_t dims[3] = {static_cast<cuuint64_t>(kDim), static_cast<cuuint64_t>(rows),
                        static_cast<cuuint64_t>(std::max<int64_t>(count, 1))};
  cuuint64_t strides[2] = {static_cast<cuuint64_t>(kDim), static_cast<cuuint64_t>(rows * kDim)};
  cuuint32_t box[3] = {static_cast<cuuint32_t>(kDim), static_cast<cuuint32_t>(box_rows), 1};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, const_cast<void*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(TID_ECUDA, "cuTensorMapEncodeTiled failed (%d)", static_cast<int>(r));
  map_cache_put(key, *map);
  return TID_OK;
}

// u8 norm-term digits [count][rows][32] -> 3-D map with box {32 B, 256, 1}, SWIZZLE_32B.
tid_status make_xmap(CUtensorMap* map, const void* base, int64_t count, int64_t rows) {
  const MapKey key{1, base, count, rows, kBN};
  if (map_cache_get(key, map)) return TID_OK;
  PFN_encodeTiled_t fn = encode_fn();
  if (!fn) return fail(TID_ECUDA, "cuTensorMapEncodeTiled entry point unavailable");
  cuuint64_t dims[3] = {static_cast<cuuint64_t>(kXDim), static_cast<cuuint64_t>(rows),
                        static_cast<cuuint64_t>(std::max<int64_t>(count, 1))};
  cuuint64_t strides[2] = {static_cast<cuuint64_t>(kXDim), static_cast<cuuint64_t>(rows * kXDim)};
  cuuint32_t box[3] = {static_cast<cuuint32_t>(kXDim), static_cast<cuuint32_t>(kBN), 1};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, const_cast<void*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(TID_ECUDA, "cuTensorMapEncodeTiled (norm digits) failed (%d)", static_cast<int>(r));
  map_cache_put(key, *map);
  return TID_OK;
}

// fp16 tensor [count][rows][128] -> 3-D map with box {64 elements = 128 B, box_rows, 1}, SWIZZLE_128B
// (a row's two K-halves are loaded as two tiles).
tid_status make_map_f16(CUtensorMap* map, const void* base, int64_t count, int64_t rows, int box_rows) {
  PFN_encodeTiled_t fn = encode_fn();
  if (!fn) return fail(TID_ECUDA, "cuTensorMapEncodeTiled entry point unavailable");
  if (reinterpret_cast<uintptr_t>(base) % 16) return fail(TID_EINVAL, "fp16 buffer must be 16-byte aligned");
  cuuint64_t dims[3] = {static_cast<cuuint64_t>(kDim), static_cast<cuuint64_t>(rows),
                        static_cast<cuuint64_t>(std::max<int64_t>(count, 1))};
  cuuint64_t strides[2] = {static_cast<cuuint64_t>(kDim * 2), static_cast<cuuint64_t>(rows * kDim * 2)};
  cuuint32_t box[3] = {64, static_cast<cuuint32_t>(box_rows), 1};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_UINT16, 3, const_cast<void*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(TID_ECUDA, "cuTensorMapEncodeTiled (fp16) failed (%d)", static_cast<int>(r));
  return TID_OK;
}

bool is_device_ptr(const void* p) {
  if (!p) return false;
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// A contiguous range of local ids [first, first + count) stored together, either in the HBM
// arena (level-1 cache: descriptors + precomputed column keys) or in the pinned host tier
// (level 2: raw descriptors, streamed and keyed on the GPU per search).  §6.1 P:784-795.
struct Segment {
  bool on_host = false;
  uint8_t* desc = nullptr;    // [cap][m][128]: device (HBM) or pinned host
  int32_t* colkey = nullptr;  // device, HBM segments only: [cap][cpr][256] column terms W (search)
  uint16_t* xop = nullptr;    // device, HBM segments of a float (f1) index: [cap][256][16] fp16 norm terms
  int64_t cap = 0, count = 0, first = 0;
  std::vector<int32_t> kp;    // keypoint count per reference (0 = deleted / empty)
};

}  // namespace

struct tid_index {
  tid_config cfg{};
  int device = 0;
  int num_sms = 148;
  int cpr = 1;                    // chunks per reference = ceil(ref_kp / 256)
  bool f16 = false;               // descriptor 1: the float path (RootSIFT / scaled SIFT in fp16, row f1)
  float f16_c = 0.0f, f16_scale = 1.0f;  // the index's norm-term constant C and the fp16 scale factor
  int32_t f16_rootsift = 1;
  int64_t ref_bytes = 0;          // bytes per stored reference (u8, or fp16 for a float index)
  int64_t in_bytes = 0;           // bytes per reference of the caller's u8 input (ref_kp * 128)
  int64_t hbm_ref_bytes = 0;      // HBM bytes per resident reference (descriptors + norm digits + column terms)
  uint64_t hbm_budget = 0, host_budget = 0;
  std::vector<Segment> segs;      // id order; HBM and host segments may interleave (FIFO policy)
  int64_t n_hbm = 0, n_host = 0;  // references held in each tier
  std::vector<uint8_t> dead;      // per local id: deleted (excluded from ranking)
  DevBuf dead_dev;                // device copy of `dead` (valid when any_dead)
  bool any_dead = false, dead_dirty = false;
  int64_t hbm_alloc = 0, host_alloc = 0;
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t ev_h2d[2] = {nullptr, nullptr}, ev_free[2] = {nullptr, nullptr};
  // every call that touches the workspaces waits for the previous call's work (whatever stream it
  // ran on) and records this event at its end: one index may be driven from several streams
  cudaEvent_t ev_last = nullptr;
  // CUDA-graph replay of repeated searches (device buffers, HBM-resident references): the
  // launch-bound small-batch path (C1) costs one graph launch instead of ~5 submissions
  uint64_t gen = 0;               // bumped by every change of the references / dead flags / tuning
  cudaStream_t graph_stream = nullptr;
  cudaEvent_t ev_gin = nullptr, ev_gout = nullptr;
  struct GraphEntry {
    const void* q; const void* nq; const void* ids; const void* cnts;
    int32_t n, k;
    int64_t B;
    uint64_t gen;
    std::vector<void*> ws;        // workspace pointers baked into the graph
    cudaGraphExec_t exec = nullptr;
    int uses = 0;
  };
  std::vector<GraphEntry> graphs;
  // workspaces
  DevBuf ws_q, ws_nq, ws_nvalid, ws_counts, ws_cand, ws_keys, ws_gather, ws_ids, ws_cnts, ws_r, ws_colkey, ws_nn,
      ws_kp, ws_mr;
  DevBuf stage_desc[2], stage_colkey[2], stage_kp[2];
  DevBuf ws_qs;                   // shifted queries q' = q ^ 0x80 (search)
  DevBuf ws_rtot;                 // collective reference count (all-reduce)
  DevBuf ws_geo_nn, ws_geo_cnt, ws_geo_xy, ws_geo_out;  // f4 post-match verification
  DevBuf ws_u8, ws_f16c, ws_f16kp, ws_f16rows, stage_xop[2];  // f1 index: conversion staging, C, xop inputs
  int64_t* h_rtot = nullptr;      // pinned host copy of it
  DevBuf ws_f16q, ws_f16r, ws_f16nq, ws_f16nr, ws_f16in;  // f1 float path
  int64_t host_chunk = 0;
  tid_tuning tune{};
  ncclComm_t comm = nullptr;
  // profiling
  bool prof = false;
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> prof_ev;
  size_t prof_used = 0;
  tid_stats stats{};
};

namespace {

tid_status set_device(tid_index* idx) {
  CU(cudaSetDevice(idx->device));
  return TID_OK;
}

void count_kernel(tid_index* idx, int n = 1) {
  if (idx->prof) idx->stats.kernel_launches += n;
}

// Cross-call ordering of the per-index workspaces (see tid_index::ev_last): the constructor makes
// `s` wait for everything the previous call enqueued; the destructor records the end of this call
// (also on early error returns, so partially enqueued work is still ordered before the next call).
struct CallGuard {
  tid_index* idx;
  cudaStream_t s;
  CallGuard(tid_index* i, cudaStream_t st) : idx(i), s(st) { cudaStreamWaitEvent(s, idx->ev_last, 0); }
  ~CallGuard() { cudaEventRecord(idx->ev_last, s); }
};

tid_status copy_in(tid_index* idx, void* dst, const void* src, size_t bytes, cudaStream_t s) {
  if (bytes == 0) return TID_OK;
  const bool dev = is_device_ptr(src);
  CU(cudaMemcpyAsync(dst, src, bytes, dev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, s));
  if (!dev && idx->prof) idx->stats.h2d_bytes += static_cast<int64_t>(bytes);
  return TID_OK;
}

tid_status copy_out(tid_index* idx, void* dst, const void* src, size_t bytes, cudaStream_t s, bool* host_out) {
  if (bytes == 0) return TID_OK;
  const bool dev = is_device_ptr(dst);
  CU(cudaMemcpyAsync(dst, src, bytes, dev ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, s));
  if (!dev) {
    *host_out = true;
    if (idx->prof) idx->stats.d2h_bytes += static_cast<int64_t>(bytes);
  }
  return TID_OK;
}

// Choose job decomposition of a search launch: refs per job G, queries per job, slot banks.
// Small batches (one chunk per reference, B * T <= 16 query tiles per job) use two banks of 2 slots:
// a job is short there, and the next job's references then load while this one runs.
void plan_search(const tid_index* idx, int64_t n_refs, int64_t B, int T, int* G_out, int* qpj_out, int* banks_out) {
  const int banks = (idx->cpr == 1 && B * T <= 16 && idx->tune.refs_per_job == 0) ? 2 : 1;
  // refs per job: one per epilogue group (group g <-> resident reference g), fewer for m > 256
  const int max_g = std::min(kMaxSlots / banks / idx->cpr, kNG);
  int G = idx->tune.refs_per_job > 0 ? std::min(idx->tune.refs_per_job, max_g) : max_g;
  const int64_t target_jobs = 2LL * idx->num_sms;
  // spread small reference sets over more CTAs (fewer resident refs per job)
  while (G > 1 && ceil_div(n_refs, G) < target_jobs) --G;
  int64_t groups = ceil_div(n_refs, G);
  int qpj = static_cast<int>(B);
  // still too few jobs: split the query batch too (each job then re-reads its refs)
  while (groups * ceil_div(B, qpj) < target_jobs && qpj > 1) qpj = (qpj + 1) / 2;
  *G_out = G;
  *qpj_out = qpj;
  *banks_out = banks;
}

tid_status launch_search_range(tid_index* idx, const CUtensorMap& qmap, const uint8_t* rbase, int64_t map_count, int64_t ref_map_base, const int32_t* colkey, int64_t n_refs, int64_t B,
                               int32_t n,
                               int T, const int32_t* nvalid, uint32_t* counts, int64_t ldc, int64_t col0,
                               cudaStream_t s) {
  if (n_refs <= 0) return TID_OK;
  CUtensorMap rmap;
  TRY(make_map(&rmap, rbase, map_count, idx->cfg.ref_kp, kBN));
  MatchParams p{};
  p.mode = kModeSearch;
  p.qs = idx->ws_qs.as<uint8_t>();
  p.rdesc = rbase;
  p.m = idx->cfg.ref_kp;
  int G, qpj, banks;
  plan_search(idx, n_refs, B, T, &G, &qpj, &banks);
  p.refs_per_job = G;
  p.slot_banks = banks;
  p.cpr = idx->cpr;
  p.tiles_per_q = T;
  p.num_q = static_cast<int32_t>(B);
  p.q_per_job = qpj;
  p.n_qchunks = static_cast<int32_t>(ceil_div(B, qpj));
  p.n_jobs = static_cast<int32_t>(ceil_div(n_refs, G) * p.n_qchunks);
  p.n_refs = n_refs;
  p.ref_map_base = ref_map_base;
  p.colkey = colkey;
  p.nq = idx->ws_nq.as<int32_t>();
  p.n_valid = nvalid;
  p.n_rows = n;
  p.counts = counts;
  p.ldc = ldc;
  p.col0 = col0;
  p.nn_out = nullptr;
  p.num2 = idx->cfg.ratio_num * idx->cfg.ratio_num;
  p.den2 = idx->cfg.ratio_den * idx->cfg.ratio_den;
  int grid = idx->tune.grid > 0 ? idx->tune.grid : idx->num_sms;
  grid = static_cast<int>(std::min<int64_t>(grid, p.n_jobs));
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  if (idx->prof) {
    if (idx->prof_used == idx->prof_ev.size()) {
      cudaEvent_t a, b;
      CU(cudaEventCreate(&a));
      CU(cudaEventCreate(&b));
      idx->prof_ev.push_back({a, b});
    }
    e0 = idx->prof_ev[idx->prof_used].first;
    e1 = idx->prof_ev[idx->prof_used].second;
    ++idx->prof_used;
    CU(cudaEventRecord(e0, s));
  }
  cudaError_t e = launch_match(p, qmap, rmap, true, grid, s);
  if (e != cudaSuccess) return fail(TID_ECUDA, "match kernel launch: %s", cudaGetErrorString(e));
  if (idx->prof) {
    CU(cudaEventRecord(e1, s));
    idx->stats.match_launches++;
    count_kernel(idx);
  }
  return TID_OK;
}

tid_status f16_norm_terms(tid_index* idx, const void* refs16, int64_t count, const int32_t* kp_dev, uint16_t* xop,
                          cudaStream_t s);

// A run of consecutive local ids [first, first + cnt) inside one segment (offset `off`), inside one
// count window.  Host-tier pieces are at most host_chunk references (one staging buffer).
struct Piece {
  const Segment* sg;
  int64_t off, cnt, first;
  int64_t win;  // window index
};

// The work list of one search pass: local ids [0, R) in id order, cut at window boundaries
// (windows of W ids) and, in the host tier, into staging chunks.
std::vector<Piece> plan_pieces(const tid_index* idx, int64_t W) {
  std::vector<Piece> out;
  const int64_t R = idx->n_hbm + idx->n_host;
  for (int64_t w0 = 0, wi = 0; w0 < R; w0 += W, ++wi) {
    const int64_t w1 = std::min(R, w0 + W);
    for (const Segment& sg : idx->segs) {
      const int64_t a = std::max(w0, sg.first), b = std::min(w1, sg.first + sg.count);
      if (a >= b) continue;
      const int64_t step = sg.on_host ? idx->host_chunk : (b - a);
      for (int64_t x = a; x < b; x += step) out.push_back({&sg, x - sg.first, std::min(step, b - x), x, wi});
    }
  }
  return out;
}

// One pass over every local reference for the B queries already on the device (dq): query prep
// (a2), then per window of W reference ids the fused match kernel into counts[B][W] (ldc = W,
// column = local id - window start), HBM segments in place (level 1) and host-tier chunks
// streamed through two staging buffers on the copy stream (level 2, double buffered: chunk i+1
// is copied while chunk i computes, across window boundaries too).  After each window's last
// piece `on_window(w0, wlen)` runs on stream s (top-k of the window); the next window's
// kernels are ordered after it on the same stream, so one counts buffer serves every window.
template <class OnWindow>
tid_status run_pass(tid_index* idx, const uint8_t* dq, const int32_t* nvalid, int32_t n, int64_t B, int64_t W,
                    uint32_t* counts, cudaStream_t s, OnWindow on_window) {
  const int T = static_cast<int>(ceil_div(n, kBM));
  const int64_t R = idx->n_hbm + idx->n_host;
  CUtensorMap qmap;
  if (idx->f16) {  // row f1: queries -> [RootSIFT] x scale -> fp16, fp32 squared norms N_Q
    TRY(idx->ws_f16q.ensure(static_cast<size_t>(B) * n * kDim * 2, "f16 queries"));
    TRY(idx->ws_f16nq.ensure(static_cast<size_t>(B) * T * kBM * 4, "f16 query norms"));
    CU(launch_f16_prepare(dq, B * n, idx->f16_rootsift, idx->f16_scale, idx->ws_f16q.p, s));
    CU(launch_f16_norms(idx->ws_f16q.p, B, n, T * kBM, 0.0f, idx->ws_f16nq.as<float>(), s));
    count_kernel(idx, 2);
    TRY(make_map_f16(&qmap, idx->ws_f16q.p, B, n, kBM));
  } else {
    TRY(idx->ws_nq.ensure(static_cast<size_t>(B) * T * kBM * 4, "query norms"));
    TRY(idx->ws_qs.ensure(static_cast<size_t>(B) * n * kDim, "shifted queries"));
    launch_query_prep(dq, B, n, T, idx->ws_nq.as<int32_t>(), idx->ws_qs.as<uint8_t>(), s);
    count_kernel(idx);
    TRY(make_map(&qmap, idx->ws_qs.p, B, n, kBM));
  }
  // row f1: one kind::f16 match launch over `cnt` references starting at map index `base`
  auto launch_f16 = [&](const void* rbase, const void* xbase, int64_t map_count, int64_t base, int64_t cnt,
                        int64_t col0) -> tid_status {
    CUtensorMap rmap, xmap;
    TRY(make_map_f16(&rmap, rbase, map_count, idx->cfg.ref_kp, kBN));
    TRY(make_xmap(&xmap, xbase, map_count, static_cast<int64_t>(kBN) * idx->cpr));
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    if (idx->prof) {
      if (idx->prof_used == idx->prof_ev.size()) {
        cudaEvent_t a, b;
        CU(cudaEventCreate(&a));
        CU(cudaEventCreate(&b));
        idx->prof_ev.push_back({a, b});
      }
      e0 = idx->prof_ev[idx->prof_used].first;
      e1 = idx->prof_ev[idx->prof_used].second;
      ++idx->prof_used;
      CU(cudaEventRecord(e0, s));
    }
    CU(launch_f16_match(qmap, rmap, xmap, idx->ws_f16c.as<float>(), idx->ws_f16nq.as<float>(), static_cast<int32_t>(B),
                        n, T, cnt, idx->cfg.ratio_num * idx->cfg.ratio_num, idx->cfg.ratio_den * idx->cfg.ratio_den,
                        counts, idx->num_sms, s, W, col0, base, nvalid, idx->cpr, idx->cfg.ref_kp));
    if (idx->prof) {
      CU(cudaEventRecord(e1, s));
      idx->stats.match_launches++;
      count_kernel(idx);
    }
    return TID_OK;
  };
  const std::vector<Piece> pieces = plan_pieces(idx, W);
  std::vector<int64_t> next_host(pieces.size() + 1, -1);  // index of the next host piece after i
  for (int64_t i = static_cast<int64_t>(pieces.size()) - 1, nh = -1; i >= 0; --i) {
    next_host[i] = nh;
    if (pieces[i].sg->on_host) nh = i;
  }
  int64_t first_host = -1;
  for (size_t i = 0; i < pieces.size() && first_host < 0; ++i)
    if (pieces[i].sg->on_host) first_host = static_cast<int64_t>(i);
  const int64_t chunk = idx->host_chunk, rb = idx->ref_bytes;
  std::vector<int> host_buf(pieces.size(), 0);
  if (first_host >= 0) {
    for (int b = 0; b < 2; ++b) {
      TRY(idx->stage_desc[b].ensure(static_cast<size_t>(chunk * rb), "host-tier staging"));
      if (idx->f16)
        TRY(idx->stage_xop[b].ensure(static_cast<size_t>(chunk) * kBN * idx->cpr * 16 * 2, "staging norm terms"));
      else
        TRY(idx->stage_colkey[b].ensure(static_cast<size_t>(chunk) * idx->cpr * kColBytes, "staging keys"));
      TRY(idx->stage_kp[b].ensure(static_cast<size_t>(chunk) * 4, "staging kp"));
    }
    // the copy stream must not overwrite staging buffers still read by a previous call
    CU(cudaEventRecord(idx->ev_free[0], s));
    CU(cudaEventRecord(idx->ev_free[1], s));
    for (size_t i = 0, h = 0; i < pieces.size(); ++i)
      if (pieces[i].sg->on_host) host_buf[i] = static_cast<int>(h++ & 1);
  }
  auto issue_copy = [&](int64_t i) -> tid_status {
    const int b = host_buf[i];
    const Piece& pc = pieces[i];
    CU(cudaStreamWaitEvent(idx->copy_stream, idx->ev_free[b], 0));
    CU(cudaMemcpyAsync(idx->stage_desc[b].p, pc.sg->desc + pc.off * rb, static_cast<size_t>(pc.cnt * rb),
                       cudaMemcpyHostToDevice, idx->copy_stream));
    CU(cudaMemcpyAsync(idx->stage_kp[b].p, pc.sg->kp.data() + pc.off, static_cast<size_t>(pc.cnt) * 4,
                       cudaMemcpyHostToDevice, idx->copy_stream));
    CU(cudaEventRecord(idx->ev_h2d[b], idx->copy_stream));
    if (idx->prof) idx->stats.h2d_bytes += pc.cnt * rb + pc.cnt * 4;
    return TID_OK;
  };
  if (first_host >= 0) TRY(issue_copy(first_host));
  int64_t cur_win = -1;
  for (size_t i = 0; i < pieces.size(); ++i) {
    const Piece& pc = pieces[i];
    const int64_t w0 = pc.win * W;
    if (pc.win != cur_win) {  // first piece of a window: clear its counts (kernels accumulate)
      cur_win = pc.win;
      CU(cudaMemsetAsync(counts, 0, static_cast<size_t>(B) * W * 4, s));
    }
    if (pc.sg->on_host) {
      const int b = host_buf[i];
      if (next_host[i] >= 0) TRY(issue_copy(next_host[i]));  // prefetch the next chunk while this one computes
      CU(cudaStreamWaitEvent(s, idx->ev_h2d[b], 0));
      if (idx->f16) {
        TRY(f16_norm_terms(idx, idx->stage_desc[b].p, pc.cnt, idx->stage_kp[b].as<int32_t>(),
                           idx->stage_xop[b].as<uint16_t>(), s));
        count_kernel(idx, 2);
        TRY(launch_f16(idx->stage_desc[b].p, idx->stage_xop[b].p, chunk, 0, pc.cnt, pc.first - w0));
        CU(cudaEventRecord(idx->ev_free[b], s));
        if (i + 1 == pieces.size() || pieces[i + 1].win != pc.win) TRY(on_window(w0, std::min(W, R - w0)));
        continue;
      }
      RefPrepParams rp{};
      rp.desc = idx->stage_desc[b].as<uint8_t>();
      rp.src = nullptr;
      rp.kp = idx->stage_kp[b].as<int32_t>();
      rp.colkey = idx->stage_colkey[b].as<int32_t>();
      rp.search = 1;
      rp.count = pc.cnt;
      rp.m = idx->cfg.ref_kp;
      rp.cpr = idx->cpr;
      launch_ref_prep(rp, s);
      count_kernel(idx);
      TRY(launch_search_range(idx, qmap, idx->stage_desc[b].as<uint8_t>(), chunk, 0, rp.colkey, pc.cnt, B,
                              n, T, nvalid, counts, W, pc.first - w0, s));
      CU(cudaEventRecord(idx->ev_free[b], s));
    } else if (idx->f16) {
      TRY(launch_f16(pc.sg->desc, pc.sg->xop, pc.sg->cap, pc.off, pc.cnt, pc.first - w0));
    } else {
      TRY(launch_search_range(idx, qmap, pc.sg->desc, pc.sg->cap, pc.off,
                              pc.sg->colkey + pc.off * idx->cpr * kColInts, pc.cnt, B, n, T, nvalid, counts, W,
                              pc.first - w0, s));
    }
    if (i + 1 == pieces.size() || pieces[i + 1].win != pc.win) TRY(on_window(w0, std::min(W, R - w0)));
  }
  return TID_OK;
}

// References per count window of a search: the whole local set when its [B][R] u32 count matrix
// fits the window budget (512 MiB, or the tuning's window_refs), else windows of that size
// (workspace independent of R: a 10 M-reference host tier needs no 10 GB count matrix).
int64_t window_refs(const tid_index* idx, int64_t B, int64_t R) {
  int64_t W = idx->tune.window_refs > 0 ? idx->tune.window_refs
                                        : std::max<int64_t>(4096, (int64_t(512) << 20) / (4 * std::max<int64_t>(B, 1)));
  return std::max<int64_t>(1, std::min(W, R));
}

// Test hook: with TID_FAULT_ALLOC=N in the environment the N-th segment allocation from then on
// fails with TID_ENOMEM (checks that tid_add_references is all-or-nothing).  Unset: no effect.
bool injected_alloc_failure() {
  static thread_local std::string armed;
  static thread_local long left = 0;
  const char* v = getenv("TID_FAULT_ALLOC");
  if (!v || !*v) {
    armed.clear();
    return false;
  }
  if (armed != v) {
    armed = v;
    left = strtol(v, nullptr, 10);
  }
  return left > 0 && --left == 0;
}

// Allocate a segment of `cap` references in one tier (all-or-nothing).
tid_status alloc_segment(tid_index* idx, bool on_host, int64_t cap, Segment* out) {
  const int64_t rb = idx->ref_bytes;
  if (injected_alloc_failure()) return fail(TID_ENOMEM, "injected allocation failure (TID_FAULT_ALLOC)");
  Segment sg;
  sg.on_host = on_host;
  sg.cap = cap;
  if (on_host) {
    if (cudaHostAlloc(reinterpret_cast<void**>(&sg.desc), static_cast<size_t>(cap * rb), cudaHostAllocPortable) !=
        cudaSuccess) {
      cudaGetLastError();
      return fail(TID_ENOMEM, "pinned host tier allocation of %lld bytes failed", static_cast<long long>(cap * rb));
    }
    idx->host_alloc += cap * rb;
  } else {
    cudaError_t e1 = cudaMalloc(&sg.desc, static_cast<size_t>(cap * rb));
    cudaError_t e2 = e1 != cudaSuccess ? e1
                     : idx->f16 ? cudaMalloc(&sg.xop, static_cast<size_t>(cap) * kBN * idx->cpr * 16 * 2)
                                : cudaMalloc(&sg.colkey, static_cast<size_t>(cap) * idx->cpr * kColBytes);
    if (e1 != cudaSuccess || e2 != cudaSuccess) {
      cudaGetLastError();
      if (sg.desc) cudaFree(sg.desc);
      if (sg.colkey) cudaFree(sg.colkey);
      if (sg.xop) cudaFree(sg.xop);
      return fail(TID_ENOMEM, "HBM arena allocation of %lld references failed", static_cast<long long>(cap));
    }
    idx->hbm_alloc += cap * idx->hbm_ref_bytes;
  }
  *out = std::move(sg);
  return TID_OK;
}

void free_segment(tid_index* idx, Segment& sg) {
  if (sg.on_host) {
    if (sg.desc) cudaFreeHost(sg.desc);
    idx->host_alloc -= sg.cap * idx->ref_bytes;
  } else {
    if (sg.desc) cudaFree(sg.desc);
    if (sg.colkey) cudaFree(sg.colkey);
    if (sg.xop) cudaFree(sg.xop);
    idx->hbm_alloc -= sg.cap * idx->hbm_ref_bytes;
  }
  sg.desc = nullptr;
  sg.colkey = nullptr;
  sg.xop = nullptr;
}

// Ingest `take` references (host or device `src`, kp_host per reference) into HBM segment sg at
// position `pos`: copy, zero padding rows, N_R -> packed column keys (Alg. 1 step 1).
// Float index (descriptor 1): u8 SIFT rows (host or device) -> [RootSIFT] x scale -> fp16 at dst
// (device), on the legacy stream.  Unaligned or host input goes through the u8 staging buffer.
tid_status convert_f16(tid_index* idx, const uint8_t* src, bool src_dev, int64_t count, void* dst) {
  const size_t ib = static_cast<size_t>(count) * idx->in_bytes;
  const uint8_t* din = src;
  if (!src_dev || reinterpret_cast<uintptr_t>(src) % 16) {
    TRY(idx->ws_u8.ensure(ib, "u8 staging"));
    CU(cudaMemcpy(idx->ws_u8.p, src, ib, cudaMemcpyDefault));
    din = idx->ws_u8.as<uint8_t>();
  }
  CU(launch_f16_prepare(din, count * idx->cfg.ref_kp, idx->f16_rootsift, idx->f16_scale, dst, nullptr));
  return TID_OK;
}

// Float index: norm-term rows (fixed C, per-reference keypoint counts) of `count` stored fp16 references.
tid_status f16_norm_terms(tid_index* idx, const void* refs16, int64_t count, const int32_t* kp_dev, uint16_t* xop,
                          cudaStream_t s) {
  TRY(idx->ws_f16rows.ensure(static_cast<size_t>(count) * idx->cfg.ref_kp * 4, "f16 reference norms"));
  CU(launch_f16_xop_fixed(refs16, count, idx->cfg.ref_kp, kp_dev, idx->f16_c, idx->ws_f16rows.as<float>(), xop, s));
  return TID_OK;
}

tid_status ingest_hbm(tid_index* idx, Segment& sg, int64_t pos, const uint8_t* src, bool src_dev,
                      const int32_t* kp_host, int64_t take) {
  const int64_t rb = idx->ref_bytes;
  if (idx->f16) {  // row f1: convert on the GPU, then the norm terms with the index's constant C
    TRY(convert_f16(idx, src, src_dev, take, sg.desc + pos * rb));
    TRY(idx->ws_kp.ensure(static_cast<size_t>(take) * 4, "kp staging"));
    CU(cudaMemcpy(idx->ws_kp.p, kp_host, static_cast<size_t>(take) * 4, cudaMemcpyHostToDevice));
    TRY(f16_norm_terms(idx, sg.desc + pos * rb, take, idx->ws_kp.as<int32_t>(),
                       sg.xop + static_cast<size_t>(pos) * kBN * idx->cpr * 16, nullptr));
    CU(cudaStreamSynchronize(nullptr));
    return TID_OK;
  }
  uint8_t* dst = sg.desc + pos * rb;
  RefPrepParams rp{};
  rp.desc = dst;
  rp.m = idx->cfg.ref_kp;
  rp.cpr = idx->cpr;
  rp.count = take;
  rp.colkey = sg.colkey + pos * idx->cpr * kColInts;
  rp.search = 1;
  if (src_dev) {
    rp.src = src;
  } else {
    CU(cudaMemcpy(dst, src, static_cast<size_t>(take * rb), cudaMemcpyHostToDevice));
    rp.src = nullptr;
  }
  TRY(idx->ws_kp.ensure(static_cast<size_t>(take) * 4, "kp staging"));
  CU(cudaMemcpy(idx->ws_kp.p, kp_host, static_cast<size_t>(take) * 4, cudaMemcpyHostToDevice));
  rp.kp = idx->ws_kp.as<int32_t>();
  launch_ref_prep(rp, nullptr);
  CU(cudaGetLastError());
  CU(cudaStreamSynchronize(nullptr));
  return TID_OK;
}

// FIFO swap-out (§6.1): move the oldest HBM segment to the pinned host tier.
tid_status evict_oldest_hbm(tid_index* idx) {
  Segment* victim = nullptr;
  for (Segment& sg : idx->segs)
    if (!sg.on_host && sg.count > 0) { victim = &sg; break; }
  if (!victim) return fail(TID_ENOMEM, "nothing to evict from HBM");
  const int64_t rb = idx->ref_bytes;
  if (static_cast<uint64_t>(idx->n_host + victim->count) * rb > idx->host_budget)
    return fail(TID_ENOMEM, "host tier full: cannot swap out %lld references", static_cast<long long>(victim->count));
  Segment hs;
  TRY(alloc_segment(idx, true, victim->count, &hs));
  // the arena copy has padding rows zeroed and is otherwise identical to what was added
  if (cudaMemcpy(hs.desc, victim->desc, static_cast<size_t>(victim->count * rb), cudaMemcpyDeviceToHost) != cudaSuccess) {
    cudaGetLastError();
    free_segment(idx, hs);
    return fail(TID_ECUDA, "swap-out copy failed");
  }
  hs.first = victim->first;
  hs.count = victim->count;
  hs.kp = std::move(victim->kp);
  idx->n_hbm -= victim->count;
  idx->n_host += victim->count;
  free_segment(idx, *victim);
  *victim = std::move(hs);
  return TID_OK;
}

Segment* find_segment(tid_index* idx, int64_t id, int64_t* off) {
  for (Segment& sg : idx->segs)
    if (id >= sg.first && id < sg.first + sg.count) { *off = id - sg.first; return &sg; }
  return nullptr;
}

tid_status sync_dead(tid_index* idx, cudaStream_t s) {
  if (!idx->any_dead || !idx->dead_dirty) return TID_OK;
  TRY(idx->dead_dev.ensure(idx->dead.size(), "dead flags"));
  CU(cudaMemcpyAsync(idx->dead_dev.p, idx->dead.data(), idx->dead.size(), cudaMemcpyHostToDevice, s));
  CU(cudaStreamSynchronize(s));
  idx->dead_dirty = false;
  return TID_OK;
}

// Stage queries / n_q on the device.
tid_status stage_queries(tid_index* idx, const uint8_t* queries, const int32_t* n_q, int32_t n, int64_t B,
                         const uint8_t** dq, const int32_t** dnv, cudaStream_t s) {
  if (is_device_ptr(queries)) {
    if (reinterpret_cast<uintptr_t>(queries) % 16) return fail(TID_EINVAL, "queries must be 16-byte aligned");
    *dq = queries;
  } else {
    TRY(idx->ws_q.ensure(static_cast<size_t>(B) * n * kDim, "query staging"));
    TRY(copy_in(idx, idx->ws_q.p, queries, static_cast<size_t>(B) * n * kDim, s));
    *dq = idx->ws_q.as<uint8_t>();
  }
  *dnv = nullptr;
  if (n_q) {
    TRY(idx->ws_nvalid.ensure(static_cast<size_t>(B) * 4, "n_q"));
    TRY(copy_in(idx, idx->ws_nvalid.p, n_q, static_cast<size_t>(B) * 4, s));
    *dnv = idx->ws_nvalid.as<int32_t>();
  }
  return TID_OK;
}

tid_status check_search_args(tid_index* idx, const uint8_t* queries, int32_t n, int64_t B) {
  if (!idx) return fail(TID_EINVAL, "null index");
  if (!queries) return fail(TID_EINVAL, "null queries");
  if (n < 1 || n > idx->cfg.query_kp_max) return fail(TID_EINVAL, "n=%d outside 1..query_kp_max=%d", n, idx->cfg.query_kp_max);
  if (B < 1) return fail(TID_EINVAL, "B=%lld must be >= 1", static_cast<long long>(B));
  if (B > (1LL << 31) / 2) return fail(TID_EINVAL, "B too large");
  return TID_OK;
}

}  // namespace

// =====================================================================================
extern "C" {

const char* tid_last_error(void) { return g_err.c_str(); }

tid_status tid_nccl_unique_id(void* out128) {
  if (!out128) return fail(TID_EINVAL, "null output");
  ncclUniqueId id;
  NC(nccl().GetUniqueId(&id));
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  memcpy(out128, &id, sizeof(id));
  return TID_OK;
}

tid_status tid_index_create(const tid_config* cfg, tid_index** out) {
  if (!cfg || !out) return fail(TID_EINVAL, "null argument");
  *out = nullptr;
  if (cfg->dim != kDim) return fail(TID_EINVAL, "dim=%d: only 128-d SIFT descriptors are supported", cfg->dim);
  if (cfg->ref_kp < 2 || cfg->ref_kp > kMaxSlots * kBN)
    return fail(TID_EINVAL, "ref_kp=%d outside 2..%d", cfg->ref_kp, kMaxSlots * kBN);
  if (cfg->query_kp_max < 1 || cfg->query_kp_max > 8192)
    return fail(TID_EINVAL, "query_kp_max=%d outside 1..8192", cfg->query_kp_max);
  if (cfg->ratio_num < 1 || cfg->ratio_num > 65535 || cfg->ratio_den < 1 || cfg->ratio_den > 65535)
    return fail(TID_EINVAL, "ratio %u/%u: num and den must be in 1..65535", cfg->ratio_num, cfg->ratio_den);
  if (cfg->world_size < 1 || cfg->rank < 0 || cfg->rank >= cfg->world_size)
    return fail(TID_EINVAL, "rank %d / world_size %d invalid", cfg->rank, cfg->world_size);
  if (cfg->world_size > 1 && !cfg->nccl_unique_id) return fail(TID_EINVAL, "world_size > 1 needs nccl_unique_id");
  if (cfg->id_base < 0) return fail(TID_EINVAL, "id_base must be >= 0");
  if (cfg->descriptor != 0 && cfg->descriptor != 1) return fail(TID_EINVAL, "descriptor must be 0 (u8) or 1 (fp16)");
  if (cfg->descriptor == 1 && cfg->ref_kp > 2 * kBN)
    return fail(TID_EINVAL, "descriptor 1 (float path): ref_kp=%d > 512", cfg->ref_kp);
  if (cfg->descriptor == 1 && !(cfg->f16_scale >= 0.0f)) return fail(TID_EINVAL, "f16_scale must be >= 0");

  int ndev = 0;
  CU(cudaGetDeviceCount(&ndev));
  if (cfg->device < 0 || cfg->device >= ndev) return fail(TID_EINVAL, "device %d not present (%d devices)", cfg->device, ndev);
  cudaDeviceProp prop;
  CU(cudaGetDeviceProperties(&prop, cfg->device));
  if (prop.major != 10 || prop.minor != 0)
    return fail(TID_EUNSUPPORTED, "device %d is sm_%d%d; this library is built for sm_100a (B200)", cfg->device,
                prop.major, prop.minor);
  CU(cudaSetDevice(cfg->device));

  tid_index* idx = new tid_index();
  idx->cfg = *cfg;
  idx->cfg.nccl_unique_id = nullptr;
  idx->device = cfg->device;
  idx->num_sms = prop.multiProcessorCount;
  idx->cpr = static_cast<int>(ceil_div(cfg->ref_kp, kBN));
  idx->in_bytes = static_cast<int64_t>(cfg->ref_kp) * kDim;
  idx->ref_bytes = idx->in_bytes;
  idx->hbm_ref_bytes = idx->ref_bytes + static_cast<int64_t>(idx->cpr) * kColBytes;
  if (cfg->descriptor == 1) {  // row f1: fp16 storage + 256 x 16 fp16 norm terms per reference
    idx->f16 = true;
    idx->f16_scale = cfg->f16_scale > 0.0f ? cfg->f16_scale : 1.0f;
    idx->f16_rootsift = cfg->f16_rootsift ? 1 : 0;
    idx->ref_bytes = 2 * idx->in_bytes;
    idx->hbm_ref_bytes = idx->ref_bytes + static_cast<int64_t>(kBN) * idx->cpr * 16 * 2;
    // C: the smallest power of two >= half the largest N_R the index can hold, so X = C + q.r - N_R/2
    // >= 0 for every reference: RootSIFT rows have unit norm (x (1 + 2^-11)^2 after
    // fp16 rounding), raw SIFT at most 128 * 255^2; both times scale^2.
    const double s2 = static_cast<double>(idx->f16_scale) * idx->f16_scale;
    const double bound = (idx->f16_rootsift ? 1.0 + 1.0 / 512 : 128.0 * 255 * 255) * s2 / 2;
    int e = 0;
    std::frexp(bound, &e);
    idx->f16_c = static_cast<float>(std::ldexp(1.0, e));
  }
  size_t free_b = 0, total_b = 0;
  cudaMemGetInfo(&free_b, &total_b);
  const uint64_t reserve = 8ull << 30;
  // the budget counts descriptor bytes; each resident reference also holds its norm digits and
  // column terms (hbm_ref_bytes - ref_bytes), which the automatic budget leaves room for
  const uint64_t avail = free_b > reserve ? free_b - reserve : free_b / 2;
  idx->hbm_budget = cfg->hbm_budget_bytes ? cfg->hbm_budget_bytes
                                          : avail / static_cast<uint64_t>(idx->hbm_ref_bytes) * idx->ref_bytes;
  idx->host_budget = cfg->host_budget_bytes;
  idx->host_chunk = 16384;
  cudaError_t e = cudaStreamCreateWithFlags(&idx->copy_stream, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&idx->ev_last, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&idx->graph_stream, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&idx->ev_gin, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&idx->ev_gout, cudaEventDisableTiming);
  for (int b = 0; b < 2 && e == cudaSuccess; ++b) {
    e = cudaEventCreateWithFlags(&idx->ev_h2d[b], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&idx->ev_free[b], cudaEventDisableTiming);
  }
  if (e != cudaSuccess) {
    tid_index_destroy(idx);
    return fail(TID_ECUDA, "stream/event creation: %s", cudaGetErrorString(e));
  }
  if (idx->f16) {
    if (idx->ws_f16c.ensure(4, "f16 constant") != TID_OK ||
        cudaMemcpy(idx->ws_f16c.p, &idx->f16_c, 4, cudaMemcpyHostToDevice) != cudaSuccess) {
      tid_index_destroy(idx);
      return fail(TID_ENOMEM, "f16 constant allocation failed");
    }
  }
  if (cfg->world_size > 1 || cfg->nccl_unique_id) {  // a 1-rank communicator exercises the same path
    ncclUniqueId id;
    memcpy(&id, cfg->nccl_unique_id, sizeof(id));
    if (!nccl().ok) {
      tid_index_destroy(idx);
      return fail(TID_ENCCL, "%s", nccl().err.c_str());
    }
    ncclResult_t r = nccl().CommInitRank(&idx->comm, cfg->world_size, id, cfg->rank);
    if (r != ncclSuccess) {
      idx->comm = nullptr;
      tid_index_destroy(idx);
      return fail(TID_ENCCL, "ncclCommInitRank: %s", nccl().GetErrorString(r));
    }
  }
  *out = idx;
  return TID_OK;
}

tid_status tid_index_destroy(tid_index* idx) {
  if (!idx) return TID_OK;
  cudaSetDevice(idx->device);
  cudaDeviceSynchronize();
  for (Segment& sg : idx->segs) free_segment(idx, sg);
  idx->dead_dev.release();
  DevBuf* bufs[] = {&idx->ws_q, &idx->ws_nq, &idx->ws_nvalid, &idx->ws_counts, &idx->ws_cand, &idx->ws_keys,
                    &idx->ws_gather, &idx->ws_ids, &idx->ws_cnts, &idx->ws_r, &idx->ws_colkey, &idx->ws_nn,
                    &idx->ws_kp, &idx->ws_mr, &idx->stage_desc[0], &idx->stage_desc[1], &idx->stage_colkey[0],
                    &idx->stage_colkey[1], &idx->stage_kp[0], &idx->stage_kp[1], &idx->ws_qs, &idx->ws_geo_nn, &idx->ws_geo_cnt,
                    &idx->ws_u8, &idx->ws_f16c, &idx->ws_f16kp, &idx->ws_f16rows, &idx->stage_xop[0], &idx->stage_xop[1],
                    &idx->ws_geo_xy, &idx->ws_geo_out, &idx->ws_f16q, &idx->ws_f16r, &idx->ws_f16nq,
                    &idx->ws_f16nr, &idx->ws_f16in};
  for (DevBuf* b : bufs) b->release();
  for (auto& pr : idx->prof_ev) { cudaEventDestroy(pr.first); cudaEventDestroy(pr.second); }
  for (int b = 0; b < 2; ++b) {
    if (idx->ev_h2d[b]) cudaEventDestroy(idx->ev_h2d[b]);
    if (idx->ev_free[b]) cudaEventDestroy(idx->ev_free[b]);
  }
  if (idx->copy_stream) cudaStreamDestroy(idx->copy_stream);
  if (idx->ev_last) cudaEventDestroy(idx->ev_last);
  for (auto& ge : idx->graphs)
    if (ge.exec) cudaGraphExecDestroy(ge.exec);
  if (idx->graph_stream) cudaStreamDestroy(idx->graph_stream);
  if (idx->ev_gin) cudaEventDestroy(idx->ev_gin);
  if (idx->ev_gout) cudaEventDestroy(idx->ev_gout);
  if (idx->h_rtot) cudaFreeHost(idx->h_rtot);
  idx->ws_rtot.release();
  if (idx->comm) nccl().CommDestroy(idx->comm);
  delete idx;
  return TID_OK;
}

tid_status tid_add_references(tid_index* idx, const uint8_t* desc, const int32_t* kp_counts, int64_t count,
                              int64_t* first_local_id) {
  if (!idx) return fail(TID_EINVAL, "null index");
  if (count < 0) return fail(TID_EINVAL, "count < 0");
  if (count > 0 && !desc) return fail(TID_EINVAL, "null descriptors");
  TRY(set_device(idx));
  CallGuard guard(idx, nullptr);
  ++idx->gen;  // segments may change (FIFO swap-outs) even if the add fails
  const int64_t first = idx->n_hbm + idx->n_host;
  if (first_local_id) *first_local_id = first;
  if (count == 0) return TID_OK;
  const int64_t rb = idx->ref_bytes;
  const bool dev_in = is_device_ptr(desc);
  // keypoint counts: host copy, validated
  std::vector<int32_t> kp(static_cast<size_t>(count), idx->cfg.ref_kp);
  if (kp_counts) {
    CU(cudaMemcpy(kp.data(), kp_counts, static_cast<size_t>(count) * 4, cudaMemcpyDefault));
    for (int64_t i = 0; i < count; ++i)
      if (kp[i] < 0 || kp[i] > idx->cfg.ref_kp)
        return fail(TID_EINVAL, "kp_counts[%lld]=%d outside 0..ref_kp", static_cast<long long>(i), kp[i]);
  }
  const int64_t hbm_cap = static_cast<int64_t>(idx->hbm_budget / rb);
  const int64_t host_cap = static_cast<int64_t>(idx->host_budget / rb);
  int64_t to_hbm, to_host;
  if (idx->cfg.cache_policy == 1) {
    // FIFO (paper §6.1): the new batch enters HBM; the oldest batches are swapped to the host tier
    if (count > hbm_cap) return fail(TID_ENOMEM, "batch of %lld exceeds the HBM budget", static_cast<long long>(count));
    int64_t evict_need = idx->n_hbm + count - hbm_cap;
    if (evict_need > 0 && idx->n_host + evict_need > host_cap)
      return fail(TID_ENOMEM, "capacity exceeded: HBM full and host tier cannot take the swapped-out batches");
    while (idx->n_hbm + count > hbm_cap) TRY(evict_oldest_hbm(idx));
    to_hbm = count;
    to_host = 0;
  } else {
    // fill: HBM first, then the host tier (ids stay in insertion order)
    const int64_t hbm_room = idx->n_host > 0 ? 0 : std::max<int64_t>(hbm_cap - idx->n_hbm, 0);
    to_hbm = std::min(count, hbm_room);
    to_host = count - to_hbm;
    if (to_host > host_cap - idx->n_host)
      return fail(TID_ENOMEM, "capacity exceeded: %lld references do not fit (HBM room %lld, host room %lld)",
                  static_cast<long long>(count), static_cast<long long>(hbm_room),
                  static_cast<long long>(host_cap - idx->n_host));
  }
  // ---- transaction: from here on a failure rolls the index back to its state before the call
  // (segments created by this call freed, the tail segment's count restored, counters restored),
  // so TID_ENOMEM / TID_ECUDA add nothing.  (FIFO swap-outs above are not undone: they move
  // whole batches between tiers and change neither ids nor search results.)
  const size_t segs0 = idx->segs.size();
  const int64_t tail_count0 = segs0 ? idx->segs.back().count : 0;
  const int64_t n_hbm0 = idx->n_hbm, n_host0 = idx->n_host;
  auto rollback = [&](tid_status st) -> tid_status {
    const std::string msg = g_err;
    cudaStreamSynchronize(nullptr);
    cudaGetLastError();
    while (idx->segs.size() > segs0) {
      free_segment(idx, idx->segs.back());
      idx->segs.pop_back();
    }
    if (segs0) {
      Segment& t = idx->segs.back();
      t.count = tail_count0;
      t.kp.resize(static_cast<size_t>(tail_count0));
    }
    idx->n_hbm = n_hbm0;
    idx->n_host = n_host0;
    g_err = msg;
    return st;
  };
#define TRY_TX(x)                            \
  do {                                       \
    tid_status s__ = (x);                    \
    if (s__ != TID_OK) return rollback(s__); \
  } while (0)
  // ---- HBM part (append to the last HBM segment if it is the id-tail and has room, else a new one)
  int64_t done = 0;
  while (done < to_hbm) {
    Segment* sg = idx->segs.empty() ? nullptr : &idx->segs.back();
    const bool can_append = sg && !sg->on_host && sg->count < sg->cap && idx->cfg.cache_policy == 0;
    if (!can_append) {
      const int64_t room = hbm_cap - idx->n_hbm;
      int64_t cap = idx->cfg.cache_policy == 1 ? (to_hbm - done)
                                               : std::max<int64_t>(to_hbm - done, std::min<int64_t>(idx->n_hbm, room));
      cap = std::min(cap, room);
      Segment ns;
      TRY_TX(alloc_segment(idx, false, cap, &ns));
      ns.first = first + done;
      idx->segs.push_back(std::move(ns));
      sg = &idx->segs.back();
    }
    const int64_t take = std::min(to_hbm - done, sg->cap - sg->count);
    TRY_TX(ingest_hbm(idx, *sg, sg->count, desc + done * idx->in_bytes, dev_in, kp.data() + done, take));
    sg->kp.insert(sg->kp.end(), kp.begin() + done, kp.begin() + done + take);
    sg->count += take;
    idx->n_hbm += take;
    done += take;
  }
  // ---- host-tier part (raw bytes; zeroing + keys happen on the GPU when streamed)
  int64_t hdone = 0;
  while (hdone < to_host) {
    Segment* sg = idx->segs.empty() ? nullptr : &idx->segs.back();
    if (!sg || !sg->on_host || sg->count == sg->cap) {
      const int64_t room = host_cap - idx->n_host;
      int64_t cap = std::max<int64_t>(to_host - hdone, std::min<int64_t>(idx->n_host, room));
      cap = std::min(cap, room);
      Segment ns;
      TRY_TX(alloc_segment(idx, true, cap, &ns));
      ns.first = first + to_hbm + hdone;
      idx->segs.push_back(std::move(ns));
      sg = &idx->segs.back();
    }
    const int64_t take = std::min(to_host - hdone, sg->cap - sg->count);
    if (idx->f16) {  // convert on the GPU, then into the pinned tier (fp16)
      for (int64_t o = 0; o < take;) {
        const int64_t c = std::min<int64_t>(take - o, 8192);
        TRY_TX(idx->ws_f16r.ensure(static_cast<size_t>(c * rb), "f16 conversion"));
        TRY_TX(convert_f16(idx, desc + (to_hbm + hdone + o) * idx->in_bytes, dev_in, c, idx->ws_f16r.p));
        if (cudaMemcpy(sg->desc + (sg->count + o) * rb, idx->ws_f16r.p, static_cast<size_t>(c * rb),
                       cudaMemcpyDeviceToHost) != cudaSuccess)
          return rollback(fail(TID_ECUDA, "host-tier copy: %s", cudaGetErrorString(cudaGetLastError())));
        o += c;
      }
    } else if (cudaMemcpy(sg->desc + sg->count * rb, desc + (to_hbm + hdone) * rb, static_cast<size_t>(take * rb),
                          cudaMemcpyDefault) != cudaSuccess) {
      return rollback(fail(TID_ECUDA, "host-tier copy: %s", cudaGetErrorString(cudaGetLastError())));
    }
    sg->kp.insert(sg->kp.end(), kp.begin() + to_hbm + hdone, kp.begin() + to_hbm + hdone + take);
    sg->count += take;
    idx->n_host += take;
    hdone += take;
  }
#undef TRY_TX
  idx->dead.resize(static_cast<size_t>(first + count), 0);
  idx->dead_dirty = true;
  ++idx->gen;  // cached search graphs are stale
  return TID_OK;
}

tid_status tid_host_tier_map(tid_index* idx, int64_t count, uint8_t** desc_out, int64_t* first_local_id) {
  if (!idx) return fail(TID_EINVAL, "null index");
  if (count < 1 || !desc_out) return fail(TID_EINVAL, "count < 1 or null desc_out");
  if (idx->cfg.cache_policy == 1) return fail(TID_ESTATE, "FIFO policy: the host tier holds evicted batches only");
  TRY(set_device(idx));
  CallGuard guard(idx, nullptr);
  CU(cudaStreamSynchronize(nullptr));  // a search may still be streaming the tier
  const int64_t rb = idx->ref_bytes;
  const int64_t host_cap = static_cast<int64_t>(idx->host_budget / rb);
  if (count > host_cap - idx->n_host)
    return fail(TID_ENOMEM, "host tier room %lld < %lld", static_cast<long long>(host_cap - idx->n_host),
                static_cast<long long>(count));
  const int64_t first = idx->n_hbm + idx->n_host;
  Segment ns;
  TRY(alloc_segment(idx, true, count, &ns));
  memset(ns.desc, 0, static_cast<size_t>(count * rb));
  ns.first = first;
  ns.count = count;
  ns.kp.assign(static_cast<size_t>(count), idx->cfg.ref_kp);
  *desc_out = ns.desc;
  idx->segs.push_back(std::move(ns));
  idx->n_host += count;
  idx->dead.resize(static_cast<size_t>(first + count), 0);
  idx->dead_dirty = true;
  ++idx->gen;  // cached search graphs are stale
  if (first_local_id) *first_local_id = first;
  return TID_OK;
}

tid_status tid_delete_references(tid_index* idx, const int64_t* local_ids, int64_t count) {
  if (!idx) return fail(TID_EINVAL, "null index");
  if (count < 0 || (count > 0 && !local_ids)) return fail(TID_EINVAL, "bad ids");
  TRY(set_device(idx));
  CallGuard guard(idx, nullptr);
  std::vector<int64_t> ids(static_cast<size_t>(count));
  if (count) CU(cudaMemcpy(ids.data(), local_ids, static_cast<size_t>(count) * 8, cudaMemcpyDefault));
  const int64_t R = idx->n_hbm + idx->n_host;
  for (int64_t id : ids)
    if (id < 0 || id >= R) return fail(TID_EINVAL, "local id %lld out of range", static_cast<long long>(id));
  const int32_t zero = 0;
  for (int64_t id : ids) {
    int64_t off;
    Segment* sg = find_segment(idx, id, &off);
    sg->kp[off] = 0;  // no keypoints: every column becomes padding -> count 0
    if (!sg->on_host && idx->f16) {
      TRY(idx->ws_kp.ensure(4, "kp"));
      CU(cudaMemcpy(idx->ws_kp.p, &zero, 4, cudaMemcpyHostToDevice));
      TRY(f16_norm_terms(idx, sg->desc + off * idx->ref_bytes, 1, idx->ws_kp.as<int32_t>(),
                         sg->xop + static_cast<size_t>(off) * kBN * idx->cpr * 16, nullptr));
      CU(cudaStreamSynchronize(nullptr));
    } else if (!sg->on_host) {
      RefPrepParams rp{};
      rp.desc = sg->desc + off * idx->ref_bytes;
      rp.src = nullptr;
      TRY(idx->ws_kp.ensure(4, "kp"));
      CU(cudaMemcpy(idx->ws_kp.p, &zero, 4, cudaMemcpyHostToDevice));
      rp.kp = idx->ws_kp.as<int32_t>();
      rp.colkey = sg->colkey + off * idx->cpr * kColInts;
      rp.search = 1;
      rp.count = 1;
      rp.m = idx->cfg.ref_kp;
      rp.cpr = idx->cpr;
      launch_ref_prep(rp, nullptr);
      CU(cudaStreamSynchronize(nullptr));
    }
    idx->dead[static_cast<size_t>(id)] = 1;
  }
  idx->any_dead = idx->any_dead || count > 0;
  idx->dead_dirty = true;
  ++idx->gen;  // cached search graphs are stale
  return TID_OK;
}

tid_status tid_update_references(tid_index* idx, const int64_t* local_ids, const uint8_t* desc,
                                 const int32_t* kp_counts, int64_t count) {
  if (!idx) return fail(TID_EINVAL, "null index");
  if (count < 0 || (count > 0 && (!local_ids || !desc))) return fail(TID_EINVAL, "bad arguments");
  TRY(set_device(idx));
  CallGuard guard(idx, nullptr);
  std::vector<int64_t> ids(static_cast<size_t>(count));
  if (count) CU(cudaMemcpy(ids.data(), local_ids, static_cast<size_t>(count) * 8, cudaMemcpyDefault));
  std::vector<int32_t> kp(static_cast<size_t>(count), idx->cfg.ref_kp);
  if (kp_counts && count) CU(cudaMemcpy(kp.data(), kp_counts, static_cast<size_t>(count) * 4, cudaMemcpyDefault));
  const int64_t R = idx->n_hbm + idx->n_host;
  for (int64_t i = 0; i < count; ++i) {
    if (ids[i] < 0 || ids[i] >= R) return fail(TID_EINVAL, "local id %lld out of range", static_cast<long long>(ids[i]));
    if (kp[i] < 0 || kp[i] > idx->cfg.ref_kp) return fail(TID_EINVAL, "kp_counts[%lld] out of range", static_cast<long long>(i));
  }
  const int64_t rb = idx->ref_bytes;
  const bool dev_in = is_device_ptr(desc);
  for (int64_t i = 0; i < count; ++i) {
    int64_t off;
    Segment* sg = find_segment(idx, ids[i], &off);
    if (sg->on_host && idx->f16) {
      TRY(idx->ws_f16r.ensure(static_cast<size_t>(rb), "f16 conversion"));
      TRY(convert_f16(idx, desc + i * idx->in_bytes, dev_in, 1, idx->ws_f16r.p));
      CU(cudaMemcpy(sg->desc + off * rb, idx->ws_f16r.p, static_cast<size_t>(rb), cudaMemcpyDeviceToHost));
    } else if (sg->on_host) {
      CU(cudaMemcpy(sg->desc + off * rb, desc + i * rb, static_cast<size_t>(rb), cudaMemcpyDefault));
    } else {
      TRY(ingest_hbm(idx, *sg, off, desc + i * idx->in_bytes, dev_in, &kp[i], 1));
    }
    sg->kp[off] = kp[i];
    idx->dead[static_cast<size_t>(ids[i])] = 0;
  }
  idx->dead_dirty = true;
  ++idx->gen;  // cached search graphs are stale
  return TID_OK;
}

// File layout (little endian): "TIDX" u32 version=1 | i32 dim | i32 ref_kp | i64 num_refs |
// i32 kp[num_refs] | u8 dead[num_refs] | u8 desc[num_refs][ref_kp][128] (padding rows zeroed).
tid_status tid_index_save(const tid_index* cidx, const char* path) {
  tid_index* idx = const_cast<tid_index*>(cidx);
  if (!idx || !path) return fail(TID_EINVAL, "null argument");
  if (idx->f16) return fail(TID_EUNSUPPORTED, "save: float (descriptor 1) indexes are not persisted");
  TRY(set_device(idx));
  CU(cudaEventSynchronize(idx->ev_last));
  FILE* f = fopen(path, "wb");
  if (!f) return fail(TID_EINVAL, "cannot open %s for writing", path);
  const int64_t R = idx->n_hbm + idx->n_host, rb = idx->ref_bytes;
  const uint32_t ver = 1;
  const int32_t dim = kDim, m = idx->cfg.ref_kp;
  bool ok = fwrite("TIDX", 1, 4, f) == 4 && fwrite(&ver, 4, 1, f) == 1 && fwrite(&dim, 4, 1, f) == 1 &&
            fwrite(&m, 4, 1, f) == 1 && fwrite(&R, 8, 1, f) == 1;
  for (const Segment& sg : idx->segs) ok = ok && fwrite(sg.kp.data(), 4, sg.kp.size(), f) == sg.kp.size();
  ok = ok && fwrite(idx->dead.data(), 1, idx->dead.size(), f) == idx->dead.size();
  std::vector<uint8_t> buf;
  for (const Segment& sg : idx->segs) {
    const int64_t chunk = 4096;
    for (int64_t off = 0; ok && off < sg.count; off += chunk) {
      const int64_t c = std::min(chunk, sg.count - off);
      buf.resize(static_cast<size_t>(c * rb));
      if (cudaMemcpy(buf.data(), sg.desc + off * rb, buf.size(), cudaMemcpyDefault) != cudaSuccess) {
        cudaGetLastError();
        ok = false;
        break;
      }
      if (sg.on_host)  // the host tier keeps raw rows: zero padding rows so the file is canonical
        for (int64_t r = 0; r < c; ++r)
          for (int32_t i = sg.kp[off + r]; i < m; ++i) memset(buf.data() + (r * m + i) * kDim, 0, kDim);
      ok = ok && fwrite(buf.data(), 1, buf.size(), f) == buf.size();
    }
  }
  fclose(f);
  if (!ok) return fail(TID_ECUDA, "write to %s failed", path);
  return TID_OK;
}

tid_status tid_index_load(tid_index* idx, const char* path, int64_t* first_local_id) {
  if (!idx || !path) return fail(TID_EINVAL, "null argument");
  if (idx->f16) return fail(TID_EUNSUPPORTED, "load: float (descriptor 1) indexes are not persisted");
  FILE* f = fopen(path, "rb");
  if (!f) return fail(TID_EINVAL, "cannot open %s", path);
  char magic[4];
  uint32_t ver = 0;
  int32_t dim = 0, m = 0;
  int64_t R = 0;
  bool ok = fread(magic, 1, 4, f) == 4 && memcmp(magic, "TIDX", 4) == 0 && fread(&ver, 4, 1, f) == 1 && ver == 1 &&
            fread(&dim, 4, 1, f) == 1 && fread(&m, 4, 1, f) == 1 && fread(&R, 8, 1, f) == 1;
  if (!ok || dim != kDim || m != idx->cfg.ref_kp || R < 0) {
    fclose(f);
    return fail(TID_EINVAL, "%s: not a tid index file for ref_kp=%d", path, idx->cfg.ref_kp);
  }
  std::vector<int32_t> kp(static_cast<size_t>(R));
  std::vector<uint8_t> dead(static_cast<size_t>(R));
  ok = fread(kp.data(), 4, kp.size(), f) == kp.size() && fread(dead.data(), 1, dead.size(), f) == dead.size();
  const int64_t rb = idx->ref_bytes, first = idx->n_hbm + idx->n_host;
  std::vector<uint8_t> buf;
  int64_t chunk = 16384;
  if (idx->cfg.cache_policy == 1)  // FIFO batches must fit in HBM; keep half of it for the swap
    chunk = std::max<int64_t>(1, std::min<int64_t>(chunk, static_cast<int64_t>(idx->hbm_budget / rb) / 2));
  for (int64_t off = 0; ok && off < R; off += chunk) {
    const int64_t c = std::min(chunk, R - off);
    buf.resize(static_cast<size_t>(c * rb));
    ok = fread(buf.data(), 1, buf.size(), f) == buf.size();
    if (ok) {
      tid_status st = tid_add_references(idx, buf.data(), kp.data() + off, c, nullptr);
      if (st != TID_OK) { fclose(f); return st; }
    }
  }
  fclose(f);
  if (!ok) return fail(TID_EINVAL, "%s: truncated", path);
  std::vector<int64_t> del;
  for (int64_t i = 0; i < R; ++i)
    if (dead[i]) del.push_back(first + i);
  if (!del.empty()) TRY(tid_delete_references(idx, del.data(), static_cast<int64_t>(del.size())));
  if (first_local_id) *first_local_id = first;
  return TID_OK;
}

tid_status tid_search_counts(tid_index* idx, const uint8_t* queries, const int32_t* n_q, int32_t n, int64_t B,
                             uint32_t* counts_out, void* stream) {
  TRY(check_search_args(idx, queries, n, B));
  if (!counts_out) return fail(TID_EINVAL, "null counts_out");
  const int64_t R = idx->n_hbm + idx->n_host;
  if (R == 0) return fail(TID_ESTATE, "index holds no references");
  TRY(set_device(idx));
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  CallGuard guard(idx, s);
  const uint8_t* dq;
  const int32_t* dnv;
  TRY(stage_queries(idx, queries, n_q, n, B, &dq, &dnv, s));
  const bool dev_out = is_device_ptr(counts_out);
  uint32_t* counts = counts_out;
  if (!dev_out) {
    TRY(idx->ws_counts.ensure(static_cast<size_t>(B) * R * 4, "count matrix"));
    counts = idx->ws_counts.as<uint32_t>();
  }
  // one window = every local reference: the output IS the full count matrix
  TRY(run_pass(idx, dq, dnv, n, B, R, counts, s, [](int64_t, int64_t) { return TID_OK; }));
  bool host_out = false;
  if (!dev_out) TRY(copy_out(idx, counts_out, counts, static_cast<size_t>(B) * R * 4, s, &host_out));
  if (host_out) CU(cudaStreamSynchronize(s));
  CU(cudaGetLastError());
  return TID_OK;
}

namespace {
// Collective: the total reference count over all ranks (one NCCL all-reduce of an int64).
tid_status total_references(tid_index* idx, cudaStream_t s, int64_t* out) {
  const int64_t R = idx->n_hbm + idx->n_host;
  if (idx->comm == nullptr) {
    *out = R;
    return TID_OK;
  }
  if (!idx->h_rtot) {
    if (cudaHostAlloc(reinterpret_cast<void**>(&idx->h_rtot), 8, cudaHostAllocPortable) != cudaSuccess) {
      cudaGetLastError();
      idx->h_rtot = nullptr;
      return fail(TID_ENOMEM, "pinned scalar allocation failed");
    }
  }
  TRY(idx->ws_rtot.ensure(8, "reference total"));
  *idx->h_rtot = R;
  CU(cudaMemcpyAsync(idx->ws_rtot.p, idx->h_rtot, 8, cudaMemcpyHostToDevice, s));
  NC(nccl().AllReduce(idx->ws_rtot.p, idx->ws_rtot.p, 1, ncclInt64, ncclSum, idx->comm, s));
  CU(cudaMemcpyAsync(idx->h_rtot, idx->ws_rtot.p, 8, cudaMemcpyDeviceToHost, s));
  CU(cudaStreamSynchronize(s));
  *out = *idx->h_rtot;
  return TID_OK;
}
}  // namespace

}  // extern "C"

namespace {
// Replay of a captured search (the launch-bound small-batch path pays one graph launch instead of
// ~5 kernel / memset submissions).  A call shape (buffers, n, B, k) is captured on its second
// occurrence (the first sizes every workspace), on the index's own non-blocking stream, joined to
// the caller's stream by events; the graph is replayed while the index generation (references,
// deleted flags, tuning) and every workspace pointer it baked in are unchanged.
std::vector<void*> graph_ws(const tid_index* idx) {
  return {idx->ws_q.p,     idx->ws_nq.p,    idx->ws_nvalid.p, idx->ws_counts.p, idx->ws_cand.p,
          idx->ws_qs.p,    idx->dead_dev.p, idx->ws_f16q.p,   idx->ws_f16nq.p,  idx->ws_f16c.p};
}

template <class Enqueue>
tid_status search_graph(tid_index* idx, const void* q, const void* nq, int32_t n, int64_t B, int32_t k, void* ids,
                        void* cnts, cudaStream_t s, Enqueue& enqueue) {
  const std::vector<void*> ws = graph_ws(idx);
  tid_index::GraphEntry* e = nullptr;
  for (auto& ge : idx->graphs)
    if (ge.q == q && ge.nq == nq && ge.ids == ids && ge.cnts == cnts && ge.n == n && ge.k == k && ge.B == B) {
      e = &ge;
      break;
    }
  if (e && (e->gen != idx->gen || e->ws != ws)) {  // stale: drop the graph, start over
    if (e->exec) cudaGraphExecDestroy(e->exec);
    e->exec = nullptr;
    e->uses = 0;
    e->gen = idx->gen;
    e->ws = ws;
  }
  if (!e) {
    if (idx->graphs.size() >= 8) {  // small cache: evict the oldest
      if (idx->graphs.front().exec) cudaGraphExecDestroy(idx->graphs.front().exec);
      idx->graphs.erase(idx->graphs.begin());
    }
    tid_index::GraphEntry ne;
    ne.q = q; ne.nq = nq; ne.ids = ids; ne.cnts = cnts; ne.n = n; ne.k = k; ne.B = B;
    ne.gen = idx->gen;
    ne.ws = ws;
    idx->graphs.push_back(ne);
    e = &idx->graphs.back();
  }
  if (e->uses < 0 || ++e->uses < 2) return enqueue(s);  // first occurrence (or not capturable): direct
  if (!e->exec) {
    // capture on the index's own stream (the caller's may be the legacy default stream, which cannot
    // be captured), ordered after the caller's prior work
    CU(cudaEventRecord(idx->ev_gin, s));
    CU(cudaStreamWaitEvent(idx->graph_stream, idx->ev_gin, 0));
    CU(cudaStreamBeginCapture(idx->graph_stream, cudaStreamCaptureModeThreadLocal));
    const tid_status st = enqueue(idx->graph_stream);
    cudaGraph_t g = nullptr;
    const cudaError_t ce = cudaStreamEndCapture(idx->graph_stream, &g);
    cudaGraphExec_t exec = nullptr;
    const bool ok = st == TID_OK && ce == cudaSuccess && g && cudaGraphInstantiate(&exec, g, 0) == cudaSuccess;
    if (g) cudaGraphDestroy(g);
    if (!ok || graph_ws(idx) != ws) {  // not capturable (or a workspace moved): direct from now on
      cudaGetLastError();
      if (exec) cudaGraphExecDestroy(exec);
      e->uses = -1;
      CU(cudaEventRecord(idx->ev_gout, idx->graph_stream));
      CU(cudaStreamWaitEvent(s, idx->ev_gout, 0));
      return enqueue(s);
    }
    e->exec = exec;
    CU(cudaEventRecord(idx->ev_gout, idx->graph_stream));  // the caller's stream waits for the capture point
    CU(cudaStreamWaitEvent(s, idx->ev_gout, 0));
  }
  CU(cudaGraphLaunch(e->exec, s));  // replay straight on the caller's stream (any stream may launch a graph)
  return TID_OK;
}
}  // namespace

extern "C" {

tid_status tid_search(tid_index* idx, const uint8_t* queries, const int32_t* n_q, int32_t n, int64_t B, int32_t k,
                      int64_t* ref_ids_out, int32_t* match_counts_out, void* stream) {
  TRY(check_search_args(idx, queries, n, B));
  if (!ref_ids_out || !match_counts_out) return fail(TID_EINVAL, "null outputs");
  if (k < 1 || k > 64) return fail(TID_EINVAL, "k=%d outside 1..64", k);
  TRY(set_device(idx));
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  CallGuard guard(idx, s);
  const int64_t R = idx->n_hbm + idx->n_host;
  // k <= total references, decided identically on every rank (collective count with NCCL), so a
  // rank never leaves the others waiting in the all-gather below
  int64_t R_total = 0;
  TRY(total_references(idx, s, &R_total));
  if (R_total == 0) return fail(TID_ESTATE, "index holds no references");
  if (k > R_total)
    return fail(TID_EINVAL, "k=%d exceeds the number of references (%lld)", k, static_cast<long long>(R_total));
  TRY(sync_dead(idx, s));
  TRY(idx->ws_ids.ensure(static_cast<size_t>(B) * k * 8, "ids"));
  TRY(idx->ws_cnts.ensure(static_cast<size_t>(B) * k * 4, "counts"));
  const bool dev_ids = is_device_ptr(ref_ids_out), dev_cnt = is_device_ptr(match_counts_out);
  int64_t* ids = dev_ids ? ref_ids_out : idx->ws_ids.as<int64_t>();
  int32_t* cnts = dev_cnt ? match_counts_out : idx->ws_cnts.as<int32_t>();
  const bool collective = idx->comm != nullptr;
  if (collective) TRY(idx->ws_keys.ensure(static_cast<size_t>(B) * k * 8, "local keys"));
  uint64_t* local_keys = collective ? idx->ws_keys.as<uint64_t>() : nullptr;
  // everything from query staging to the final ranking, enqueued on stream st (also the body of a
  // captured CUDA graph: device-only work, no host synchronisation)
  auto enqueue = [&](cudaStream_t st) -> tid_status {
  const uint8_t* dq = nullptr;
  const int32_t* dnv = nullptr;
  TRY(stage_queries(idx, queries, n_q, n, B, &dq, &dnv, st));
  if (R > 0) {
    // a6: per window, per-(query, segment) top-k of the window's counts, then merge.  One window:
    // merge the segments straight into the result (one segment, no comm: the top-k kernel
    // writes it).  Several windows: the running top-k is list 0 of every query's candidate
    // lists, merged in place with the window's segments after each window.
    const int64_t W = window_refs(idx, B, R);
    const int64_t nwin = ceil_div(R, W);
    auto segs_for = [&](int64_t len) {
      int64_t sg = std::max<int64_t>(1, std::min<int64_t>(ceil_div(2LL * idx->num_sms, B), ceil_div(len, 4096)));
      return static_cast<int32_t>(std::min<int64_t>(sg, 1024));
    };
    const int32_t lists = (nwin > 1 ? 1 : 0) + segs_for(W);
    TRY(idx->ws_cand.ensure(static_cast<size_t>(B) * lists * k * 8, "top-k candidates"));
    TRY(idx->ws_counts.ensure(static_cast<size_t>(B) * W * 4, "count window"));
    uint64_t* cand = idx->ws_cand.as<uint64_t>();
    if (nwin > 1) CU(cudaMemsetAsync(cand, 0, static_cast<size_t>(B) * lists * k * 8, st));  // empty running lists
    const uint8_t* dead = idx->any_dead ? idx->dead_dev.as<uint8_t>() : nullptr;
    uint32_t* counts = idx->ws_counts.as<uint32_t>();
    auto on_window = [&](int64_t w0, int64_t wlen) -> tid_status {
      const int32_t segs = segs_for(wlen);
      const bool last = w0 + wlen >= R;
      if (nwin == 1) {
        const bool direct = !collective && segs == 1;
        launch_topk(counts, B, wlen, W, idx->cfg.id_base + w0, k, segs, dead, cand, lists, 0, st,
                    direct ? ids : nullptr, direct ? cnts : nullptr);
        count_kernel(idx);
        if (!direct) {
          launch_merge(cand, segs, B, k, static_cast<int64_t>(lists) * k, k, local_keys, collective ? nullptr : ids,
                       collective ? nullptr : cnts, st);
          count_kernel(idx);
        }
      } else {
        launch_topk(counts, B, wlen, W, idx->cfg.id_base + w0, k, segs, dead ? dead + w0 : nullptr, cand, lists, 1, st);
        // running top-k (list 0) + this window's segments -> list 0, or the result after the last window
        if (!last) {
          launch_merge(cand, 1 + segs, B, k, static_cast<int64_t>(lists) * k, k, cand, nullptr, nullptr, st,
                       static_cast<int64_t>(lists) * k);
        } else {
          launch_merge(cand, 1 + segs, B, k, static_cast<int64_t>(lists) * k, k, local_keys, collective ? nullptr : ids,
                       collective ? nullptr : cnts, st);
        }
        count_kernel(idx, 2);
      }
      return TID_OK;
    };
    TRY(run_pass(idx, dq, dnv, n, B, W, counts, st, on_window));
  } else {
    // empty shard (collective only): contribute empty candidate lists to the all-gather
    CU(cudaMemsetAsync(local_keys, 0, static_cast<size_t>(B) * k * 8, st));
  }
  if (collective) {
    // a9: local top-k -> NCCL all-gather over NVLink -> identical merge on every rank
    const int G = idx->cfg.world_size;
    TRY(idx->ws_gather.ensure(static_cast<size_t>(G) * B * k * 8, "gathered keys"));
    NC(nccl().AllGather(local_keys, idx->ws_gather.p, static_cast<size_t>(B) * k, ncclUint64, idx->comm, st));
    launch_merge(idx->ws_gather.as<uint64_t>(), G, B, k, k, B * k, nullptr, ids, cnts, st);
    count_kernel(idx);
  }
  return TID_OK;
  };
  // graph path: device queries / outputs, HBM-resident references, no collective, not profiling
  const bool graphable = !collective && idx->n_host == 0 && !idx->prof && dev_ids && dev_cnt &&
                         is_device_ptr(queries) && (!n_q || is_device_ptr(n_q));
  if (graphable) {
    TRY(search_graph(idx, queries, n_q, n, B, k, ids, cnts, s, enqueue));
  } else {
    TRY(enqueue(s));
  }
  CU(cudaGetLastError());
  bool host_out = false;
  if (!dev_ids) TRY(copy_out(idx, ref_ids_out, ids, static_cast<size_t>(B) * k * 8, s, &host_out));
  if (!dev_cnt) TRY(copy_out(idx, match_counts_out, cnts, static_cast<size_t>(B) * k * 4, s, &host_out));
  if (host_out) CU(cudaStreamSynchronize(s));
  return TID_OK;
}

tid_status tid_verify(tid_index* idx, const uint8_t* q, int32_t n, const uint8_t* r, int32_t m, int64_t P,
                      const int32_t* n_q, const int32_t* m_r, uint32_t* counts_out, int32_t* nn_out, void* stream) {
  if (!idx) return fail(TID_EINVAL, "null index");
  if (!q || !r || !counts_out) return fail(TID_EINVAL, "null argument");
  if (n < 1 || n > idx->cfg.query_kp_max) return fail(TID_EINVAL, "n=%d outside 1..query_kp_max", n);
  if (m < 2 || m > kMaxSlots * kBN) return fail(TID_EINVAL, "m=%d outside 2..%d", m, kMaxSlots * kBN);
  if (P < 1 || P > (1LL << 31) - 1) return fail(TID_EINVAL, "P=%lld invalid", static_cast<long long>(P));
  TRY(set_device(idx));
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  CallGuard guard(idx, s);
  const int cpr = static_cast<int>(ceil_div(m, kBN));
  const int T = static_cast<int>(ceil_div(n, kBM));
  const uint8_t* dq;
  const int32_t* dnv;
  TRY(stage_queries(idx, q, n_q, n, P, &dq, &dnv, s));
  // references: read in place on the device (a host or unaligned buffer is copied); their keys
  // N_R * 256 + i and the masking of rows >= m_r happen inside the match kernel
  const uint8_t* dr = r;
  const size_t rbytes = static_cast<size_t>(P) * m * kDim;
  if (!is_device_ptr(r) || reinterpret_cast<uintptr_t>(r) % 16) {
    TRY(idx->ws_r.ensure(rbytes, "pair references"));
    TRY(copy_in(idx, idx->ws_r.p, r, rbytes, s));
    dr = idx->ws_r.as<uint8_t>();
  }
  const int32_t* dmr = nullptr;
  if (m_r) {
    TRY(idx->ws_mr.ensure(static_cast<size_t>(P) * 4, "m_r"));
    TRY(copy_in(idx, idx->ws_mr.p, m_r, static_cast<size_t>(P) * 4, s));
    dmr = idx->ws_mr.as<int32_t>();
  }
  // counts only: the search path's folded kernel in pair mode (s8 x u8 + the norm K-step, no per-element
  // key arithmetic; column terms and digits computed on chip) — exact like the packed-key kernel, which
  // remains the path that also returns (d1, i1, d2, i2).  TID_VERIFY_FOLD=0 disables it (A/B).
  static const bool fold_ok = [] {
    const char* e = getenv("TID_VERIFY_FOLD");
    return !(e && e[0] == '0');
  }();
  const bool fold = fold_ok && nn_out == nullptr;
  // pairs streamed through per-chunk reference slots, queries shifted / normed on chip (TID_VERIFY_STREAM=0:
  // the job kernel after a query-prep pass, for A/B).  The stream kernel's parity waits assume every
  // group runs a tile of every pair (T >= 3 = kNG); with fewer tiles per query a group skips pairs, so
  // n <= 256 takes the job kernel.
  static const bool stream_ok = [] {
    const char* e = getenv("TID_VERIFY_STREAM");
    return !(e && e[0] == '0');
  }();
  const bool streamed = stream_ok && T >= kNG;
  if (!streamed) {
    TRY(idx->ws_nq.ensure(static_cast<size_t>(P) * T * kBM * 4, "query norms"));
    if (fold) TRY(idx->ws_qs.ensure(static_cast<size_t>(P) * n * kDim, "shifted queries"));
    launch_query_prep(dq, P, n, T, idx->ws_nq.as<int32_t>(), fold ? idx->ws_qs.as<uint8_t>() : nullptr, s);
    count_kernel(idx);
  }
  const bool dev_counts = is_device_ptr(counts_out);
  TRY(idx->ws_counts.ensure(static_cast<size_t>(P) * 4, "pair counts"));
  uint32_t* counts = dev_counts ? counts_out : idx->ws_counts.as<uint32_t>();
  CU(cudaMemsetAsync(counts, 0, static_cast<size_t>(P) * 4, s));
  int32_t* nn = nullptr;
  const bool dev_nn = nn_out && is_device_ptr(nn_out);
  if (nn_out) {
    if (dev_nn) {
      nn = nn_out;
    } else {
      TRY(idx->ws_nn.ensure(static_cast<size_t>(P) * n * 16, "nn output"));
      nn = idx->ws_nn.as<int32_t>();
    }
  }
  CUtensorMap qmap, rmap;
  TRY(make_map(&qmap, (fold && !streamed) ? idx->ws_qs.p : dq, P, n, kBM));
  TRY(make_map(&rmap, dr, P, m, kBN));
  MatchParams p{};
  p.mode = kModeVerify;
  p.m = m;  // stored rows per reference: the last chunk's all-padding pieces are skipped
  p.n_jobs = static_cast<int32_t>(P);
  p.refs_per_job = 1;
  p.cpr = cpr;
  p.tiles_per_q = T;
  p.num_q = static_cast<int32_t>(P);
  p.q_per_job = 1;
  p.n_qchunks = 1;
  p.n_refs = P;
  p.ref_map_base = 0;
  p.colkey = nullptr;  // computed in the kernel
  p.m_valid = dmr;
  p.nq = streamed ? nullptr : idx->ws_nq.as<int32_t>();
  p.n_valid = dnv;
  p.n_rows = n;
  p.counts = counts;
  p.ldc = 0;
  p.col0 = 0;
  p.nn_out = nn;
  p.num2 = idx->cfg.ratio_num * idx->cfg.ratio_num;
  p.den2 = idx->cfg.ratio_den * idx->cfg.ratio_den;
  int grid = idx->tune.grid > 0 ? idx->tune.grid : idx->num_sms;
  grid = static_cast<int>(std::min<int64_t>(grid, P));
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  if (idx->prof) {
    if (idx->prof_used == idx->prof_ev.size()) {
      cudaEvent_t a, b;
      CU(cudaEventCreate(&a));
      CU(cudaEventCreate(&b));
      idx->prof_ev.push_back({a, b});
    }
    e0 = idx->prof_ev[idx->prof_used].first;
    e1 = idx->prof_ev[idx->prof_used].second;
    ++idx->prof_used;
    CU(cudaEventRecord(e0, s));
  }
  if (fold) {
    // exact recompute of the rare +-1-undecided rows (the stream kernel reads the raw queries)
    p.qs = streamed ? dq : idx->ws_qs.as<uint8_t>();
    p.rdesc = dr;
    p.slot_banks = 1;
  }
  cudaError_t e = streamed ? launch_verify_stream(p, qmap, rmap, fold, grid, s) : launch_match(p, qmap, rmap, fold, grid, s);
  if (e != cudaSuccess) return fail(TID_ECUDA, "match kernel launch: %s", cudaGetErrorString(e));
  if (idx->prof) {
    CU(cudaEventRecord(e1, s));
    idx->stats.match_launches++;
    count_kernel(idx);
  }
  bool host_out = false;
  if (!dev_counts) TRY(copy_out(idx, counts_out, counts, static_cast<size_t>(P) * 4, s, &host_out));
  if (nn_out && !dev_nn) TRY(copy_out(idx, nn_out, nn, static_cast<size_t>(P) * n * 16, s, &host_out));
  if (host_out) CU(cudaStreamSynchronize(s));
  CU(cudaGetLastError());
  return TID_OK;
}

tid_status tid_verify_geometric(tid_index* idx, const uint8_t* q, int32_t n, const uint8_t* r, int32_t m, int64_t P,
                                const int32_t* n_q, const int32_t* m_r, const float* q_xy, const float* r_xy,
                                const tid_geom_params* gp, uint32_t* counts_out, uint32_t* good_out,
                                uint32_t* inliers_out, double* model_out, void* stream) {
  if (!idx) return fail(TID_EINVAL, "null index");
  if (!q_xy || !r_xy || !gp || !good_out || !inliers_out) return fail(TID_EINVAL, "null argument");
  if (!(gp->inlier_px > 0.0f) || !(gp->border >= 0.0f)) return fail(TID_EINVAL, "inlier_px must be > 0, border >= 0");
  if (gp->iterations < 0) return fail(TID_EINVAL, "iterations < 0");
  if (P < 1 || P > (1LL << 31) - 1 || n < 1 || m < 2) return fail(TID_EINVAL, "bad P / n / m");
  TRY(set_device(idx));
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  CallGuard guard(idx, s);
  // 1) one-to-one verification (a3-a5): exact (d1, i1, d2, i2) of every query row, into the workspace
  TRY(idx->ws_geo_nn.ensure(static_cast<size_t>(P) * n * 16, "geometric nn"));
  TRY(idx->ws_geo_cnt.ensure(static_cast<size_t>(P) * 4 * 4, "geometric counts"));
  uint32_t* dcnt = idx->ws_geo_cnt.as<uint32_t>();
  uint32_t* dgood = dcnt + P;
  uint32_t* dinl = dcnt + 2 * P;
  TRY(tid_verify(idx, q, n, r, m, P, n_q, m_r, dcnt, idx->ws_geo_nn.as<int32_t>(), s));
  // 2) coordinates and per-pair counts on the device
  const size_t qb = static_cast<size_t>(P) * n * 8, rb = static_cast<size_t>(P) * m * 8;
  TRY(idx->ws_geo_xy.ensure(qb + rb + static_cast<size_t>(P) * 8 + 64, "keypoint coordinates"));
  float* dq = idx->ws_geo_xy.as<float>();
  float* dr = reinterpret_cast<float*>(idx->ws_geo_xy.as<uint8_t>() + qb);
  TRY(copy_in(idx, dq, q_xy, qb, s));
  TRY(copy_in(idx, dr, r_xy, rb, s));
  const int32_t* dnq = nullptr;
  const int32_t* dmr = nullptr;
  int32_t* dvalid = reinterpret_cast<int32_t*>(idx->ws_geo_xy.as<uint8_t>() + qb + rb);
  if (n_q) {
    TRY(copy_in(idx, dvalid, n_q, static_cast<size_t>(P) * 4, s));
    dnq = dvalid;
  }
  if (m_r) {
    TRY(copy_in(idx, dvalid + P, m_r, static_cast<size_t>(P) * 4, s));
    dmr = dvalid + P;
  }
  // 3) edge-feature removal + RANSAC per pair (f4)
  GeomParams g{};
  g.border = gp->border;
  g.qw = gp->query_width;
  g.qh = gp->query_height;
  g.rw = gp->ref_width;
  g.rh = gp->ref_height;
  g.thr = gp->inlier_px;
  g.iters = gp->iterations;
  g.seed = gp->seed;
  g.num2 = idx->cfg.ratio_num * idx->cfg.ratio_num;
  g.den2 = idx->cfg.ratio_den * idx->cfg.ratio_den;
  double* dmodel = nullptr;
  const bool dev_model = model_out && is_device_ptr(model_out);
  if (model_out) {
    TRY(idx->ws_geo_out.ensure(static_cast<size_t>(P) * 32, "geometric models"));
    dmodel = dev_model ? model_out : idx->ws_geo_out.as<double>();
  }
  CU(launch_geometric(idx->ws_geo_nn.as<int32_t>(), n, m, P, dnq, dmr, dq, dr, g, dgood, dinl, dmodel, s));
  count_kernel(idx);
  bool host_out = false;
  if (counts_out) TRY(copy_out(idx, counts_out, dcnt, static_cast<size_t>(P) * 4, s, &host_out));
  TRY(copy_out(idx, good_out, dgood, static_cast<size_t>(P) * 4, s, &host_out));
  TRY(copy_out(idx, inliers_out, dinl, static_cast<size_t>(P) * 4, s, &host_out));
  if (model_out && !dev_model) TRY(copy_out(idx, model_out, dmodel, static_cast<size_t>(P) * 32, s, &host_out));
  if (host_out) CU(cudaStreamSynchronize(s));
  CU(cudaGetLastError());
  return TID_OK;
}

tid_status tid_merge_topk(tid_index* idx, const int64_t* ids_in, const int32_t* counts_in, int32_t G, int64_t B,
                          int32_t k, int64_t* ids_out, int32_t* counts_out, void* stream) {
  if (!idx || !ids_in || !counts_in || !ids_out || !counts_out) return fail(TID_EINVAL, "null argument");
  if (G < 1 || B < 1 || k < 1 || k > 64) return fail(TID_EINVAL, "bad G/B/k");
  TRY(set_device(idx));
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  CallGuard guard(idx, s);
  const int64_t tot = static_cast<int64_t>(G) * B * k;
  TRY(idx->ws_ids.ensure(static_cast<size_t>(tot) * 8, "merge ids"));
  TRY(idx->ws_cnts.ensure(static_cast<size_t>(tot) * 4, "merge counts"));
  TRY(idx->ws_gather.ensure(static_cast<size_t>(tot) * 8, "merge keys"));
  TRY(copy_in(idx, idx->ws_ids.p, ids_in, static_cast<size_t>(tot) * 8, s));
  TRY(copy_in(idx, idx->ws_cnts.p, counts_in, static_cast<size_t>(tot) * 4, s));
  launch_pack_lists(idx->ws_ids.as<int64_t>(), idx->ws_cnts.as<int32_t>(), tot, idx->ws_gather.as<uint64_t>(), s);
  TRY(idx->ws_keys.ensure(static_cast<size_t>(B) * k * 12, "merge out"));
  int64_t* dids = reinterpret_cast<int64_t*>(idx->ws_keys.p);
  int32_t* dcnt = reinterpret_cast<int32_t*>(idx->ws_keys.as<uint8_t>() + static_cast<size_t>(B) * k * 8);
  launch_merge(idx->ws_gather.as<uint64_t>(), G, B, k, k, B * k, nullptr, dids, dcnt, s);
  count_kernel(idx, 2);
  CU(cudaGetLastError());
  bool host_out = false;
  TRY(copy_out(idx, ids_out, dids, static_cast<size_t>(B) * k * 8, s, &host_out));
  TRY(copy_out(idx, counts_out, dcnt, static_cast<size_t>(B) * k * 4, s, &host_out));
  if (host_out) CU(cudaStreamSynchronize(s));
  return TID_OK;
}

// ---------------------------------------------------------------- f1: float-descriptor path
tid_status tid_f16_prepare(tid_index* idx, const uint8_t* sift, int64_t rows, int32_t rootsift, float scale,
                           uint16_t* out, void* stream) {
  if (!idx || !sift || !out) return fail(TID_EINVAL, "null argument");
  if (rows < 0) return fail(TID_EINVAL, "rows < 0");
  if (!(scale > 0.0f)) return fail(TID_EINVAL, "scale must be > 0");
  if (rows == 0) return TID_OK;
  TRY(set_device(idx));
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  CallGuard guard(idx, s);
  const size_t in_b = static_cast<size_t>(rows) * kDim, out_b = in_b * 2;
  const uint8_t* din = sift;
  // the kernel moves 16-byte words: unaligned device buffers are staged through the workspace too
  const bool aligned = reinterpret_cast<uintptr_t>(sift) % 16 == 0 && reinterpret_cast<uintptr_t>(out) % 16 == 0;
  if (!is_device_ptr(sift) || !aligned) {
    TRY(idx->ws_f16in.ensure(in_b, "f16 prepare input"));
    TRY(copy_in(idx, idx->ws_f16in.p, sift, in_b, s));
    din = idx->ws_f16in.as<uint8_t>();
  }
  const bool dev_out = is_device_ptr(out) && aligned;
  void* dout = out;
  if (!dev_out) {
    TRY(idx->ws_f16r.ensure(out_b, "f16 prepare output"));
    dout = idx->ws_f16r.p;
  }
  CU(launch_f16_prepare(din, rows, rootsift, scale, dout, s));
  count_kernel(idx);
  if (!dev_out) {
    bool host_out = false;
    TRY(copy_out(idx, out, dout, out_b, s, &host_out));
    CU(cudaStreamSynchronize(s));
  }
  return TID_OK;
}

tid_status tid_f16_search_counts(tid_index* idx, const uint16_t* q, int32_t n, int64_t B, const uint16_t* r,
                                 int32_t m, int64_t R, uint32_t* counts_out, void* stream) {
  if (!idx || !q || !r || !counts_out) return fail(TID_EINVAL, "null argument");
  if (n < 1 || n > idx->cfg.query_kp_max) return fail(TID_EINVAL, "n=%d outside 1..query_kp_max", n);
  if (m < 2 || m > 2 * kBN) return fail(TID_EINVAL, "m=%d outside 2..512 (float path)", m);
  if (B < 1 || R < 1) return fail(TID_EINVAL, "B and R must be >= 1");
  if (B > (1LL << 30) || R > (1LL << 31) - 1) return fail(TID_EINVAL, "B or R too large");
  TRY(set_device(idx));
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  CallGuard guard(idx, s);
  const int T = static_cast<int>(ceil_div(n, kBM));
  const size_t qb = static_cast<size_t>(B) * n * kDim * 2, rb = static_cast<size_t>(R) * m * kDim * 2;
  const uint16_t* dq = q;
  const uint16_t* dr = r;
  if (!is_device_ptr(q)) {
    TRY(idx->ws_f16q.ensure(qb, "f16 queries"));
    TRY(copy_in(idx, idx->ws_f16q.p, q, qb, s));
    dq = idx->ws_f16q.as<uint16_t>();
  }
  if (!is_device_ptr(r)) {
    TRY(idx->ws_f16r.ensure(rb, "f16 references"));
    TRY(copy_in(idx, idx->ws_f16r.p, r, rb, s));
    dr = idx->ws_f16r.as<uint16_t>();
  }
  TRY(idx->ws_f16nq.ensure(static_cast<size_t>(B) * T * kBM * 4, "f16 query norms"));
  // norm-term operand (R x 256 rows x 32 B) + the scalars max N_R (bits) and C
  const int fcpr = static_cast<int>(ceil_div(m, kBN));  // 256-row chunks per reference (1 or 2)
  const size_t xb = static_cast<size_t>(R) * kBN * fcpr * 32;
  TRY(idx->ws_f16nr.ensure(xb + 256 + static_cast<size_t>(R) * m * 4, "f16 reference norm terms"));
  uint8_t* xop = idx->ws_f16nr.as<uint8_t>();
  uint32_t* nrmax = reinterpret_cast<uint32_t*>(xop + xb);
  float* cterm = reinterpret_cast<float*>(xop + xb + 128);
  float* nr_rows = reinterpret_cast<float*>(xop + xb + 256);
  CU(launch_f16_norms(dq, B, n, T * kBM, 0.0f, idx->ws_f16nq.as<float>(), s));
  CU(launch_f16_xop(dr, R, m, nrmax, nr_rows, xop, cterm, s));
  count_kernel(idx, 2);
  const bool dev_counts = is_device_ptr(counts_out);
  TRY(idx->ws_counts.ensure(static_cast<size_t>(B) * R * 4, "count matrix"));
  uint32_t* counts = dev_counts ? counts_out : idx->ws_counts.as<uint32_t>();
  CU(cudaMemsetAsync(counts, 0, static_cast<size_t>(B) * R * 4, s));
  CUtensorMap qmap, rmap, xmap;
  TRY(make_map_f16(&qmap, dq, B, n, kBM));
  TRY(make_map_f16(&rmap, dr, R, m, kBN));
  TRY(make_xmap(&xmap, xop, R, static_cast<int64_t>(kBN) * fcpr));  // 32-B rows, SWIZZLE_32B
  CU(launch_f16_match(qmap, rmap, xmap, cterm, idx->ws_f16nq.as<float>(), static_cast<int32_t>(B), n, T, R,
                      idx->cfg.ratio_num * idx->cfg.ratio_num, idx->cfg.ratio_den * idx->cfg.ratio_den, counts,
                      idx->num_sms, s, 0, 0, 0, nullptr, fcpr, m));
  count_kernel(idx);
  if (!dev_counts) {
    bool host_out = false;
    TRY(copy_out(idx, counts_out, counts, static_cast<size_t>(B) * R * 4, s, &host_out));
    CU(cudaStreamSynchronize(s));
  }
  return TID_OK;
}

tid_status tid_get_info(const tid_index* idx, tid_info* out) {
  if (!idx || !out) return fail(TID_EINVAL, "null argument");
  out->num_references = idx->n_hbm + idx->n_host;
  out->hbm_references = idx->n_hbm;
  out->host_references = idx->n_host;
  out->hbm_bytes = idx->hbm_alloc;
  out->host_bytes = idx->host_alloc;
  out->num_sms = idx->num_sms;
  out->hbm_capacity_references = static_cast<int64_t>(idx->hbm_budget / idx->ref_bytes);
  out->host_capacity_references = static_cast<int64_t>(idx->host_budget / idx->ref_bytes);
  out->hbm_bytes_per_reference = idx->hbm_ref_bytes;
  out->world_size = idx->cfg.world_size;
  int nranks = 0;  // with a communicator: the rank count NCCL itself reports
  if (idx->comm && nccl().CommCount && nccl().CommCount(idx->comm, &nranks) == ncclSuccess) out->world_size = nranks;
  return TID_OK;
}

tid_status tid_profile(tid_index* idx, int32_t enable) {
  if (!idx) return fail(TID_EINVAL, "null index");
  idx->prof = enable != 0;
  idx->prof_used = 0;
  memset(&idx->stats, 0, sizeof(idx->stats));
  return TID_OK;
}

tid_status tid_get_stats(tid_index* idx, tid_stats* out) {
  if (!idx || !out) return fail(TID_EINVAL, "null argument");
  TRY(set_device(idx));
  double ms = 0;
  for (size_t i = 0; i < idx->prof_used; ++i) {
    CU(cudaEventSynchronize(idx->prof_ev[i].second));
    float t = 0;
    CU(cudaEventElapsedTime(&t, idx->prof_ev[i].first, idx->prof_ev[i].second));
    ms += t;
  }
  *out = idx->stats;
  out->match_ms = ms;
  return TID_OK;
}

tid_status tid_set_tuning(tid_index* idx, const tid_tuning* t) {
  if (!idx || !t) return fail(TID_EINVAL, "null argument");
  if (t->refs_per_job < 0 || t->refs_per_job > kMaxSlots) return fail(TID_EINVAL, "refs_per_job outside 0..4");
  if (t->grid < 0) return fail(TID_EINVAL, "grid < 0");
  if (t->host_chunk_refs < 0) return fail(TID_EINVAL, "host_chunk_refs < 0");
  if (t->window_refs < 0) return fail(TID_EINVAL, "window_refs < 0");
  idx->tune = *t;
  ++idx->gen;
  if (t->host_chunk_refs > 0) idx->host_chunk = t->host_chunk_refs;
  return TID_OK;
}

}  // extern "C"
