// abi.cu -- the extern "C" boundary of libgzkp.so (declared in include/gzkp.h).
//
// Argument checking, curve dispatch, prepared-point handles, host-buffer
// wrappers, and the multi-GPU path (one NCCL all-gather of per-rank XYZZ
// partials, §5.2).  No exception crosses this boundary.
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <atomic>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <set>
#include <string>
#include <thread>
#include <vector>

#include "internal.h"

namespace gzkp {

static thread_local std::string g_last_error;

Tunables& tunables() {
  static Tunables t;
  return t;
}

gzkp_status set_error(gzkp_status st, const std::string& msg) {
  g_last_error = msg;
  return st;
}

gzkp_status cuda_status(cudaError_t e, const char* where) {
  g_last_error = std::string(where) + ": " + cudaGetErrorString(e);
  return e == cudaErrorMemoryAllocation ? GZKP_ERROR_OUT_OF_MEMORY : GZKP_ERROR_CUDA;
}

int device_sm_count() {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return sms > 0 ? sms : 148;
}

static std::atomic<int> g_profiling{-1};
bool profiling_enabled() {
  int v = g_profiling.load(std::memory_order_relaxed);
  if (v < 0) {
    const char* e = getenv("GZKP_PROFILE");
    int expect = -1;
    g_profiling.compare_exchange_strong(expect, (e && atoi(e) != 0) ? 1 : 0);
    v = g_profiling.load(std::memory_order_relaxed);
  }
  return v == 1;
}

// pending records of this thread, harvested by gzkp_profile_read
static thread_local std::vector<ProfileRecord*> g_pending;
static thread_local double g_phase_sum[5] = {0, 0, 0, 0, 0};
static thread_local uint64_t g_calls = 0, g_last_launches = 0, g_last_entries = 0, g_last_c = 0;

ProfileRecord* profile_begin(cudaStream_t s) {
  if (!profiling_enabled()) return nullptr;
  // one pinned word per thread, allocated on first use (every record writes
  // the entry count of its call there; only the last call's value is read)
  static thread_local uint32_t* pinned = nullptr;
  if (!pinned && cudaMallocHost((void**)&pinned, sizeof(uint32_t)) != cudaSuccess) return nullptr;
  ProfileRecord* r = new ProfileRecord;
  r->entries_host = pinned;
  r->launches = 0;
  r->c = 0;
  (void)s;
  return r;
}
cudaEvent_t profile_event(ProfileRecord* r, cudaStream_t s) {
  if (!r) return nullptr;
  cudaEvent_t e;
  cudaEventCreate(&e);
  cudaEventRecord(e, s);
  return e;
}
void profile_interval(ProfileRecord* r, int phase, cudaEvent_t a, cudaEvent_t b) {
  if (r && a && b) r->iv.push_back({phase, a, b});
}
void profile_end(ProfileRecord* r, const uint32_t* entries_dev, int launches, int c, cudaStream_t s) {
  if (!r) return;
  cudaMemcpyAsync(r->entries_host, entries_dev, sizeof(uint32_t), cudaMemcpyDeviceToHost, s);
  r->launches = launches;
  r->c = c;
  g_pending.push_back(r);
}

const CurveImpl* impl_for(int curve) {
  switch (curve) {
    case GZKP_BN254: return impl_bn254();
    case GZKP_BLS12_381: return impl_bls12_381();
    case GZKP_MNT4_753: return impl_mnt4_753();
    case GZKP_TOY_A0: return impl_toy_a0();
    case GZKP_TOY_A2: return impl_toy_a2();
    case GZKP_BN254_G2: return impl_bn254_g2();
    case GZKP_BLS12_381_G2: return impl_bls12_381_g2();
    default: return nullptr;
  }
}

int current_device() {
  int dev = 0;
  cudaGetDevice(&dev);
  return dev;
}

gzkp_status once_per_device(const void* key, const std::function<gzkp_status()>& f) {
  static std::mutex mu;
  static std::set<std::pair<int, const void*>> done;
  const std::pair<int, const void*> k{current_device(), key};
  std::lock_guard<std::mutex> lock(mu);
  if (done.count(k)) return GZKP_SUCCESS;
  gzkp_status st = f();
  if (st == GZKP_SUCCESS) done.insert(k);
  return st;
}

static std::mutex g_pool_mu;
static std::map<int, cudaMemPool_t> g_pools;

static cudaMemPool_t device_pool(int dev) {
  std::lock_guard<std::mutex> lock(g_pool_mu);
  auto it = g_pools.find(dev);
  return it == g_pools.end() ? nullptr : it->second;
}

// per device: the library's private stream-ordered pool (freed workspace is
// kept for the next call without changing the application's default pool)
// and the call-stack limit of the out-of-line MNT4-753 paths (~2.6 KB per
// thread, ptxas "cumulative stack size"; the default limit is 1 KB)
void init_pool_once() {
  static int tag;
  once_per_device(&tag, [] {
    const int dev = current_device();
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaMemPool_t pool = nullptr;
    if (cudaMemPoolCreate(&pool, &props) == cudaSuccess) {
      uint64_t thr = UINT64_MAX;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
      std::lock_guard<std::mutex> lock(g_pool_mu);
      g_pools[dev] = pool;
    }
    cudaGetLastError();
    size_t stack = 0;
    cudaDeviceGetLimit(&stack, cudaLimitStackSize);
    if (stack < 4096) cudaDeviceSetLimit(cudaLimitStackSize, 4096);
    return GZKP_SUCCESS;
  });
}

cudaError_t pool_malloc(void** p, size_t bytes, cudaStream_t s) {
  cudaMemPool_t pool = device_pool(current_device());
  return pool ? cudaMallocFromPoolAsync(p, bytes, pool, s) : cudaMallocAsync(p, bytes, s);
}

bool debug_checks_enabled() {
  static const bool on = [] {
    const char* e = getenv("GZKP_DEBUG_CHECKS");
    return e && atoi(e) != 0;
  }();
  return on;
}

gzkp_status debug_validate(const CurveImpl* c, const void* pts, const void* sc, size_t n, cudaStream_t s) {
  if (!debug_checks_enabled() || !n) return GZKP_SUCCESS;
  uint32_t flags = 0;
  if (gzkp_status st = c->validate(pts, sc, n, &flags, s)) return st;
  if (!flags) return GZKP_SUCCESS;
  std::string m = "GZKP_DEBUG_CHECKS:";
  if (flags & 1) m += " a coordinate is >= p;";
  if (flags & 2) m += " a point is not on the curve;";
  if (flags & 4) m += " a scalar is >= 2^b;";
  return set_error(GZKP_ERROR_INVALID_VALUE, m);
}

static bool aligned16(const void* p) { return ((uintptr_t)p & 15u) == 0; }

// Per-stream library state, keyed by (device, stream handle, thread): calls
// on one stream are ordered, so they can share a workspace; different streams
// never do.  cudaStreamPerThread is one handle for many per-thread streams, so
// it is keyed by the calling thread as well.  gzkp_release_stream drops the
// entries of a stream before the application destroys it.
struct StreamKey {
  int dev;
  cudaStream_t s;
  size_t tid;
  bool operator<(const StreamKey& o) const {
    return dev != o.dev ? dev < o.dev : s != o.s ? s < o.s : tid < o.tid;
  }
};
static StreamKey stream_key(cudaStream_t s) {
  size_t tid = 0;
  if (s == cudaStreamPerThread) tid = std::hash<std::thread::id>{}(std::this_thread::get_id());
  return {current_device(), s, tid};
}
struct WsEntry { void* p; size_t bytes; };
static std::mutex g_ws_mu;
static std::map<StreamKey, WsEntry> g_ws;
static std::mutex g_ctx_mu;
static std::map<StreamKey, StreamCtx*> g_ctx;

gzkp_status stream_workspace(cudaStream_t s, size_t bytes, void** ptr) {
  std::lock_guard<std::mutex> lock(g_ws_mu);
  WsEntry& e = g_ws[stream_key(s)];
  if (e.bytes < bytes) {
    // stream-ordered: the old buffer is released after the work already queued on s
    if (e.p) cudaFreeAsync(e.p, s);
    e.p = nullptr;
    e.bytes = 0;
    const size_t want = bytes + bytes / 8;   // headroom against small n changes
    cudaError_t err = pool_malloc(&e.p, want, s);
    if (err != cudaSuccess) {
      e.p = nullptr;
      return cuda_status(err, "cudaMallocAsync(workspace)");
    }
    e.bytes = want;
  }
  *ptr = e.p;
  return GZKP_SUCCESS;
}

gzkp_status stream_ctx(cudaStream_t s, StreamCtx** out) {
  std::lock_guard<std::mutex> lock(g_ctx_mu);
  StreamCtx*& c = g_ctx[stream_key(s)];
  if (!c) {
    StreamCtx* n = new StreamCtx;
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);      // hi = greatest priority
    cudaError_t e = cudaStreamCreateWithPriority(&n->side, cudaStreamNonBlocking, hi);
    if (e == cudaSuccess) e = cudaStreamCreateWithPriority(&n->side2, cudaStreamNonBlocking, hi);
    if (e != cudaSuccess) { delete n; return cuda_status(e, "cudaStreamCreateWithPriority"); }
    n->nev = 64;
    for (int i = 0; i < n->nev; ++i) cudaEventCreateWithFlags(&n->ev[i], cudaEventDisableTiming);
    c = n;
  }
  *out = c;
  return GZKP_SUCCESS;
}

// frees the workspace (stream-ordered) and the side stream of (device, s)
static gzkp_status release_stream(cudaStream_t s) {
  const StreamKey k = stream_key(s);
  {
    std::lock_guard<std::mutex> lock(g_ws_mu);
    auto it = g_ws.find(k);
    if (it != g_ws.end()) {
      if (it->second.p) cudaFreeAsync(it->second.p, s);
      g_ws.erase(it);
    }
  }
  std::lock_guard<std::mutex> lock(g_ctx_mu);
  auto it = g_ctx.find(k);
  if (it != g_ctx.end()) {
    StreamCtx* c = it->second;
    cudaStreamSynchronize(c->side);
    cudaStreamSynchronize(c->side2);
    for (int i = 0; i < c->nev; ++i) cudaEventDestroy(c->ev[i]);
    cudaStreamDestroy(c->side);
    cudaStreamDestroy(c->side2);
    delete c;
    g_ctx.erase(it);
  }
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GZKP_SUCCESS : cuda_status(e, "gzkp_release_stream");
}

struct Prepared {
  int curve;
  size_t n;
  void* pts;          // Montgomery affine: n x 2N u32, or the copies x n checkpoint table
  bool weighted;      // NEXT-1 checkpoint table 2^(c M j) P_i (cross-window consolidation)
  int c, W;           // window bits; table copies (weighted) or 1
  size_t bytes;
  int interval;       // Algorithm 1 checkpoint interval M (weighted only)
};

// ------------------------------------------------------------- NCCL (dlopen)
// NCCL is resolved at run time so libgzkp.so loads without it; when torch has
// already loaded its libnccl.so.2 the same copy is reused (RTLD_NOLOAD first).
typedef struct ncclComm* ncclComm_t;
typedef struct { char internal[128]; } ncclUniqueId;
typedef int ncclResult_t;
enum { ncclUint8_ = 1 };

struct Nccl {
  void* h = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, int, ncclComm_t, cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  bool ok = false;
};

static Nccl& nccl() {
  static Nccl n;
  static std::once_flag once;
  std::call_once(once, [] {
    const char* names[] = {"libnccl.so.2", "libnccl.so"};
    for (const char* nm : names) {
      n.h = dlopen(nm, RTLD_NOW | RTLD_NOLOAD);
      if (n.h) break;
    }
    if (!n.h) {
      for (const char* nm : names) {
        n.h = dlopen(nm, RTLD_NOW | RTLD_GLOBAL);
        if (n.h) break;
      }
    }
    if (!n.h) return;
    n.GetUniqueId = (decltype(n.GetUniqueId))dlsym(n.h, "ncclGetUniqueId");
    n.CommInitRank = (decltype(n.CommInitRank))dlsym(n.h, "ncclCommInitRank");
    n.CommDestroy = (decltype(n.CommDestroy))dlsym(n.h, "ncclCommDestroy");
    n.AllGather = (decltype(n.AllGather))dlsym(n.h, "ncclAllGather");
    n.GetErrorString = (decltype(n.GetErrorString))dlsym(n.h, "ncclGetErrorString");
    n.ok = n.GetUniqueId && n.CommInitRank && n.CommDestroy && n.AllGather;
  });
  return n;
}

struct Comm {
  ncclComm_t comm = nullptr;
  int world = 1, rank = 0;
  void* partial = nullptr;    // 4N u32 (max N)
  void* gathered = nullptr;   // world x 4N u32
};

static gzkp_status nccl_status(ncclResult_t r, const char* where) {
  if (r == 0) return GZKP_SUCCESS;
  std::string m = std::string(where) + ": nccl error " + std::to_string(r);
  if (nccl().GetErrorString) m += std::string(" (") + nccl().GetErrorString(r) + ")";
  return set_error(GZKP_ERROR_NCCL, m);
}

}  // namespace gzkp

using namespace gzkp;

extern "C" {

size_t gzkp_field_bytes(int curve) {
  const CurveImpl* c = impl_for(curve);
  return c ? (size_t)c->limbs * 4 : 0;
}
size_t gzkp_scalar_bytes(int curve) {
  const CurveImpl* c = impl_for(curve);
  return c ? (size_t)c->scalar_limbs * 4 : 0;
}
size_t gzkp_partial_bytes(int curve) {
  const CurveImpl* c = impl_for(curve);
  return c ? (size_t)c->limbs * 16 : 0;
}

int gzkp_window_bits(int curve, size_t n) {
  const CurveImpl* c = impl_for(curve);
  return c ? c->window_bits(n) : -1;
}

size_t gzkp_msm_workspace_bytes(int curve, size_t n) {
  const CurveImpl* c = impl_for(curve);
  return c ? c->workspace_bytes(n, false) : 0;
}

static gzkp_status check_args(const CurveImpl* c, const void* pts, const void* sc, size_t n, const void* out) {
  if (!c) return set_error(GZKP_ERROR_UNSUPPORTED_CURVE, "unknown curve");
  if (!out) return set_error(GZKP_ERROR_INVALID_VALUE, "out is NULL");
  if (n && (!pts || !sc)) return set_error(GZKP_ERROR_INVALID_VALUE, "NULL input with n > 0");
  if (!aligned16(pts) || !aligned16(sc) || !aligned16(out))
    return set_error(GZKP_ERROR_INVALID_VALUE, "buffers must be 16-byte aligned");
  return GZKP_SUCCESS;
}

gzkp_status gzkp_msm_ex(int curve, const void* points_affine, const void* scalars, size_t n, void* out,
                        void* workspace, size_t workspace_bytes, gzkp_stream stream) {
  const CurveImpl* c = impl_for(curve);
  if (gzkp_status st = check_args(c, points_affine, scalars, n, out)) return st;
  init_pool_once();
  if (gzkp_status st = debug_validate(c, points_affine, scalars, n, (cudaStream_t)stream)) return st;
  MsmCall call;
  call.points = points_affine;
  call.scalars = scalars;
  call.n = n;
  call.out_affine = out;
  call.workspace = workspace;
  call.workspace_bytes = workspace_bytes;
  call.stream = (cudaStream_t)stream;
  return c->msm(call);
}

gzkp_status gzkp_msm(int curve, const void* points_affine, const void* scalars, size_t n, void* out,
                     gzkp_stream stream) {
  return gzkp_msm_ex(curve, points_affine, scalars, n, out, nullptr, 0, stream);
}

gzkp_status gzkp_msm_partial(int curve, const void* points_affine, const void* scalars, size_t n,
                             void* partial_xyzz, gzkp_stream stream) {
  const CurveImpl* c = impl_for(curve);
  if (gzkp_status st = check_args(c, points_affine, scalars, n, partial_xyzz)) return st;
  init_pool_once();
  if (gzkp_status st = debug_validate(c, points_affine, scalars, n, (cudaStream_t)stream)) return st;
  MsmCall call;
  call.points = points_affine;
  call.scalars = scalars;
  call.n = n;
  call.out_partial = partial_xyzz;
  call.stream = (cudaStream_t)stream;
  return c->msm(call);
}

gzkp_status gzkp_combine_partials(int curve, const void* partials_xyzz, int count, void* out_affine,
                                  gzkp_stream stream) {
  init_pool_once();
  const CurveImpl* c = impl_for(curve);
  if (!c) return set_error(GZKP_ERROR_UNSUPPORTED_CURVE, "unknown curve");
  if (count < 0 || !out_affine || (count && !partials_xyzz)) return set_error(GZKP_ERROR_INVALID_VALUE, "bad arguments");
  return c->combine(partials_xyzz, count, out_affine, (cudaStream_t)stream);
}

gzkp_status gzkp_msm_host(int curve, const void* points_host, const void* scalars_host, size_t n, void* out_host,
                          gzkp_stream stream) {
  const CurveImpl* c = impl_for(curve);
  if (!c) return set_error(GZKP_ERROR_UNSUPPORTED_CURVE, "unknown curve");
  if (!out_host || (n && (!points_host || !scalars_host))) return set_error(GZKP_ERROR_INVALID_VALUE, "NULL argument");
  init_pool_once();
  cudaStream_t s = (cudaStream_t)stream;
  const size_t pb = n * 2 * c->limbs * 4, sb = n * c->scalar_limbs * 4, ob = 2 * c->limbs * 4;
  // staging (canonical points as copied), Montgomery points, scalars, out
  char* d = nullptr;
  const size_t total = 2 * align_up(pb) + align_up(sb) + align_up(ob);
  cudaError_t e = pool_malloc((void**)&d, total, s);
  if (e != cudaSuccess) return cuda_status(e, "cudaMallocAsync");
  char *dstage = d, *dp = d + align_up(pb), *ds = d + 2 * align_up(pb), *dout = ds + align_up(sb);
  gzkp_status st = GZKP_SUCCESS;
  StreamCtx* ctx = nullptr;
  if ((st = stream_ctx(s, &ctx))) { cudaFreeAsync(d, s); return st; }
  cudaStream_t ss = ctx->side;
  cudaEvent_t ev_alloc = ctx->ev[ctx->nev - 3], ev_points = ctx->ev[ctx->nev - 2];
  // points on the side stream, in chunks, each converted to Montgomery form as
  // it lands; the scalars go first on the caller's stream so the digits and
  // the sort overlap the (larger) point transfer ("async copies")
  if ((e = cudaEventRecord(ev_alloc, s)) != cudaSuccess || (e = cudaStreamWaitEvent(ss, ev_alloc, 0)) != cudaSuccess)
    st = cuda_status(e, "event");
  const size_t chunk = std::max<size_t>(1, (64u << 20) / (2 * c->limbs * 4));
  for (size_t off = 0; !st && off < n; off += chunk) {
    const size_t cnt = std::min(chunk, n - off);
    const size_t boff = off * 2 * c->limbs * 4;
    if ((e = cudaMemcpyAsync(dstage + boff, (const char*)points_host + boff, cnt * 2 * c->limbs * 4,
                             cudaMemcpyHostToDevice, ss)) != cudaSuccess)
      st = cuda_status(e, "H2D points");
    if (!st) st = c->to_mont(dstage + boff, dp + boff, cnt, ss);
  }
  if (!st && (e = cudaEventRecord(ev_points, ss)) != cudaSuccess) st = cuda_status(e, "event");
  if (!st && n && (e = cudaMemcpyAsync(ds, scalars_host, sb, cudaMemcpyHostToDevice, s)) != cudaSuccess)
    st = cuda_status(e, "H2D scalars");
  if (!st && debug_checks_enabled() && n) {   // staged canonical copies (debug only: synchronises)
    if ((e = cudaStreamSynchronize(ss)) != cudaSuccess) st = cuda_status(e, "sync");
    if (!st) st = debug_validate(c, dstage, ds, n, s);
  }
  if (!st) {
    MsmCall call;
    call.points = dp;
    call.prepared = true;            // already Montgomery (converted per chunk above)
    call.scalars = ds;
    call.n = n;
    call.out_affine = dout;
    call.stream = s;
    call.points_ready = n ? ev_points : nullptr;
    st = c->msm(call);
  }
  if (!st && (e = cudaMemcpyAsync(out_host, dout, ob, cudaMemcpyDeviceToHost, s)) != cudaSuccess) st = cuda_status(e, "D2H out");
  cudaStreamWaitEvent(s, ev_points, 0);   // never free while the side stream may still copy
  cudaFreeAsync(d, s);
  if ((e = cudaStreamSynchronize(s)) != cudaSuccess && !st) st = cuda_status(e, "cudaStreamSynchronize");
  return st;
}

gzkp_status gzkp_points_prepare_ex(int curve, const void* points_affine, size_t n, int window_bits, int weighted,
                                   void** handle, gzkp_stream stream) {
  init_pool_once();
  const CurveImpl* c = impl_for(curve);
  if (!c) return set_error(GZKP_ERROR_UNSUPPORTED_CURVE, "unknown curve");
  if (!handle || (n && !points_affine) || !aligned16(points_affine) || window_bits < 0 || window_bits > 22)
    return set_error(GZKP_ERROR_INVALID_VALUE, "bad arguments");
  // the standard (per-window bucket sets) pipeline plans c <= 16, as gzkp_set_config
  if (weighted < 0) return set_error(GZKP_ERROR_INVALID_VALUE, "weighted (checkpoint interval) must be >= 0");
  if (weighted == 0 && (window_bits == 1 || window_bits > 18))
    return set_error(GZKP_ERROR_INVALID_VALUE, "window_bits must be 0 or 2..18 for unweighted points");
  if (weighted >= 1 && window_bits == 1) return set_error(GZKP_ERROR_INVALID_VALUE, "window_bits must be 0 or 2..22");
  if (gzkp_status st = debug_validate(c, points_affine, nullptr, n, (cudaStream_t)stream)) return st;
  Prepared* h = new (std::nothrow) Prepared{curve, n, nullptr, false, 0, 1, 0, 1};
  if (!h) return set_error(GZKP_ERROR_OUT_OF_MEMORY, "handle");
  const size_t pt_bytes = 2 * (size_t)c->limbs * 4;
  if (weighted >= 1 && n) {
    // checkpoint table 2^(c M j) P_i (Algorithm 1, interval M = weighted)
    h->interval = weighted;
    const int W = c->table_windows(n, window_bits, weighted);
    if ((uint64_t)n * W >= (1ull << 31)) { delete h; return set_error(GZKP_ERROR_INVALID_VALUE, "table >= 2^31 points"); }
    h->bytes = n * W * pt_bytes;
    cudaError_t e = cudaMalloc(&h->pts, h->bytes);
    if (e != cudaSuccess) { delete h; return cuda_status(e, "cudaMalloc(weighted table)"); }
    gzkp_status st = c->precompute(points_affine, n, window_bits, weighted, h->pts, &h->c, &h->W, (cudaStream_t)stream);
    if (st) { cudaFree(h->pts); delete h; return st; }
    h->weighted = true;
  } else if (n) {
    h->bytes = n * pt_bytes;
    cudaError_t e = cudaMalloc(&h->pts, h->bytes);
    if (e != cudaSuccess) { delete h; return cuda_status(e, "cudaMalloc(prepared)"); }
    gzkp_status st = c->to_mont(points_affine, h->pts, n, (cudaStream_t)stream);
    if (st) { cudaFree(h->pts); delete h; return st; }
    h->c = window_bits;
  }
  *handle = h;
  return GZKP_SUCCESS;
}

gzkp_status gzkp_points_prepare(int curve, const void* points_affine, size_t n, void** handle, gzkp_stream stream) {
  // default: the paper's weighted points when they fit, else plain Montgomery points
  gzkp_status st = gzkp_points_prepare_ex(curve, points_affine, n, 0, 1, handle, stream);
  if (st == GZKP_ERROR_OUT_OF_MEMORY || st == GZKP_ERROR_INVALID_VALUE) {
    cudaGetLastError();   // clear a failed allocation
    st = gzkp_points_prepare_ex(curve, points_affine, n, 0, 0, handle, stream);
  }
  return st;
}

gzkp_status gzkp_prepared_info(const void* handle, int* window_bits, int* windows, int* weighted, size_t* bytes) {
  const Prepared* h = (const Prepared*)handle;
  if (!h) return set_error(GZKP_ERROR_INVALID_VALUE, "NULL handle");
  if (window_bits) *window_bits = h->c;
  if (windows) *windows = h->W;
  if (weighted) *weighted = h->weighted ? h->interval : 0;
  if (bytes) *bytes = h->bytes;
  return GZKP_SUCCESS;
}

static gzkp_status msm_prepared_impl(const void* handle, const void* scalars, size_t n, void* out_affine,
                                     void* out_partial, gzkp_stream stream) {
  const Prepared* h = (const Prepared*)handle;
  if (!h) return set_error(GZKP_ERROR_INVALID_VALUE, "NULL handle");
  if (n > h->n) return set_error(GZKP_ERROR_INVALID_VALUE, "n exceeds prepared point count");
  const CurveImpl* c = impl_for(h->curve);
  if (gzkp_status st = check_args(c, h->pts, scalars, n, out_affine ? out_affine : out_partial)) return st;
  init_pool_once();
  if (gzkp_status st = debug_validate(c, nullptr, scalars, n, (cudaStream_t)stream)) return st;
  MsmCall call;
  call.points = h->pts;
  call.prepared = true;
  call.consolidated = h->weighted;
  call.interval = h->interval;
  call.window_bits = h->c;
  call.table_n = h->n;
  call.scalars = scalars;
  call.n = n;
  call.out_affine = out_affine;
  call.out_partial = out_partial;
  call.stream = (cudaStream_t)stream;
  return c->msm(call);
}

gzkp_status gzkp_msm_prepared(const void* handle, const void* scalars, size_t n, void* out, gzkp_stream stream) {
  return msm_prepared_impl(handle, scalars, n, out, nullptr, stream);
}

gzkp_status gzkp_msm_prepared_host(const void* handle, const void* scalars_host, size_t n, void* out_host,
                                   gzkp_stream stream) {
  const Prepared* h = (const Prepared*)handle;
  if (!h) return set_error(GZKP_ERROR_INVALID_VALUE, "NULL handle");
  const CurveImpl* c = impl_for(h->curve);
  if (!c || !out_host || (n && !scalars_host)) return set_error(GZKP_ERROR_INVALID_VALUE, "bad arguments");
  cudaStream_t s = (cudaStream_t)stream;
  const size_t sb = n * c->scalar_limbs * 4, ob = 2 * c->limbs * 4;
  char* d = nullptr;
  cudaError_t e = pool_malloc((void**)&d, align_up(sb) + align_up(ob), s);
  if (e != cudaSuccess) return cuda_status(e, "cudaMallocAsync");
  void *ds = d, *dout = d + align_up(sb);
  gzkp_status st = GZKP_SUCCESS;
  if (n && (e = cudaMemcpyAsync(ds, scalars_host, sb, cudaMemcpyHostToDevice, s)) != cudaSuccess) st = cuda_status(e, "H2D scalars");
  if (!st) st = gzkp_msm_prepared(handle, ds, n, dout, stream);
  if (!st && (e = cudaMemcpyAsync(out_host, dout, ob, cudaMemcpyDeviceToHost, s)) != cudaSuccess) st = cuda_status(e, "D2H out");
  cudaFreeAsync(d, s);
  if ((e = cudaStreamSynchronize(s)) != cudaSuccess && !st) st = cuda_status(e, "cudaStreamSynchronize");
  return st;
}

gzkp_status gzkp_points_release(void* handle) {
  Prepared* h = (Prepared*)handle;
  if (!h) return GZKP_SUCCESS;
  if (h->pts) cudaFree(h->pts);
  delete h;
  return GZKP_SUCCESS;
}

gzkp_status gzkp_fixed_base_mul(int curve, const void* scalars, size_t n, void* out_affine, gzkp_stream stream) {
  init_pool_once();
  const CurveImpl* c = impl_for(curve);
  if (gzkp_status st = check_args(c, out_affine, scalars, n, out_affine)) return st;
  return c->fixed_base(scalars, n, out_affine, (cudaStream_t)stream);
}

gzkp_status gzkp_field_op(int curve, int op, const void* a, const void* b, void* out, size_t n, gzkp_stream stream) {
  init_pool_once();
  const CurveImpl* c = impl_for(curve);
  if (!c) return set_error(GZKP_ERROR_UNSUPPORTED_CURVE, "unknown curve");
  if (op < 0 || op > 8 || (n && (!a || !b || !out))) return set_error(GZKP_ERROR_INVALID_VALUE, "bad arguments");
  return c->field_op(op, a, b, out, n, (cudaStream_t)stream);
}

gzkp_status gzkp_ec_op(int curve, int op, const void* P, const void* Q, void* out, size_t n, gzkp_stream stream) {
  init_pool_once();
  const CurveImpl* c = impl_for(curve);
  if (!c) return set_error(GZKP_ERROR_UNSUPPORTED_CURVE, "unknown curve");
  if (op < 0 || op > 3 || (n && (!P || !Q || !out))) return set_error(GZKP_ERROR_INVALID_VALUE, "bad arguments");
  return c->ec_op(op, P, Q, out, n, (cudaStream_t)stream);
}

gzkp_status gzkp_set_config(int window_bits, int chunk_entries) {
  if (window_bits < 0 || window_bits > 18 || window_bits == 1 || chunk_entries < 0 || chunk_entries > (1 << 20))
    return set_error(GZKP_ERROR_INVALID_VALUE, "window_bits must be 0 or 2..18");
  tunables().window_bits = window_bits;
  tunables().chunk_entries = chunk_entries;
  return GZKP_SUCCESS;
}

gzkp_status gzkp_set_profiling(int on) {
  g_profiling.store(on ? 1 : 0);
  return GZKP_SUCCESS;
}

gzkp_status gzkp_profile_read(double phase_ms[5], uint64_t stats[4], int reset) {
  for (ProfileRecord* r : g_pending) {
    std::vector<cudaEvent_t> seen;
    for (auto& iv : r->iv) {
      cudaEventSynchronize(iv.b);
      float ms = 0.f;
      cudaEventElapsedTime(&ms, iv.a, iv.b);
      if (iv.phase >= 0 && iv.phase < 5) g_phase_sum[iv.phase] += ms;
      seen.push_back(iv.a);
      seen.push_back(iv.b);
    }
    cudaDeviceSynchronize();   // the pinned entry count
    ++g_calls;
    g_last_launches = r->launches;
    g_last_entries = *r->entries_host;
    g_last_c = r->c;
    std::sort(seen.begin(), seen.end());
    seen.erase(std::unique(seen.begin(), seen.end()), seen.end());
    for (auto e : seen) cudaEventDestroy(e);
    delete r;
  }
  g_pending.clear();
  if (phase_ms)
    for (int i = 0; i < 5; ++i) phase_ms[i] = g_phase_sum[i];
  if (stats) {
    stats[0] = g_calls;
    stats[1] = g_last_launches;
    stats[2] = g_last_entries;
    stats[3] = g_last_c;
  }
  if (reset) {
    for (int i = 0; i < 5; ++i) g_phase_sum[i] = 0;
    g_calls = 0;
  }
  return GZKP_SUCCESS;
}

// ------------------------------------------------------------- multi-GPU
gzkp_status gzkp_nccl_unique_id(unsigned char id[128]) {
  Nccl& n = nccl();
  if (!n.ok) return set_error(GZKP_ERROR_NCCL, "libnccl.so.2 not found");
  ncclUniqueId u;
  if (gzkp_status st = nccl_status(n.GetUniqueId(&u), "ncclGetUniqueId")) return st;
  memcpy(id, u.internal, 128);
  return GZKP_SUCCESS;
}

gzkp_status gzkp_comm_init(int world, int rank, const unsigned char id[128], void** comm) {
  Nccl& n = nccl();
  if (!n.ok) return set_error(GZKP_ERROR_NCCL, "libnccl.so.2 not found");
  if (world < 1 || rank < 0 || rank >= world || !id || !comm) return set_error(GZKP_ERROR_INVALID_VALUE, "bad arguments");
  Comm* c = new (std::nothrow) Comm;
  if (!c) return set_error(GZKP_ERROR_OUT_OF_MEMORY, "comm");
  c->world = world;
  c->rank = rank;
  ncclUniqueId u;
  memcpy(u.internal, id, 128);
  if (gzkp_status st = nccl_status(n.CommInitRank(&c->comm, world, u, rank), "ncclCommInitRank")) { delete c; return st; }
  const size_t pmax = 24 * 16;   // largest XYZZ partial (MNT4-753)
  cudaError_t e;
  if ((e = cudaMalloc(&c->partial, pmax)) != cudaSuccess || (e = cudaMalloc(&c->gathered, pmax * world)) != cudaSuccess) {
    n.CommDestroy(c->comm);
    delete c;
    return cuda_status(e, "cudaMalloc(comm buffers)");
  }
  *comm = c;
  return GZKP_SUCCESS;
}

gzkp_status gzkp_comm_destroy(void* comm) {
  Comm* c = (Comm*)comm;
  if (!c) return GZKP_SUCCESS;
  if (c->comm && nccl().ok) nccl().CommDestroy(c->comm);
  cudaFree(c->partial);
  cudaFree(c->gathered);
  delete c;
  return GZKP_SUCCESS;
}

gzkp_status gzkp_msm_sharded(int curve, const void* points_affine, const void* scalars, size_t n_local, void* out,
                             gzkp_stream stream, void* comm) {
  Comm* cm = (Comm*)comm;
  const CurveImpl* c = impl_for(curve);
  if (!cm) return set_error(GZKP_ERROR_INVALID_VALUE, "NULL comm");
  if (gzkp_status st = check_args(c, points_affine, scalars, n_local, out)) return st;
  cudaStream_t s = (cudaStream_t)stream;
  // 1. full Pippenger on this rank's shard -> XYZZ partial
  if (gzkp_status st = gzkp_msm_partial(curve, points_affine, scalars, n_local, cm->partial, stream)) return st;
  // 2. the one collective: all-gather of the per-rank partials (rank order)
  const size_t pb = gzkp_partial_bytes(curve);
  if (gzkp_status st = nccl_status(nccl().AllGather(cm->partial, cm->gathered, pb, ncclUint8_, cm->comm, s), "ncclAllGather"))
    return st;
  // 3. fold in rank order + normalise; identical bytes on every rank
  return c->combine(cm->gathered, cm->world, out, s);
}

/* Sharded MSM on prepared points: each rank prepared ITS shard of the point
 * vector (gzkp_points_prepare on the local slice, e.g. with the weighted
 * table), so the per-rank Pippenger has no window combination; the partials
 * meet in the same single all-gather. */
gzkp_status gzkp_msm_prepared_sharded(const void* handle, const void* scalars, size_t n_local, void* out,
                                      gzkp_stream stream, void* comm) {
  Comm* cm = (Comm*)comm;
  const Prepared* h = (const Prepared*)handle;
  if (!cm || !h) return set_error(GZKP_ERROR_INVALID_VALUE, "NULL comm or handle");
  const CurveImpl* c = impl_for(h->curve);
  if (!c) return set_error(GZKP_ERROR_UNSUPPORTED_CURVE, "unknown curve");
  cudaStream_t s = (cudaStream_t)stream;
  if (gzkp_status st = msm_prepared_impl(handle, scalars, n_local, nullptr, cm->partial, stream)) return st;
  const size_t pb = gzkp_partial_bytes(h->curve);
  if (gzkp_status st = nccl_status(nccl().AllGather(cm->partial, cm->gathered, pb, ncclUint8_, cm->comm, s), "ncclAllGather"))
    return st;
  return c->combine(cm->gathered, cm->world, out, s);
}

gzkp_status gzkp_debug_buckets(int curve, const void* scalars, size_t n, int window_bits, uint32_t* offsets_host,
                               size_t offsets_cap, uint32_t* vals_host, size_t vals_cap, gzkp_stream stream) {
  const CurveImpl* c = impl_for(curve);
  if (!c) return set_error(GZKP_ERROR_UNSUPPORTED_CURVE, "unknown curve");
  if (window_bits < 2 || window_bits > 18 || !offsets_host || (n && (!scalars || !vals_host)) || !aligned16(scalars))
    return set_error(GZKP_ERROR_INVALID_VALUE, "bad arguments");
  init_pool_once();
  return c->debug_buckets(scalars, n, window_bits, offsets_host, offsets_cap, vals_host, vals_cap,
                          (cudaStream_t)stream);
}

gzkp_status gzkp_release_stream(gzkp_stream stream) { return release_stream((cudaStream_t)stream); }

const char* gzkp_status_string(gzkp_status status) {
  switch (status) {
    case GZKP_SUCCESS: return "success";
    case GZKP_ERROR_INVALID_VALUE: return "invalid value";
    case GZKP_ERROR_UNSUPPORTED_CURVE: return "unsupported curve";
    case GZKP_ERROR_OUT_OF_MEMORY: return "out of memory";
    case GZKP_ERROR_CUDA: return "CUDA error";
    case GZKP_ERROR_NCCL: return "NCCL error";
    default: return "unknown status";
  }
}

const char* gzkp_last_error(void) { return g_last_error.c_str(); }

}  // extern "C"
