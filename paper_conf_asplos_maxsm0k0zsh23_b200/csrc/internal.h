// internal.h -- interface between the C ABI (abi.cu) and the per-curve
// template instantiations (curve_*.cu).  Not part of the public ABI.
#pragma once
#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>
#include <functional>
#include <string>
#include <vector>

#include "../../include/gzkp.h"

namespace gzkp {

inline size_t align_up(size_t x, size_t a = 256) { return (x + a - 1) / a * a; }

struct Tunables {
  int window_bits = 0;     // 0 = cost model
  int chunk_entries = 0;   // 0 = default
};
Tunables& tunables();

// one MSM invocation (device pointers)
struct MsmCall {
  const void* points = nullptr;   // canonical affine, or Montgomery when prepared
  bool prepared = false;
  bool consolidated = false;      // points = checkpoint table [ceil(W/interval)][table_n] (NEXT-1)
  int interval = 1;               // Algorithm 1 checkpoint interval M (consolidated only)
  int window_bits = 0;            // forced c (0 = planner); set for consolidated tables
  size_t table_n = 0;
  cudaEvent_t points_ready = nullptr;   // if set: the accumulation waits for it (overlapped H2D)
  const void* scalars = nullptr;
  size_t n = 0;
  void* out_affine = nullptr;     // canonical affine result (may be null)
  void* out_partial = nullptr;    // XYZZ partial (may be null)
  void* workspace = nullptr;      // null = stream-ordered allocation inside
  size_t workspace_bytes = 0;
  cudaStream_t stream = nullptr;
};

struct CurveImpl {
  int id;
  int limbs;          // N
  int scalar_limbs;   // NS
  int scalar_bits;
  int (*window_bits)(size_t n);
  size_t (*workspace_bytes)(size_t n, bool prepared);
  gzkp_status (*msm)(const MsmCall& call);
  gzkp_status (*to_mont)(const void* in, void* out, size_t n, cudaStream_t s);
  gzkp_status (*combine)(const void* partials, int count, void* out, cudaStream_t s);
  gzkp_status (*fixed_base)(const void* scalars, size_t n, void* out, cudaStream_t s);
  gzkp_status (*field_op)(int op, const void* a, const void* b, void* out, size_t n, cudaStream_t s);
  gzkp_status (*ec_op)(int op, const void* P, const void* Q, void* out, size_t n, cudaStream_t s);
  // checkpoint table: copies j < ceil(W / interval) of 2^(c interval j) P_i
  gzkp_status (*precompute)(const void* in, size_t n, int c, int interval, void* table, int* c_out, int* w_out,
                            cudaStream_t s);
  int (*table_windows)(size_t n, int c, int interval);   // copies in the table
  // GZKP_DEBUG_CHECKS: points (canonical, may be null) / scalars (may be null)
  // -> flags (bit 0 coordinate >= p, 1 off curve, 2 scalar >= 2^b); synchronises
  gzkp_status (*validate)(const void* pts, const void* sc, size_t n, uint32_t* flags_host, cudaStream_t s);
  gzkp_status (*debug_buckets)(const void* sc, size_t n, int c, uint32_t* off_host, size_t off_cap,
                               uint32_t* vals_host, size_t vals_cap, cudaStream_t s);
};
// GZKP_DEBUG_CHECKS=1 in the environment (read once)
bool debug_checks_enabled();
// validates when debug checks are on: GZKP_ERROR_INVALID_VALUE on bad inputs
gzkp_status debug_validate(const CurveImpl* c, const void* pts, const void* sc, size_t n, cudaStream_t s);

const CurveImpl* impl_bn254();
const CurveImpl* impl_bls12_381();
const CurveImpl* impl_mnt4_753();
const CurveImpl* impl_toy_a0();
const CurveImpl* impl_toy_a2();
const CurveImpl* impl_bn254_g2();
const CurveImpl* impl_bls12_381_g2();
const CurveImpl* impl_for(int curve);

gzkp_status set_error(gzkp_status st, const std::string& msg);
gzkp_status cuda_status(cudaError_t e, const char* where);
int device_sm_count();
bool profiling_enabled();
// library-owned workspace, one grow-only buffer per (device, stream): calls on
// one stream are ordered, so they can share it; different streams never do.
gzkp_status stream_workspace(cudaStream_t s, size_t bytes, void** ptr);
// profiling hooks (no synchronisation).  A record is a list of timed
// intervals, each (phase, start event, end event) on any stream; phases:
// 0 sort, 1 accumulate, 2 merge, 3 reduce, 4 tail.  entries_dev = device
// address of the call's entry count (copied async into pinned memory).
struct ProfileRecord {
  struct Iv { int phase; cudaEvent_t a, b; };
  std::vector<Iv> iv;
  uint32_t* entries_host;
  int launches;
  int c;
};
ProfileRecord* profile_begin(cudaStream_t s);          // null when profiling is off
cudaEvent_t profile_event(ProfileRecord* r, cudaStream_t s);   // records a fresh event (null if off)
void profile_interval(ProfileRecord* r, int phase, cudaEvent_t a, cudaEvent_t b);
void profile_end(ProfileRecord* r, const uint32_t* entries_dev, int launches, int c, cudaStream_t s);

// per (device, caller stream): a high-priority side stream and reusable
// sync events for the window-group pipeline
struct StreamCtx {
  cudaStream_t side = nullptr;    // merge + bucket reduction of the window groups
  cudaStream_t side2 = nullptr;   // window combination (Horner), group after group
  cudaEvent_t ev[64];
  int nev = 0;
};
gzkp_status stream_ctx(cudaStream_t s, StreamCtx** ctx);
// once per DEVICE (every entry point calls it for the current device): the
// library's private stream-ordered memory pool (release threshold = max, so
// freed workspace is kept; the device's default pool is left untouched) and a
// 4 KB per-thread stack for the out-of-line MNT4-753 products.
void init_pool_once();
// Runs f() once per (key, current device), under a process-wide lock;
// per-device state (kernel attributes, limits) must never hide behind a
// process-wide flag.  A failing f() is retried by the next call.
gzkp_status once_per_device(const void* key, const std::function<gzkp_status()>& f);
int current_device();
// stream-ordered allocation from the library's private pool of the current device
cudaError_t pool_malloc(void** p, size_t bytes, cudaStream_t s);

}  // namespace gzkp
