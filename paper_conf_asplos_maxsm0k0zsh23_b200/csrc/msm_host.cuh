// msm_host.cuh -- host orchestration of the MSM pipeline for one curve.
//
// Planner (window size c, chunk size), workspace layout, and the stream-
// ordered launch sequence.  Everything is enqueued on the caller's stream; no
// host synchronisation happens inside gzkp_msm (the merge depth is sized from
// the worst case so no device->host read of the entry count is needed).
#pragma once
#include <cmath>
#include <cstdlib>
#include <vector>

#include "internal.h"
#include "msm_kernels.cuh"

namespace gzkp {

#define GZ_CHECK(expr)                                              \
  do {                                                              \
    cudaError_t _e = (expr);                                        \
    if (_e != cudaSuccess) return cuda_status(_e, #expr);           \
  } while (0)

struct Plan {
  int c = 0, W = 0;
  uint32_t B = 0;        // buckets per window = 2^(c-1)
  int S = 64;            // entries per level-0 chunk
  int S2 = 32;           // slots per merge chunk
  int seg = 16;          // buckets per reduction segment
  int levels = 0;        // merge levels
  size_t n = 0;
  uint64_t E_max = 0;
  uint64_t slots_max = 0;
  // workspace byte offsets
  size_t o_pts = 0, o_counts = 0, o_offsets = 0, o_cursor = 0, o_tiles = 0, o_keys = 0, o_vals = 0,
         o_info = 0, o_slot_k[2] = {0, 0}, o_slot_p[2] = {0, 0}, o_buckets = 0, o_seg = 0, o_win = 0,
         o_partial = 0, total = 0;
};

template <class C>
struct Impl {
  static constexpr int N = C::N;
  static constexpr int NS = C::NS;

  // ---- window size: App. B cost model of SURVEY.md ("profiling-
  // based window configuration"; reading R8).  Units: Montgomery muls.
  static int window_bits(size_t n) {
    if (tunables().window_bits > 0) return tunables().window_bits;
    if (const char* e = getenv("GZKP_WINDOW_BITS")) {
      int v = atoi(e);
      if (v >= 2 && v <= 16) return v;
    }
    const double madd = 10.0, add = 14.0, dbl = 10.0;
    const double lat = 6000.0;   // a serial op on one thread vs the whole chip's throughput
    int best = 8;
    double best_cost = 1e300;
    const int cmax = C::SCALAR_BITS < 16 ? 4 : 16;
    for (int c = 2; c <= cmax; ++c) {
      const int W = (C::SCALAR_BITS + 1 + c - 1) / c;
      const double B = std::ldexp(1.0, c - 1);
      const double entries = (double)n * W * (1.0 - std::ldexp(1.0, -c));
      const double reduce = W * B * 3.4 * add + 60.0 * add * lat / 8.0;
      const double tail = (W - 1) * (c * dbl + add) * lat;
      const double cost = entries * madd + reduce + tail;
      if (cost < best_cost) { best_cost = cost; best = c; }
    }
    return best;
  }

  static Plan plan(size_t n, bool prepared) {
    Plan p;
    p.n = n;
    p.c = window_bits(n);
    p.W = (C::SCALAR_BITS + 1 + p.c - 1) / p.c;
    p.B = 1u << (p.c - 1);
    int S = tunables().chunk_entries;
    if (S <= 0) {
      if (const char* e = getenv("GZKP_SEGMENT")) S = atoi(e);
    }
    if (S <= 0) S = 64;
    p.S = S;
    p.seg = (int)std::min<uint32_t>(16u, p.B);
    p.E_max = (uint64_t)n * p.W;
    const uint64_t chunks_max = (p.E_max + p.S - 1) / p.S;
    p.slots_max = 2 * chunks_max;
    uint64_t slots = p.slots_max;
    p.levels = 0;
    while (true) {
      ++p.levels;                       // this level consumes `slots`
      if (slots <= (uint64_t)p.S2) break;
      slots = 2 * ((slots + p.S2 - 1) / p.S2);
    }
    const uint64_t M = (uint64_t)p.W * p.B;
    const uint32_t G = p.B / p.seg;
    size_t o = 0;
    auto take = [&](size_t bytes) { size_t r = o; o = align_up(o + bytes); return r; };
    p.o_pts = prepared ? 0 : take(n * 2 * N * 4);
    p.o_counts = take(M * 4);
    p.o_offsets = take((M + 1) * 4);
    p.o_cursor = take(M * 4);
    p.o_tiles = take(SCAN_TILE * 4);
    p.o_keys = take(std::max<uint64_t>(p.E_max, 1) * 4);
    p.o_vals = take(std::max<uint64_t>(p.E_max, 1) * 4);
    p.o_info = take(sizeof(LevelInfo));
    for (int b = 0; b < 2; ++b) {
      p.o_slot_k[b] = take(std::max<uint64_t>(p.slots_max, 2) * 4);
      p.o_slot_p[b] = take(std::max<uint64_t>(p.slots_max, 2) * 4 * N * 4);
    }
    p.o_buckets = take(M * 4 * N * 4);
    p.o_seg = take((size_t)p.W * G * 4 * N * 4);
    p.o_win = take((size_t)p.W * 4 * N * 4);
    p.o_partial = take(4 * N * 4);
    p.total = o;
    return p;
  }

  static size_t workspace_bytes(size_t n, bool prepared) { return plan(n, prepared).total; }

  static int occupancy_grid(const void* fn, int threads, size_t smem) {
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, threads, smem);
    if (per_sm < 1) per_sm = 1;
    return per_sm * device_sm_count();
  }

  static gzkp_status to_mont(const void* in, void* out, size_t n, cudaStream_t s) {
    if (!n) return GZKP_SUCCESS;
    const int threads = 256;
    const int grid = (int)std::min<size_t>((n + threads - 1) / threads, (size_t)device_sm_count() * 16);
    k_to_mont<C><<<grid, threads, 0, s>>>((const uint32_t*)in, (uint32_t*)out, n);
    GZ_CHECK(cudaGetLastError());
    return GZKP_SUCCESS;
  }

  static gzkp_status msm(const MsmCall& call) {
    const size_t n = call.n;
    cudaStream_t s = call.stream;
    if (n == 0) {
      if (call.out_affine) GZ_CHECK(cudaMemsetAsync(call.out_affine, 0, 2 * N * 4, s));
      if (call.out_partial) {
        // XYZZ identity: ZZ = ZZZ = 0 (X, Y irrelevant)
        GZ_CHECK(cudaMemsetAsync(call.out_partial, 0, 4 * N * 4, s));
      }
      return GZKP_SUCCESS;
    }
    if ((uint64_t)n >= (1ull << 31)) return set_error(GZKP_ERROR_INVALID_VALUE, "n >= 2^31 not supported");
    const Plan p = plan(n, call.prepared);
    if (p.E_max >= (1ull << 32) - 1) return set_error(GZKP_ERROR_INVALID_VALUE, "n * windows >= 2^32");

    char* ws = (char*)call.workspace;
    bool own = false;
    if (!ws) {
      GZ_CHECK(cudaMallocAsync((void**)&ws, p.total, s));
      own = true;
    } else if (call.workspace_bytes < p.total) {
      return set_error(GZKP_ERROR_INVALID_VALUE, "workspace too small");
    }
    gzkp_status st = run(call, p, ws);
    if (own) {
      cudaError_t e = cudaFreeAsync(ws, s);
      if (st == GZKP_SUCCESS && e != cudaSuccess) st = cuda_status(e, "cudaFreeAsync");
    }
    return st;
  }

  static gzkp_status run(const MsmCall& call, const Plan& p, char* ws) {
    cudaStream_t s = call.stream;
    const size_t n = call.n;
    const uint64_t M = (uint64_t)p.W * p.B;
    auto U = [&](size_t off) { return (uint32_t*)(ws + off); };
    ProfileRecord* prof = profile_begin(s);
    int launches = 0;

    // a1: points -> Montgomery (skipped for prepared handles)
    const uint32_t* pts = (const uint32_t*)call.points;
    if (!call.prepared) {
      gzkp_status st = to_mont(call.points, U(p.o_pts), n, s);
      if (st) return st;
      pts = U(p.o_pts);
      ++launches;
    }
    // a2: histogram
    const int hist_threads = 512;
    const size_t hist_smem = (size_t)p.B * 4;
    GZ_CHECK(cudaFuncSetAttribute(k_hist<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)hist_smem));
    GZ_CHECK(cudaFuncSetAttribute(k_scatter<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)hist_smem));
    int nb = std::max(1, (2 * device_sm_count() + p.W - 1) / p.W);
    nb = (int)std::min<size_t>(nb, (n + 1023) / 1024);
    nb = std::max(nb, 1);
    dim3 hgrid(nb, p.W);
    GZ_CHECK(cudaMemsetAsync(U(p.o_counts), 0, M * 4, s));
    k_hist<C><<<hgrid, hist_threads, hist_smem, s>>>((const uint32_t*)call.scalars, n, p.c, p.B, U(p.o_counts));
    GZ_CHECK(cudaGetLastError());
    launches += 1 + 3 + 1 + 1;   // hist, scan x3, plan, scatter
    // scan -> offsets (+ cursor copy), offsets[M] = E
    const uint32_t ntiles = (uint32_t)((M + SCAN_TILE - 1) / SCAN_TILE);
    k_scan_tiles<<<ntiles, SCAN_THREADS, 0, s>>>(U(p.o_counts), U(p.o_offsets), (uint32_t)M, U(p.o_tiles));
    k_scan_top<<<1, SCAN_THREADS, 0, s>>>(U(p.o_tiles), ntiles, U(p.o_offsets) + M);
    k_scan_add<<<ntiles, SCAN_THREADS, 0, s>>>(U(p.o_offsets), U(p.o_cursor), (uint32_t)M, U(p.o_tiles));
    k_plan<<<1, 1, 0, s>>>(U(p.o_offsets), (uint32_t)M, p.S, p.S2, p.levels, (LevelInfo*)U(p.o_info));
    // a3: scatter
    k_scatter<C><<<hgrid, hist_threads, hist_smem, s>>>((const uint32_t*)call.scalars, n, p.c, p.B, U(p.o_cursor),
                                                         U(p.o_keys), U(p.o_vals));
    GZ_CHECK(cudaGetLastError());
    profile_mark(prof, 1, s);

    // a4: accumulation
    {
      const int threads = 128;
      const size_t smem = (size_t)threads * Stage<C>::SLOT_WORDS * 4;
      static int grid = 0;
      if (!grid) {
        cudaFuncSetAttribute(k_accum<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        grid = occupancy_grid((const void*)k_accum<C>, threads, smem);
      }
      const uint64_t chunks_max = (p.E_max + p.S - 1) / p.S;
      const int g = (int)std::min<uint64_t>(grid, (chunks_max + threads - 1) / threads);
      k_accum<C><<<std::max(g, 1), threads, smem, s>>>(U(p.o_keys), U(p.o_vals), pts, (const LevelInfo*)U(p.o_info),
                                                       p.S, U(p.o_buckets), U(p.o_slot_k[1]), U(p.o_slot_p[1]));
      GZ_CHECK(cudaGetLastError());
      ++launches;
    }
    profile_mark(prof, 2, s);
    // a5: merge levels (ping-pong slot buffers)
    {
      const int threads = 128;
      static int grid = 0;
      if (!grid) grid = occupancy_grid((const void*)k_merge<C>, threads, 0);
      uint64_t slots = p.slots_max;
      for (int l = 1; l <= p.levels; ++l) {
        const int in = l & 1, out = in ^ 1;
        const uint64_t chunks = (slots + p.S2 - 1) / p.S2;
        const int g = (int)std::min<uint64_t>(grid, (chunks + threads - 1) / threads);
        k_merge<C><<<std::max(g, 1), threads, 0, s>>>(U(p.o_slot_k[in]), U(p.o_slot_p[in]), (const LevelInfo*)U(p.o_info),
                                                      l, p.S2, U(p.o_buckets), U(p.o_slot_k[out]), U(p.o_slot_p[out]));
        GZ_CHECK(cudaGetLastError());
        ++launches;
        slots = 2 * chunks;
      }
    }
    profile_mark(prof, 3, s);
    // a6: bucket reduction
    const uint32_t G = p.B / p.seg;
    {
      const int threads = 128;
      const uint32_t total = (uint32_t)p.W * G;
      k_reduce_seg<C><<<(total + threads - 1) / threads, threads, 0, s>>>(U(p.o_buckets), U(p.o_offsets), p.W, p.B,
                                                                          p.seg, U(p.o_seg));
      GZ_CHECK(cudaGetLastError());
      const int rthreads = 128;
      const size_t smem = (size_t)rthreads * 4 * N * 4;
      GZ_CHECK(cudaFuncSetAttribute(k_reduce_win<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      k_reduce_win<C><<<p.W, rthreads, smem, s>>>(U(p.o_seg), G, U(p.o_win));
      GZ_CHECK(cudaGetLastError());
      launches += 2;
    }
    profile_mark(prof, 4, s);
    // a7 + a8
    k_tail<C><<<1, 1, 0, s>>>(U(p.o_win), p.W, p.c, (uint32_t*)call.out_partial, (uint32_t*)call.out_affine);
    GZ_CHECK(cudaGetLastError());
    ++launches;
    profile_end(prof, U(p.o_info), launches, p.c, s);   // LevelInfo::E is its first field
    return GZKP_SUCCESS;
  }

  static gzkp_status combine(const void* partials, int count, void* out, cudaStream_t s) {
    k_combine<C><<<1, 1, 0, s>>>((const uint32_t*)partials, count, (uint32_t*)out);
    GZ_CHECK(cudaGetLastError());
    return GZKP_SUCCESS;
  }

  static gzkp_status fixed_base(const void* sc, size_t n, void* out, cudaStream_t s) {
    if (!n) return GZKP_SUCCESS;
    const int threads = 128;
    const int grid = (int)std::min<size_t>((n + threads - 1) / threads, (size_t)device_sm_count() * 64);
    k_fixed_base<C><<<grid, threads, 0, s>>>((const uint32_t*)sc, n, (uint32_t*)out);
    GZ_CHECK(cudaGetLastError());
    return GZKP_SUCCESS;
  }

  static gzkp_status field_op(int op, const void* a, const void* b, void* out, size_t n, cudaStream_t s) {
    if (!n) return GZKP_SUCCESS;
    const int threads = 128;
    const int grid = (int)std::min<size_t>((n + threads - 1) / threads, 4096);
    k_field_op<C><<<grid, threads, 0, s>>>(op, (const uint32_t*)a, (const uint32_t*)b, (uint32_t*)out, n);
    GZ_CHECK(cudaGetLastError());
    return GZKP_SUCCESS;
  }

  static gzkp_status ec_op(int op, const void* P, const void* Q, void* out, size_t n, cudaStream_t s) {
    if (!n) return GZKP_SUCCESS;
    const int threads = 128;
    const int grid = (int)std::min<size_t>((n + threads - 1) / threads, 4096);
    k_ec_op<C><<<grid, threads, 0, s>>>(op, (const uint32_t*)P, (const uint32_t*)Q, (uint32_t*)out, n);
    GZ_CHECK(cudaGetLastError());
    return GZKP_SUCCESS;
  }

  static const CurveImpl* get() {
    static const CurveImpl impl = {C::ID, C::N, C::NS, C::SCALAR_BITS,
                                   &Impl::window_bits, &Impl::workspace_bytes, &Impl::msm, &Impl::to_mont,
                                   &Impl::combine, &Impl::fixed_base, &Impl::field_op, &Impl::ec_op};
    return &impl;
  }
};

}  // namespace gzkp
