// msm_host.cuh -- host orchestration of the MSM pipeline for one curve.
//
// Planner (window size c, chunk size), workspace layout, and the stream-
// ordered launch sequence.  Everything is enqueued on the caller's stream; no
// host synchronisation happens inside gzkp_msm: every data-dependent size
// (entry count, heavy buckets) is read by the kernels from device memory and
// the grids are sized for the worst case.
#pragma once
#include <cmath>
#include <cstdlib>
#include <map>
#include <mutex>
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
  bool consolidated = false;   // NEXT-1: windows share bucket sets (weighted points, Algorithm 1)
  int Mi = 0;            // bucket set of window t = t mod Mi: W (standard) or the checkpoint interval M
  int Wb = 0;            // bucket windows (sets): Mi
  uint32_t val_stride = 0;     // table stride of the weighted points (consolidated)
  uint32_t M = 0;        // Wb * B bucket keys
  int S = 64;            // entries per accumulation chunk
  // batch-affine levels (affine.cuh): level arrays A (odd levels) / B (even),
  // their offsets, the thread-distribution offsets, per-thread prefix scratch
  int aff_levels = 0;
  uint32_t aff_ctas = 0;
  size_t o_aoff = 0, o_aoffA = 0, o_aoffB = 0, o_lvlA = 0, o_lvlB = 0, o_ascr = 0;
  int seg = 16;          // buckets per reduction segment
  int heavy_levels = 0;  // depth of the heavy-bucket tree (max over groups)
  size_t n = 0;
  uint64_t E_max = 0, chunks_max = 0;
  // workspace byte offsets
  size_t o_scc = 0, o_idx = 0, o_ncnt = 0;   // zero-scalar compaction (non-prepared calls)
  size_t o_ones = 0, o_opart = 0, o_oping = 0;  // the scalar-1 points (k_ones_sum) and their run sums
  uint32_t ones_runs = 0;
  size_t o_pts = 0, o_codes = 0, o_counts = 0, o_offsets = 0, o_cursor = 0, o_tiles = 0, o_vals = 0,
         o_spay = 0, o_heavy = 0, o_hlist = 0, o_hjobs = 0, o_state = 0, o_buckets = 0, o_seg = 0, o_mid = 0, o_terms = 0, o_hot = 0, o_cb = 0, o_mcnt = 0, o_win = 0, total = 0;
  size_t seg_stride = 0;  // points between segT and segR in o_seg
  struct Grp {
    int t_lo, t_hi;             // windows (inclusive)
    uint32_t key_lo, key_hi;    // bucket keys
    uint64_t chunk_base, chunks_max;
    int heavy_levels;
    uint32_t hmax, hbase;       // heavy-list capacity and first entry
    int seg = 16;               // reduction segment (buckets per thread)
    // reduction sub-groups, top windows first: the Horner tail of sub-group k
    // (side stream 2) overlaps the reduction of sub-group k+1 (GZKP_REDUCE_GROUPS)
    struct Sub { int t_lo, t_hi, seg; };
    std::vector<Sub> subs;
  };
  std::vector<Grp> groups;
  bool split_reduce = false;    // more than one reduction sub-group somewhere: side streams needed
};

inline int ilog2_u64(uint64_t v) { int r = 0; while (v > 1) { v >>= 1; ++r; } return r; }

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
      if (v >= 2 && v <= 18) return v;
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
      // bucket reduction: 2 adds per bucket (k_reduce_seg) + the bit-set sums'
      // latency (round-1 measurement: 1.17 ms for 16 x 2^15 buckets)
      const double reduce = W * B * 2.0 * add + 30.0 * add * lat / 8.0;
      const double tail = (W - 1) * (c * dbl + add) * lat;
      const double cost = entries * madd + reduce + tail + top_window_merge(n, c, W) * add * lat;
      if (cost < best_cost) { best_cost = cost; best = c; }
    }
    // Measured override for the ~255-bit scalar fields at n >= 2^24 (round 2,
    // BLS12-381 2^26: uniform at c = 16 / 17 / 18 = 423.7 / 408.5 / 399.1 ms,
    // the sparse witness 42.77 / 42.75 / 44.61 ms; 2^22 uniform 28.7 / 29.8 /
    // 30.4 ms): c = 17 leaves the top window one bit wide, so ~15.5 windows
    // carry entries instead of 16, which the model's n W entries miss; 18 is
    // faster still on uniform scalars but slower on the sparse witness.
    if (C::SCALAR_BITS >= 250 && C::SCALAR_BITS <= 256 && n >= (1ull << 24) && best == 16) best = 17;
    return best;
  }

  // Serial adds the merge of the top window costs: it holds only the
  // b + 1 - c (W - 1) leftover scalar bits, so its few buckets are heavy
  // (2^19 points at c = 14: 8 buckets of 2^16 entries, a 2-level heavy tree,
  // 0.4 ms measured) -- the k_heavy_tree depth, 15 serial adds per level.
  static double top_window_merge(size_t n, int c, int W) {
    const int top_bits = C::SCALAR_BITS + 1 - c * (W - 1);
    const double per_bucket = (double)n / std::ldexp(1.0, std::max(top_bits - 1, 0));
    const double q = per_bucket / 64.0;               // partials of one top bucket (S = 64)
    if (q <= 1.0) return 0.0;
    if (q <= MERGE_QMAX) return q - 1.0;
    return 15.0 * std::ceil(std::log(q) / std::log((double)HEAVY_SPAN));
  }

  // Window size when the windows share M bucket sets (weighted points,
  // checkpoint interval M): M reductions of 2^(c-1) buckets and (M-1) c
  // doublings instead of W and (W-1) c, so a larger c pays.
  static int window_bits_consolidated(size_t n, int interval = 1) {
    if (const char* e = getenv("GZKP_WINDOW_BITS_PREPARED")) {
      int v = atoi(e);
      if (v >= 2 && v <= 22) return v;
    }
    const double madd = 10.0, add = 14.0, lat = 6000.0;
    int best = 8;
    double best_cost = 1e300;
    const int cmax = C::SCALAR_BITS < 16 ? 4 : 22;
    for (int c = 2; c <= cmax; ++c) {
      const int W = (C::SCALAR_BITS + 1 + c - 1) / c;
      const double B = std::ldexp(1.0, c - 1);
      const double entries = (double)n * W * (1.0 - std::ldexp(1.0, -c));
      const int Mi = std::min(std::max(interval, 1), W);
      // per-bucket reduction + merge cost: 8 adds for the ~255-bit fields
      // (round-2 sweep, profiles/r02_reduce_groups_prepared_c_sweep.txt:
      // BLS12-381 2^19 best at c = 16, 4.33 ms, where 3.4 picked c = 18, 4.74
      // ms; 2^22 keeps c = 20); MNT4-753's sweep is not monotone in c (the
      // merge phase), 3.4 picks its second-best c there
      const double per_bucket = N >= 24 ? 3.4 : 8.0;
      const double reduce = Mi * B * per_bucket * add + 60.0 * add * lat / 8.0;
      const double tail = (Mi - 1) * (c * 10.0 + add) * lat;
      const double cost = entries * madd + reduce + tail;
      if (cost < best_cost) { best_cost = cost; best = c; }
    }
    return best;
  }

  // Accumulation chunk size S (entries per thread).  64 by default; for small
  // shards the grid is a few waves of the resident threads and a partly
  // filled last wave idles SMs (n = 2^19 at c = 16: 3.46 waves, ~13 % lost),
  // so S in [40, 64] is picked to make the wave count just below an integer
  // (E estimated as n W, exact for uniform scalars up to zero digits).
  static uint64_t accum_resident_threads() {
    // per device (a multi-GPU process may drive GPUs of different SM counts)
    static std::mutex mu;
    static std::map<int, uint64_t> cache;
    const int dev = current_device();
    std::lock_guard<std::mutex> lock(mu);
    auto it = cache.find(dev);
    if (it != cache.end()) return it->second;
    int per_sm = 0;
    const size_t smem = (size_t)128 * Stage<C>::SLOT_WORDS * 4;
    if (smem > 48 * 1024 ||
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_accum<C>, 128, smem) != cudaSuccess)
      per_sm = 0;
    cudaGetLastError();
    const uint64_t v = (uint64_t)per_sm * device_sm_count() * 128;
    cache[dev] = v;
    return v;
  }
  static int chunk_entries_for(uint64_t E) {
    const uint64_t T = accum_resident_threads();
    if (!T || E == 0) return 64;
    auto eff = [&](int S) {
      const double w = (double)E / ((double)S * (double)T);
      return w / std::ceil(w);
    };
    if ((double)E / (64.0 * (double)T) >= 24.0) return 64;     // many waves: quantisation < 4 %
    int best = 64;
    double be = eff(64);
    for (int S = 63; S >= 40; --S)
      if (eff(S) > be + 0.02) { be = eff(S); best = S; }
    return best;
  }

  // Batch-affine levels before the XYZZ hot loop (affine.cuh): enough halvings
  // that an average bucket (E / M entries) is finished, at most 8 (a heavier
  // bucket -- the sparse witness's bucket 1 -- is left to the XYZZ chunks and
  // the heavy-bucket tree).  GZKP_AFFINE_LEVELS overrides (0 = XYZZ only).
  static int affine_levels(const Plan& p) {
    if constexpr (!AffineCfg<C>::ON) {
      return 0;
    } else {
      static const int env = [] {
        const char* e = getenv("GZKP_AFFINE_LEVELS");
        return e ? atoi(e) : -1;
      }();
      if (env >= 0) return std::min(env, 16);
      if (!AffineCfg<C>::DEFAULT_ON) return 0;
      const double avg = (double)p.E_max / (double)std::max<uint32_t>(p.M, 1);
      int L = 0;
      while (L < 8 && std::ldexp(1.0, L) < avg) ++L;
      return L;
    }
  }

  static Plan plan(size_t n, bool prepared, bool consolidated = false, int c_forced = 0, size_t table_n = 0,
                   int interval = 1) {
    Plan p;
    p.n = n;
    p.consolidated = consolidated;
    p.c = c_forced > 0 ? c_forced : window_bits(n);
    p.W = (C::SCALAR_BITS + 1 + p.c - 1) / p.c;
    p.B = 1u << (p.c - 1);
    p.Mi = consolidated ? std::min(std::max(interval, 1), p.W) : p.W;
    p.Wb = p.Mi;
    p.val_stride = consolidated ? (uint32_t)table_n : 0u;
    p.M = (uint32_t)p.Wb * p.B;
    int S = tunables().chunk_entries;
    if (S <= 0) {
      if (const char* e = getenv("GZKP_SEGMENT")) S = atoi(e);
    }
    if (S <= 0) S = chunk_entries_for((uint64_t)n * p.W);
    p.S = S;
    // reduction segment: up to 16 buckets, fewer when that leaves < ~32K threads
    {
      uint64_t seg = 16;
      while (seg > 1 && (uint64_t)p.Wb * p.B / seg < 32768) seg >>= 1;
      p.seg = (int)std::min<uint64_t>(seg, p.B);
    }
    p.E_max = (uint64_t)n * p.W;
    // window groups, top windows first, sizes halving down to a last group of
    // one window (window 0): the side stream merges / reduces / combines group
    // g while group g+1 accumulates, so only the last group's post-processing
    // is exposed.  Weighted points share one bucket set: a single group.
    p.groups.clear();
    // (Grp: t_lo, t_hi, key_lo, key_hi, chunk_base, chunks_max, heavy_levels, hmax, hbase)
    static const int pipeline = [] {
      const char* e = getenv("GZKP_PIPELINE");
      return e ? atoi(e) : 0;
    }();
    if (consolidated || !pipeline) {
      p.groups.push_back({0, p.W - 1, 0, p.M, 0, 0, 0, 0, 0});
    } else if (consolidated) {
      p.groups.push_back({0, p.W - 1, 0, p.B, 0, 0, 0, 0, 0});
    } else if (pipeline == 2 && p.W >= 2) {
      // two groups: the top windows' merge / reduction / Horner run on the
      // side stream while the bottom `low` windows accumulate (equal halves
      // unless GZKP_PIPELINE_LOW sets the bottom group's size)
      static const int low_env = [] {
        const char* e = getenv("GZKP_PIPELINE_LOW");
        return e ? atoi(e) : 0;
      }();
      const int low = low_env > 0 ? std::min(low_env, p.W - 1) : p.W / 2;
      const int mid = low;
      p.groups.push_back({mid, p.W - 1, (uint32_t)mid * p.B, (uint32_t)p.W * p.B, 0, 0, 0, 0, 0});
      p.groups.push_back({0, mid - 1, 0, (uint32_t)mid * p.B, 0, 0, 0, 0, 0});
    } else {
      int hi = p.W - 1;
      while (hi >= 0) {
        const int rem = hi + 1;
        const int sz = rem > 1 ? (rem + 1) / 2 : 1;
        p.groups.push_back({hi - sz + 1, hi, (uint32_t)(hi - sz + 1) * p.B, (uint32_t)(hi + 1) * p.B, 0, 0, 0, 0, 0});
        hi -= sz;
      }
    }
    p.chunks_max = 0;
    p.heavy_levels = 0;
    uint64_t seg_elems = 1, mid_elems = 1, terms_elems = 1, hlist_elems = 0;
    for (auto& g : p.groups) {
      const uint64_t wins = consolidated ? (uint64_t)p.W : (uint64_t)(g.t_hi - g.t_lo + 1);
      const uint64_t bwins = consolidated ? (uint64_t)p.Mi : wins;
      // reduction segment of this group: <= 16 buckets, fewer until >= 32K threads
      static const uint64_t target = [] {
        const char* e = getenv("GZKP_REDUCE_THREADS");
        const long v = e ? atol(e) : 32768;
        return (uint64_t)(v > 0 ? v : 32768);
      }();
      // one bucket set (weighted points) of the <= 12-limb fields: 8K threads
      // (round-2 sweep: BLS12-381 2^19 prepared reduce 0.407 -> 0.388 ms,
      // BN254 2^20 0.349 -> 0.304; MNT4-753 prefers 32K)
      const uint64_t tgt = (consolidated && N <= 12 && !getenv("GZKP_REDUCE_THREADS")) ? 8192 : target;
      auto seg_for = [&](uint64_t w) {
        uint64_t sg = 16;
        while (sg > 1 && w * p.B / sg < tgt) sg >>= 1;
        return (int)std::min<uint64_t>(sg, p.B);
      };
      g.seg = seg_for(bwins);
      // sub-groups: consolidated tables keep one (their M bucket sets are short)
      static const int rgroups = [] {
        const char* e = getenv("GZKP_REDUCE_GROUPS");
        const int v = e ? atoi(e) : 1;
        return v >= 1 ? v : 1;
      }();
      g.subs.clear();
      const int R = consolidated ? 1 : std::max(1, std::min<int>(rgroups, (int)wins));
      {
        int hi = consolidated ? p.Mi - 1 : g.t_hi;
        const int lo_all = consolidated ? 0 : g.t_lo;
        for (int k = 0; k < R; ++k) {
          const int rem = hi - lo_all + 1, sz = (rem + (R - k) - 1) / (R - k);
          g.subs.push_back({hi - sz + 1, hi, seg_for((uint64_t)sz)});
          hi -= sz;
        }
      }
      if (R > 1) p.split_reduce = true;
      for (const auto& sb : g.subs) {
        const uint64_t sw = (uint64_t)(sb.t_hi - sb.t_lo + 1);
        const uint64_t gsegs = p.B / sb.seg;
        seg_elems = std::max<uint64_t>(seg_elems, sw * gsegs);
        const uint64_t nb_bits = (uint64_t)ilog2_u64(gsegs) + 1;           // NB + 1 sets
        mid_elems = std::max<uint64_t>(mid_elems, sw * nb_bits * ((gsegs + RB_PER - 1) / RB_PER));
        terms_elems = std::max<uint64_t>(terms_elems, sw * nb_bits);
      }
      g.chunk_base = p.chunks_max;
      g.chunks_max = (n * wins + p.S - 1) / p.S + 1;
      // a heavy bucket spans > MERGE_QMAX chunks: at most chunks / MERGE_QMAX of them
      g.hmax = (uint32_t)(g.chunks_max / MERGE_QMAX + 2);
      g.hbase = (uint32_t)hlist_elems;
      hlist_elems += g.hmax;
      g.heavy_levels = 0;
      for (uint64_t span = 1; span < g.chunks_max; span *= HEAVY_SPAN) ++g.heavy_levels;
      p.heavy_levels = std::max(p.heavy_levels, g.heavy_levels);
      p.chunks_max += g.chunks_max;
    }
    const uint32_t G = p.B / p.seg;
    size_t o = 0;
    auto take = [&](size_t bytes) { size_t r = o; o = align_up(o + bytes); return r; };
    p.o_pts = prepared ? 0 : take(n * 2 * N * 4);
    if (!prepared) {
      p.o_scc = take(n * NS * 4);
      p.o_idx = take(n * 4);
      p.o_ncnt = take(4 * 8);      // counters [2] + ranges [4] + ones counter [1]
      p.ones_runs = (uint32_t)((n + ONES_RUN - 1) / ONES_RUN);
      p.o_ones = take(n * 4);
      p.o_opart = take((size_t)p.ones_runs * 4 * N * 4);
      p.o_oping = take(((size_t)p.ones_runs + TREE_SLICE - 1) / TREE_SLICE * 4 * N * 4);
    }
    p.o_codes = take((size_t)p.W * n * 4);
    p.o_counts = take((size_t)p.M * 4);
    p.o_hot = take(((size_t)p.M + 31) / 32 * 4);
    p.o_offsets = take(((size_t)p.M + 1) * 4);
    p.o_cursor = take((size_t)p.M * 4);
    p.o_tiles = take(SCAN_TILE * 4);
    p.o_vals = take(std::max<uint64_t>(p.E_max, 1) * 4);
    p.o_spay = take(2 * p.chunks_max * 4 * N * 4);
    p.o_cb = take(p.chunks_max * 8);                       // merge list (uint2 per spanning bucket)
    p.o_mcnt = take(4 * (p.groups.size() + 1));
    p.o_heavy = take(4 * (p.groups.size() + 4));
    p.o_hlist = take(16 * std::max<uint64_t>(hlist_elems, 1));
    p.o_hjobs = take(4 * (size_t)std::max(p.heavy_levels, 1) * (hlist_elems + p.groups.size()));
    p.o_state = take(4 * N * 4);
    p.o_buckets = take((size_t)p.M * 4 * N * 4);
    (void)G;
    p.seg_stride = (size_t)seg_elems * 4 * N;
    p.o_seg = take(2 * (size_t)seg_elems * 4 * N * 4);
    p.o_mid = take((size_t)mid_elems * 4 * N * 4);
    p.o_terms = take((size_t)terms_elems * 4 * N * 4);
    p.o_win = take((size_t)p.Wb * 4 * N * 4);
    // batch-affine levels: E_{l+1} <= E_l / 2 + min(M, E_l / 3) / 2 (a bucket
    // of c >= 3 entries keeps ceil(c / 2) <= (c + 1) / 2; c <= 2 finishes)
    p.aff_levels = affine_levels(p);
    if (p.aff_levels > 0) {
      auto next_cap = [&](uint64_t cap) { return cap / 2 + std::min<uint64_t>(p.M, cap / 3) / 2 + 1; };
      const uint64_t cap1 = next_cap(p.E_max), cap2 = next_cap(cap1);
      p.aff_ctas = (uint32_t)device_sm_count() * AffineCfg<C>::MINB;
      p.o_aoff = take(((size_t)p.M + 1) * 4);
      p.o_aoffA = take(((size_t)p.M + 1) * 4);
      p.o_aoffB = take(((size_t)p.M + 1) * 4);
      p.o_lvlA = take(cap1 * 2 * N * 4);
      p.o_lvlB = take(p.aff_levels > 1 ? cap2 * 2 * N * 4 : 4);
      p.o_ascr = take((size_t)p.aff_ctas * AffineCfg<C>::THREADS * AffineCfg<C>::BL * N * 4);
    }
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

  static gzkp_status to_mont(const void* in, void* out, size_t n, cudaStream_t s) { return to_mont_sc(in, out, n, nullptr, s); }
  static gzkp_status to_mont_sc(const void* in, void* out, size_t n, const void* sc, cudaStream_t s) {
    if (!n) return GZKP_SUCCESS;
    const int threads = 256;
    const size_t tiles = (n + 255) / 256;                    // one 256-point tile per warp
    const int grid = (int)std::min<size_t>((tiles + 7) / 8, (size_t)device_sm_count() * 16);
    k_to_mont<C><<<grid, threads, 0, s>>>((const uint32_t*)in, (uint32_t*)out, n, (const uint32_t*)sc);
    GZ_CHECK(cudaGetLastError());
    return GZKP_SUCCESS;
  }

  static gzkp_status msm(const MsmCall& call) {
    const size_t n = call.n;
    cudaStream_t s = call.stream;
    if (n == 0) {
      if (call.out_affine) GZ_CHECK(cudaMemsetAsync(call.out_affine, 0, 2 * N * 4, s));
      if (call.out_partial) GZ_CHECK(cudaMemsetAsync(call.out_partial, 0, 4 * N * 4, s));  // ZZ = ZZZ = 0: O
      return GZKP_SUCCESS;
    }
    if ((uint64_t)n >= (1ull << 31)) return set_error(GZKP_ERROR_INVALID_VALUE, "n >= 2^31 not supported");
    const Plan p = plan(n, call.prepared, call.consolidated, call.window_bits, call.table_n, call.interval);
    if (p.E_max >= (1ull << 32) - 1) return set_error(GZKP_ERROR_INVALID_VALUE, "n * windows >= 2^32");
    // the bucket-offset scan is two-level: <= SCAN_TILE tiles of SCAN_TILE keys
    if ((uint64_t)p.M > (uint64_t)SCAN_TILE * SCAN_TILE)
      return set_error(GZKP_ERROR_INVALID_VALUE, "too many bucket keys (window bits too large for this curve)");
    if (p.consolidated && (uint64_t)p.val_stride * ((p.W + p.Mi - 1) / p.Mi) >= (1ull << 31))
      return set_error(GZKP_ERROR_INVALID_VALUE, "weighted-point table >= 2^31 points");
    char* ws = (char*)call.workspace;
    if (!ws) {
      void* cached = nullptr;
      if (gzkp_status st = stream_workspace(s, p.total, &cached)) return st;
      ws = (char*)cached;
    } else if (call.workspace_bytes < p.total) {
      return set_error(GZKP_ERROR_INVALID_VALUE, "workspace too small");
    }
    return run(call, p, ws);
  }

  // a2 + a3: signed-window digits of every (point, window), bucket
  // histogram, exclusive scan -> offsets[0..M] (offsets[M] = E), and the
  // scatter of (point index | sign) into bucket order -> vals[0..E).
  static gzkp_status sort_stage(const MsmCall& call, const Plan& p, char* ws, int* launches,
                                const uint32_t* scalars = nullptr, const uint32_t* rng = nullptr,
                                const uint32_t* remap = nullptr) {
    cudaStream_t s = call.stream;
    const size_t n = call.n;
    auto U = [&](size_t off) { return (uint32_t*)(ws + off); };
    if (!scalars) scalars = (const uint32_t*)call.scalars;
    // a2: digits + histogram
    GZ_CHECK(cudaMemsetAsync(U(p.o_counts), 0, (size_t)p.M * 4, s));
    GZ_CHECK(cudaMemsetAsync(U(p.o_hot), 0, ((size_t)p.M + 31) / 32 * 4, s));
    GZ_CHECK(cudaMemsetAsync(U(p.o_mcnt), 0, 4 * (p.groups.size() + 1), s));
    GZ_CHECK(cudaMemsetAsync(U(p.o_heavy), 0, 4 * (p.groups.size() + 4), s));
    const uint32_t bpw = (uint32_t)((n + DIGIT_THREADS - 1) / DIGIT_THREADS);
    // rng (compaction): big range [rng[0], rng[1]) every window, small range
    // [rng[2], rng[3]) window 0 only; grids sized for n, blocks past a range exit
    k_digits<C><<<bpw, DIGIT_THREADS, 0, s>>>(scalars, n, p.c, p.W, p.B, (uint32_t)p.Mi, U(p.o_codes),
                                              U(p.o_counts), rng);
    if (rng)
      k_digits<C><<<bpw, DIGIT_THREADS, 0, s>>>(scalars, n, p.c, 1, p.B, (uint32_t)p.Mi, U(p.o_codes),
                                                U(p.o_counts), rng + 2);
    GZ_CHECK(cudaGetLastError());
    // exclusive scan -> offsets (+ cursor copy); offsets[M] = E
    const uint32_t ntiles = (uint32_t)((p.M + SCAN_TILE - 1) / SCAN_TILE);
    k_scan_tiles<<<ntiles, SCAN_THREADS, 0, s>>>(U(p.o_counts), U(p.o_offsets), p.M, U(p.o_tiles), U(p.o_hot));
    k_scan_top<<<1, SCAN_THREADS, 0, s>>>(U(p.o_tiles), ntiles, U(p.o_offsets) + p.M);
    k_scan_add<<<ntiles, SCAN_THREADS, 0, s>>>(U(p.o_offsets), U(p.o_cursor), p.M, U(p.o_tiles));
    // a3: scatter into bucket order (window-major grid)
    const uint32_t bpw_s = (uint32_t)((n + SCATTER_TILE - 1) / SCATTER_TILE);
    k_scatter<<<(unsigned)((uint64_t)bpw_s * p.W), SCATTER_THREADS, 0, s>>>(U(p.o_codes), n, bpw_s, p.B, (uint32_t)p.Mi,
                                                                         p.val_stride, U(p.o_hot), U(p.o_cursor), U(p.o_vals),
                                                                         rng, remap);
    if (rng)
      k_scatter<<<bpw_s, SCATTER_THREADS, 0, s>>>(U(p.o_codes), n, bpw_s, p.B, (uint32_t)p.Mi, p.val_stride, U(p.o_hot),
                                                  U(p.o_cursor), U(p.o_vals), rng + 2, remap);
    GZ_CHECK(cudaGetLastError());
    *launches += 5;
    return GZKP_SUCCESS;
  }

  // Test hook (gzkp_debug_buckets): the sort stage alone for window bits c;
  // copies offsets (M + 1 words) and vals (E words) to the host.
  static gzkp_status debug_buckets(const void* sc, size_t n, int c, uint32_t* off_host, size_t off_cap,
                                   uint32_t* vals_host, size_t vals_cap, cudaStream_t s) {
    const Plan p = plan(n, true, false, c);
    if (off_cap < (size_t)p.M + 1) return set_error(GZKP_ERROR_INVALID_VALUE, "offsets buffer too small");
    void* ws = nullptr;
    if (gzkp_status st = stream_workspace(s, p.total, &ws)) return st;
    MsmCall call;
    call.scalars = sc;
    call.n = n;
    call.prepared = true;
    call.stream = s;
    int launches = 0;
    if (n)
      if (gzkp_status st = sort_stage(call, p, (char*)ws, &launches)) return st;
    GZ_CHECK(cudaMemcpyAsync(off_host, (char*)ws + p.o_offsets, ((size_t)p.M + 1) * 4, cudaMemcpyDeviceToHost, s));
    GZ_CHECK(cudaStreamSynchronize(s));
    if (!n) {
      for (size_t k = 0; k <= p.M; ++k) off_host[k] = 0;
      return GZKP_SUCCESS;
    }
    const size_t E = off_host[p.M];
    if (vals_cap < E) return set_error(GZKP_ERROR_INVALID_VALUE, "vals buffer too small");
    GZ_CHECK(cudaMemcpyAsync(vals_host, (char*)ws + p.o_vals, E * 4, cudaMemcpyDeviceToHost, s));
    GZ_CHECK(cudaStreamSynchronize(s));
    return GZKP_SUCCESS;
  }

  // exclusive scan of in[0..count) -> out[0..count), out[count] = total
  static gzkp_status scan(const uint32_t* in, uint32_t* out, uint32_t count, uint32_t* tiles, cudaStream_t s) {
    const uint32_t ntiles = (count + SCAN_TILE - 1) / SCAN_TILE;
    if (ntiles > (uint32_t)SCAN_TILE) return set_error(GZKP_ERROR_INVALID_VALUE, "scan too large");
    k_scan_tiles<<<ntiles, SCAN_THREADS, 0, s>>>(in, out, count, tiles, nullptr);
    k_scan_top<<<1, SCAN_THREADS, 0, s>>>(tiles, ntiles, out + count);
    k_scan_add<<<ntiles, SCAN_THREADS, 0, s>>>(out, nullptr, count, tiles);
    GZ_CHECK(cudaGetLastError());
    return GZKP_SUCCESS;
  }

  // a4, batch-affine levels (affine.cuh): halve every bucket p.aff_levels
  // times; buckets left with one element are written to the bucket array.
  // Returns the residual level array and its offsets for the XYZZ hot loop.
  static gzkp_status affine_stage(const Plan& p, char* ws, const uint32_t* pts, cudaStream_t s,
                                  const uint32_t** offs_out, const uint32_t** pts_out, int* launches) {
    auto U = [&](size_t off) { return (uint32_t*)(ws + off); };
    const uint32_t* off_in = U(p.o_offsets);
    const uint32_t* in = pts;
    for (int l = 0; l < p.aff_levels; ++l) {
      uint32_t* cnt_out = U(p.o_counts);       // dead after the sort
      uint32_t* cnt_next = U(p.o_cursor);
      uint32_t* off_out = U(p.o_aoff);
      uint32_t* off_next = U((l & 1) ? p.o_aoffB : p.o_aoffA);
      uint32_t* out = U((l & 1) ? p.o_lvlB : p.o_lvlA);
      k_level_counts<<<(p.M + 255) / 256, 256, 0, s>>>(off_in, p.M, cnt_out, cnt_next);
      GZ_CHECK(cudaGetLastError());
      if (gzkp_status st = scan(cnt_out, off_out, p.M, U(p.o_tiles), s)) return st;
      if (gzkp_status st = scan(cnt_next, off_next, p.M, U(p.o_tiles), s)) return st;
      const size_t smem = (size_t)AffineCfg<C>::THREADS * AffineIn<C, true>::SLOT_WORDS * 4;
      if (l == 0)
        k_affine_level<C, true><<<p.aff_ctas, AffineCfg<C>::THREADS, smem, s>>>(
            U(p.o_vals), in, off_in, off_out, off_next, p.M, out, U(p.o_buckets), U(p.o_ascr));
      else
        k_affine_level<C, false><<<p.aff_ctas, AffineCfg<C>::THREADS, smem, s>>>(
            nullptr, in, off_in, off_out, off_next, p.M, out, U(p.o_buckets), U(p.o_ascr));
      GZ_CHECK(cudaGetLastError());
      *launches += 8;
      off_in = off_next;
      in = out;
    }
    *offs_out = off_in;
    *pts_out = in;
    return GZKP_SUCCESS;
  }

  static gzkp_status run(const MsmCall& call, const Plan& p, char* ws) {
    cudaStream_t s = call.stream;
    const size_t n = call.n;
    auto U = [&](size_t off) { return (uint32_t*)(ws + off); };
    ProfileRecord* prof = profile_begin(s);
    cudaEvent_t ev_begin = profile_event(prof, s);
    int launches = 0;
    const int sms = device_sm_count();

    // NEXT-2's mixed hot loop (GZKP_DFP=1), the 3-CTA build and the
    // batch-affine levels read Montgomery points, and so does the default;
    // GZKP_CANON=1 reads the caller's canonical points directly
    static const bool mixed = [] {
      const char* e = getenv("GZKP_DFP");
      return AccumCfg<C>::DFP && (e ? atoi(e) != 0 : AccumCfg<C>::DFP_DEFAULT);
    }();
    // GZKP_ACCUM_MINB=3: the BLS12-381 hot loop compiled for 3 CTAs / SM
    static const bool minb3 = [] {
      const char* e = getenv("GZKP_ACCUM_MINB");
      return AccumCfg<C>::DFP && e && atoi(e) == 3;
    }();
    // GZKP_CANON=1: the canonical-input hot loop (Canon, msm_kernels.cuh) --
    // no conversion pass, but each run start / flush does 1 / 2 products on
    // a divergent lane; measured slower (BLS12-381 2^22 accumulation 24.2 ->
    // 42.2 ms, ncu: no_instruction stalls 0.17M -> 1.53M samples), so off
    static const bool canon_env = [] {
      const char* e = getenv("GZKP_CANON");
      return e ? atoi(e) != 0 : false;
    }();
    const bool canon = Canon<C>::ON && canon_env && !call.prepared && !mixed && !minb3 && p.aff_levels == 0;
    // the scalar-1 points summed apart from the buckets (k_ones_sum; G1
    // curves up to 12 limbs; GZKP_ONES=0 keeps them in window 0's bucket 1)
    static const bool ones_env = [] {
      const char* e = getenv("GZKP_ONES");
      return e ? atoi(e) != 0 : true;
    }();
    const bool ones_on = Canon<C>::ON && N <= 12 && ones_env && !call.prepared && !canon;
    const uint32_t* ones_total = nullptr;
    // a1: points -> Montgomery (skipped for prepared handles and the canonical hot loop)
    const uint32_t* pts = (const uint32_t*)call.points;
    const uint32_t* sc_sorted = nullptr;
    const uint32_t* rng = nullptr;
    const uint32_t* remap = nullptr;
    if (!call.prepared) {
      // drop the zero scalars (small ones to the back), then convert the
      // remaining points in the compacted order
      GZ_CHECK(cudaMemsetAsync(U(p.o_ncnt), 0, 7 * 4, s));
      k_compact<C><<<(unsigned)((n + 255) / 256), 256, 0, s>>>((const uint32_t*)call.scalars, n, p.c, U(p.o_scc),
                                                              U(p.o_idx), U(p.o_ncnt),
                                                              ones_on ? U(p.o_ones) : nullptr);
      k_compact_ranges<<<1, 1, 0, s>>>(U(p.o_ncnt), (uint32_t)n, U(p.o_ncnt) + 2);
      if (canon) {
        remap = U(p.o_idx);                  // entries name the original point
      } else {
        const int cgrid = (int)std::min<size_t>((n + 255) / 256, (size_t)sms * 16);
        k_to_mont_c<C><<<cgrid, 256, 0, s>>>((const uint32_t*)call.points, U(p.o_idx), U(p.o_ncnt) + 2, U(p.o_pts));
        pts = U(p.o_pts);
        ++launches;
      }
      GZ_CHECK(cudaGetLastError());
      sc_sorted = U(p.o_scc);
      rng = U(p.o_ncnt) + 2;
      launches += 4;
      if constexpr (Canon<C>::ON && N <= 12) if (ones_on) {
        // run sums of the ones, then slice trees level by level (ping-pong)
        k_ones_sum<C><<<(p.ones_runs + 127) / 128, 128, 0, s>>>((const uint32_t*)call.points, U(p.o_ones),
                                                               U(p.o_ncnt) + 6, p.ones_runs, U(p.o_opart));
        uint32_t* src = U(p.o_opart);
        uint32_t* dst = U(p.o_oping);
        uint32_t cnt = p.ones_runs, div = 1;
        ++launches;
        while (cnt > 1) {
          const uint32_t nb = (cnt + TREE_SLICE - 1) / TREE_SLICE;
          k_tree_slices<C><<<nb, 128, 32 * CoopS<C>::WORDS * 4, s>>>(src, cnt, dst, U(p.o_ncnt) + 6, div);
          cnt = nb;
          div *= TREE_SLICE;
          std::swap(src, dst);
          ++launches;
        }
        GZ_CHECK(cudaGetLastError());
        ones_total = src;
      }
    }
    // a2 + a3: signed digits, bucket histogram, offsets, sort by bucket
    if (gzkp_status st = sort_stage(call, p, ws, &launches, sc_sorted, rng, remap)) return st;
    cudaEvent_t ev_sorted = profile_event(prof, s);
    profile_interval(prof, 0, ev_begin, ev_sorted);

    // a4..a8, pipelined by window group: accumulate group g on the caller's
    // stream; merge / reduce / combine it on the high-priority side stream
    // while group g+1 accumulates.  One group (weighted points): no side stream.
    const int ngroups = (int)p.groups.size();
    StreamCtx* ctx = nullptr;
    cudaStream_t ss = s, st2 = s;
    if (ngroups > 1 || p.split_reduce) {
      if (gzkp_status st = stream_ctx(s, &ctx)) return st;
      if (ngroups > 16) return set_error(GZKP_ERROR_INVALID_VALUE, "too many window groups");
      ss = ngroups > 1 ? ctx->side : s;
      st2 = ctx->side2;
    }
    const int threads = 128;
    // accumulation CTA size: small CTAs let the register file hold more warps
    // per SM (at ~176 regs/thread, 64-thread CTAs fit 10 warps, 128-thread 8)
    static const int acc_threads = [] {
      const char* e = getenv("GZKP_ACCUM_THREADS");
      const int v = e ? atoi(e) : AccumCfg<C>::THREADS;
      return (v >= 32 && v <= 128 && v % 32 == 0) ? v : AccumCfg<C>::THREADS;
    }();
    const size_t acc_smem = (size_t)acc_threads * Stage<C>::SLOT_WORDS * 4;
    // NEXT-2: the hot loop with 4 of 10 products on the FP64 pipe (BLS12-381): `mixed` above

    static int attr_tag;   // kernel attributes are per device
    if (gzkp_status st = once_per_device(&attr_tag, [] {
          GZ_CHECK(cudaFuncSetAttribute(k_accum<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        (int)((size_t)128 * Stage<C>::SLOT_WORDS * 4)));
          if constexpr (Canon<C>::ON)
            GZ_CHECK(cudaFuncSetAttribute(k_accum<C, false, AccumCfg<C>::MIN_CTAS, false, true>,
                                          cudaFuncAttributeMaxDynamicSharedMemorySize,
                                          (int)((size_t)128 * Stage<C>::SLOT_WORDS * 4)));
          if constexpr (AccumCfg<C>::DFP)
            GZ_CHECK(cudaFuncSetAttribute(k_accum<C, false, 3>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                          (int)((size_t)128 * Stage<C>::SLOT_WORDS * 4)));
          if constexpr (AccumCfg<C>::DFP)
            GZ_CHECK(cudaFuncSetAttribute(k_accum<C, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                          (int)((size_t)128 * Stage<C>::SLOT_WORDS * 4)));
          GZ_CHECK(cudaFuncSetAttribute(k_accum<C, false, AccumCfg<C>::MIN_CTAS, true>,
                                        cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        (int)((size_t)128 * Stage<C>::SLOT_WORDS * 4)));
          if constexpr (AffineCfg<C>::ON) {
            const int asm_ = (int)((size_t)AffineCfg<C>::THREADS * AffineIn<C, true>::SLOT_WORDS * 4);
            GZ_CHECK(cudaFuncSetAttribute(k_affine_level<C, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, asm_));
            GZ_CHECK(cudaFuncSetAttribute(k_affine_level<C, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, asm_));
          }
          GZ_CHECK(cudaFuncSetAttribute(k_reduce_bits<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        (int)rb_smem_bytes<C>()));
          if constexpr (coop_tree<C>())
            GZ_CHECK(cudaFuncSetAttribute(k_reduce_seg_coop<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                          (int)(32 * CoopS<C>::WORDS * 4)));
          GZ_CHECK(cudaFuncSetAttribute(k_heavy_tree<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        (int)((size_t)HEAVY_THREADS * 4 * N * 4)));
          return GZKP_SUCCESS;
        }))
      return st;
    // overlapped host->device path: the points are still arriving on another
    // stream while the digits / sort ran; only the accumulation needs them
    if (call.points_ready) GZ_CHECK(cudaStreamWaitEvent(s, call.points_ready, 0));
    cudaEvent_t ev_last_acc = nullptr, ev_merged = nullptr, ev_reduced = nullptr, ev_tailed = nullptr;
    // bucket layout of the accumulation's input (the residual level array's
    // after batch-affine levels); the reduction keeps the sorted layout's
    // offsets for "bucket non-empty"
    const uint32_t* offs = U(p.o_offsets);
    for (int gi = 0; gi < ngroups; ++gi) {
      const auto& gr = p.groups[gi];
      const Group grp{gr.key_lo, gr.key_hi, (uint32_t)gr.chunk_base};
      uint2* mlist = (uint2*)U(p.o_cb) + gr.chunk_base;
      uint32_t* mcnt = U(p.o_mcnt) + gi;
      // a4 (main stream)
      cudaEvent_t a0 = profile_event(prof, s);
      const unsigned acc_grid = (unsigned)((gr.chunks_max + acc_threads - 1) / acc_threads);
      bool affine = false;
      if constexpr (AffineCfg<C>::ON) {
        if (p.aff_levels > 0 && ngroups == 1) {
          const uint32_t* apts = nullptr;
          if (gzkp_status st = affine_stage(p, ws, pts, s, &offs, &apts, &launches)) return st;
          k_accum<C, false, AccumCfg<C>::MIN_CTAS, true><<<acc_grid, acc_threads, acc_smem, s>>>(
              nullptr, offs, grp, apts, p.S, U(p.o_buckets), U(p.o_spay), mlist, mcnt);
          affine = true;
        }
      }
      if (affine) {
      } else if constexpr (AccumCfg<C>::DFP) {
        if (mixed)
          k_accum<C, true><<<acc_grid, acc_threads, acc_smem, s>>>(U(p.o_vals), U(p.o_offsets), grp, pts, p.S,
                                                                   U(p.o_buckets), U(p.o_spay), mlist, mcnt);
        else if (minb3)
          k_accum<C, false, 3><<<acc_grid, acc_threads, acc_smem, s>>>(U(p.o_vals), U(p.o_offsets), grp, pts, p.S,
                                                                       U(p.o_buckets), U(p.o_spay), mlist, mcnt);
        else if (canon)
          k_accum<C, false, AccumCfg<C>::MIN_CTAS, false, true><<<acc_grid, acc_threads, acc_smem, s>>>(
              U(p.o_vals), U(p.o_offsets), grp, pts, p.S, U(p.o_buckets), U(p.o_spay), mlist, mcnt);
        else
          k_accum<C><<<acc_grid, acc_threads, acc_smem, s>>>(U(p.o_vals), U(p.o_offsets), grp, pts, p.S,
                                                             U(p.o_buckets), U(p.o_spay), mlist, mcnt);
      } else if constexpr (Canon<C>::ON) {
        if (canon)
          k_accum<C, false, AccumCfg<C>::MIN_CTAS, false, true><<<acc_grid, acc_threads, acc_smem, s>>>(
              U(p.o_vals), U(p.o_offsets), grp, pts, p.S, U(p.o_buckets), U(p.o_spay), mlist, mcnt);
        else
          k_accum<C><<<acc_grid, acc_threads, acc_smem, s>>>(U(p.o_vals), U(p.o_offsets), grp, pts, p.S,
                                                             U(p.o_buckets), U(p.o_spay), mlist, mcnt);
      } else {
        k_accum<C><<<acc_grid, acc_threads, acc_smem, s>>>(U(p.o_vals), U(p.o_offsets), grp, pts, p.S,
                                                           U(p.o_buckets), U(p.o_spay), mlist, mcnt);
      }
      GZ_CHECK(cudaGetLastError());
      cudaEvent_t a1 = profile_event(prof, s);
      profile_interval(prof, 1, a0, a1);
      ev_last_acc = a1;
      ++launches;
      if (ctx) {
        GZ_CHECK(cudaEventRecord(ctx->ev[gi], s));
        GZ_CHECK(cudaStreamWaitEvent(ss, ctx->ev[gi], 0));
      }
      // a5 (side stream): boundary partials -> buckets, heavy-bucket tree
      uint32_t* heavy = U(p.o_heavy) + gi;
      uint4* hlist = (uint4*)U(p.o_hlist) + gr.hbase;
      uint32_t* hjobs = U(p.o_hjobs) + (size_t)std::max(p.heavy_levels, 1) * (gr.hbase + gi);
      const int gm = (int)std::min<uint64_t>((gr.chunks_max + threads - 1) / threads, (uint64_t)sms * 16);
      k_merge_bucket<C><<<gm, threads, 0, ss>>>(offs, grp, p.S, mlist, mcnt, U(p.o_spay), U(p.o_buckets),
                                                heavy, hlist, gr.hmax);
      GZ_CHECK(cudaGetLastError());
      if (gr.heavy_levels > 0) {
        k_heavy_plan<<<1, 32, 0, ss>>>(heavy, hlist, gr.hmax, gr.heavy_levels, hjobs);
        GZ_CHECK(cudaGetLastError());
        ++launches;
      }
      const size_t hsmem = (size_t)HEAVY_THREADS * 4 * N * 4;
      uint64_t stride = 1;
      for (int l = 0; l < gr.heavy_levels; ++l, stride *= HEAVY_SPAN) {
        k_heavy_tree<C><<<sms * 2, HEAVY_THREADS, hsmem, ss>>>(heavy, hlist, gr.hmax, hjobs + (size_t)l * (gr.hmax + 1),
                                                             stride, grp, U(p.o_spay));
        GZ_CHECK(cudaGetLastError());
      }
      k_heavy_final<C><<<sms, threads, 0, ss>>>(heavy, hlist, gr.hmax, grp, U(p.o_spay), U(p.o_buckets));
      GZ_CHECK(cudaGetLastError());
      launches += 2 + gr.heavy_levels;
      ev_merged = profile_event(prof, ss);
      // a6 (side stream): bucket reduction of the group's windows, by
      // sub-group from the top; a7 (+ a8 on the last one): Horner over each
      // sub-group's windows on side stream 2, so a sub-group's chain runs while
      // the next sub-group is reduced and the next group merged (the chain
      // itself runs sub-group after sub-group)
      for (size_t k = 0; k < gr.subs.size(); ++k) {
        const auto& sb = gr.subs[k];
        const int gw = sb.t_hi - sb.t_lo + 1;
        const int t_lo = sb.t_lo;
        const uint32_t G = p.B / sb.seg;
        const uint32_t total = (uint32_t)gw * G;
        uint32_t* segT = U(p.o_seg);
        uint32_t* segR = segT + p.seg_stride;
        // small CTAs spread the ~W 2^(c-1) / s segment threads evenly over the
        // SMs (32K threads on 148 SMs: 128-thread CTAs leave some SMs at 1 CTA)
        static const int rcta = [] {
          const char* e = getenv("GZKP_REDUCE_CTA");
          const int v = e ? atoi(e) : 64;              // measured: 64 / 32 / 128 = 1.02 / 1.03 / 1.05 ms
          return (v >= 32 && v <= 128 && v % 32 == 0) ? v : 64;
        }();
        static const bool seg_coop = [] {
          const char* e = getenv("GZKP_SEG_COOP");
          return coop_tree<C>() && (e ? atoi(e) != 0 : true);
        }();
        // cooperative chains only where the reduction is small enough to be
        // latency-bound (round 2: BLS12-381 2^19 prepared, 64K adds, reduce
        // 0.393 -> 0.288 ms; 1M-add reductions -- standard 2^19 / 2^22,
        // prepared 2^22, MNT4-753 -- measured 10-12 % slower)
        if (seg_coop && (uint64_t)gw * p.B * 2 <= 262144) {
          const unsigned cgrid = (unsigned)((total + 31) / 32);
          k_reduce_seg_coop<C><<<cgrid, 128, 32 * CoopS<C>::WORDS * 4, ss>>>(U(p.o_buckets), U(p.o_offsets), t_lo,
                                                                            gw, p.B, sb.seg, segT, segR);
        } else {
          k_reduce_seg<C><<<(total + rcta - 1) / rcta, rcta, 0, ss>>>(U(p.o_buckets), U(p.o_offsets), t_lo, gw,
                                                                      p.B, sb.seg, segT, segR);
        }
        GZ_CHECK(cudaGetLastError());
        const int NB = ilog2_u64(G);
        const uint32_t nsl = (G + RB_PER - 1) / RB_PER;
        const size_t rsmem = rb_smem_bytes<C>();
        const uint32_t nslR = (G / 2 + RB_PER - 1) / RB_PER;
        k_reduce_bits<C><<<dim3(NB * nslR + nsl, gw), RB_THREADS, rsmem, ss>>>(segT, segR, G, NB, nsl, U(p.o_mid));
        GZ_CHECK(cudaGetLastError());
        k_reduce_bits_fin<C><<<dim3(NB + 1, gw), 32, 0, ss>>>(U(p.o_mid), G, NB, nsl, ilog2_u64(sb.seg),
                                                              U(p.o_terms));
        GZ_CHECK(cudaGetLastError());
        k_reduce_bits_sum<C><<<gw, 32, 0, ss>>>(U(p.o_terms), NB, U(p.o_win) + (size_t)t_lo * 4 * N);
        GZ_CHECK(cudaGetLastError());
        launches += 4;
        if constexpr (Canon<C>::ON && N <= 12) if (ones_total && t_lo == 0) {   // W_0 += the ones' sum (weight 1)
          k_add_point<C><<<1, 32, 0, ss>>>(U(p.o_win), ones_total);
          GZ_CHECK(cudaGetLastError());
          ++launches;
        }
        ev_reduced = profile_event(prof, ss);
        if (ctx) {
          const int evi = 16 + (int)(gi * 8 + k) % 40;
          GZ_CHECK(cudaEventRecord(ctx->ev[evi], ss));
          GZ_CHECK(cudaStreamWaitEvent(st2, ctx->ev[evi], 0));
        }
        const bool first = gi == 0 && k == 0;
        const bool last = gi == ngroups - 1 && k + 1 == gr.subs.size();
        k_tail<C><<<1, 32, 0, st2>>>(U(p.o_win), sb.t_hi, t_lo, p.c, first, last, U(p.o_state),
                                    last ? (uint32_t*)call.out_partial : nullptr,
                                    last ? (uint32_t*)call.out_affine : nullptr);
        GZ_CHECK(cudaGetLastError());
        ++launches;
        ev_tailed = profile_event(prof, st2);
      }
    }
    // phases 2-4 = the exposed post-processing of the last group
    profile_interval(prof, 2, ev_last_acc, ev_merged);
    profile_interval(prof, 3, ev_merged, ev_reduced);
    profile_interval(prof, 4, ev_reduced, ev_tailed);
    if (ctx) {   // join: later work on the caller's stream follows both side streams
      GZ_CHECK(cudaEventRecord(ctx->ev[ctx->nev - 1], ss));
      GZ_CHECK(cudaStreamWaitEvent(s, ctx->ev[ctx->nev - 1], 0));
      GZ_CHECK(cudaEventRecord(ctx->ev[ctx->nev - 4], st2));
      GZ_CHECK(cudaStreamWaitEvent(s, ctx->ev[ctx->nev - 4], 0));
    }
    profile_end(prof, U(p.o_offsets) + p.M, launches, p.c, s);
    return GZKP_SUCCESS;
  }

  // NEXT-1 prepare (Algorithm 1): the checkpoint table
  // table[j*n + i] = 2^(c M j) P_i (Montgomery affine), j < ceil(W / M), for
  // checkpoint interval M (M = 1: every window's weighted copy).  Returns the
  // window bits and the number of copies (the MSMs on this table use them).
  static gzkp_status precompute(const void* in, size_t n, int c, int interval, void* table, int* c_out, int* w_out,
                                cudaStream_t s) {
    if (c <= 0) c = window_bits_consolidated(n, interval);
    const int copies = table_windows(n, c, interval);
    const int M = std::min(std::max(interval, 1), (C::SCALAR_BITS + 1 + c - 1) / c);
    *c_out = c;
    *w_out = copies;
    if (!n) return GZKP_SUCCESS;
    uint32_t* T = (uint32_t*)table;
    if (gzkp_status st = to_mont(in, T, n, s)) return st;
    const int threads = 128;
    const int grid = (int)std::min<size_t>((n + threads - 1) / threads, (size_t)device_sm_count() * 32);
    for (int j = 1; j < copies; ++j) {
      k_precompute_step<C><<<grid, threads, 0, s>>>(T + (size_t)(j - 1) * n * 2 * N, T + (size_t)j * n * 2 * N, n,
                                                    c * M);
      GZ_CHECK(cudaGetLastError());
    }
    return GZKP_SUCCESS;
  }

  static int table_windows(size_t n, int c, int interval) {
    if (c <= 0) c = window_bits_consolidated(n, interval);
    const int W = (C::SCALAR_BITS + 1 + c - 1) / c;
    const int M = std::min(std::max(interval, 1), W);
    return (W + M - 1) / M;
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
    if (op == 8) {
      const int grid = (int)std::min<size_t>((n + 3) / 4, (size_t)device_sm_count() * 32);
      k_coop_mul_test<C><<<grid, 32, 0, s>>>((const uint32_t*)a, (const uint32_t*)b, (uint32_t*)out, n);
      GZ_CHECK(cudaGetLastError());
      return GZKP_SUCCESS;
    }
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

  static gzkp_status validate(const void* pts, const void* sc, size_t n, uint32_t* flags_host, cudaStream_t s) {
    *flags_host = 0;
    if (!n) return GZKP_SUCCESS;
    uint32_t* f = nullptr;
    GZ_CHECK(pool_malloc((void**)&f, 4, s));
    GZ_CHECK(cudaMemsetAsync(f, 0, 4, s));
    const int threads = 128;
    const int grid = (int)std::min<size_t>((n + threads - 1) / threads, (size_t)device_sm_count() * 16);
    k_validate<C><<<grid, threads, 0, s>>>((const uint32_t*)pts, (const uint32_t*)sc, n, f);
    GZ_CHECK(cudaGetLastError());
    GZ_CHECK(cudaMemcpyAsync(flags_host, f, 4, cudaMemcpyDeviceToHost, s));
    GZ_CHECK(cudaFreeAsync(f, s));
    GZ_CHECK(cudaStreamSynchronize(s));
    return GZKP_SUCCESS;
  }

  static const CurveImpl* get() {
    static const CurveImpl impl = {C::ID, C::N, C::NS, C::SCALAR_BITS,
                                   &Impl::window_bits, &Impl::workspace_bytes, &Impl::msm, &Impl::to_mont,
                                   &Impl::combine, &Impl::fixed_base, &Impl::field_op, &Impl::ec_op,
                                   &Impl::precompute, &Impl::table_windows, &Impl::validate, &Impl::debug_buckets};
    return &impl;
  }
};

}  // namespace gzkp
