// msm_kernels.cuh -- the Pippenger pipeline kernels (one template per curve).
//
// Steps:
//   a1 k_to_mont        canonical affine -> Montgomery affine           ("P ... unchanged")
//   a2 k_digits         signed c-bit digits of every (point, window) + bucket histogram
//      k_scan_*         exclusive scan -> bucket offsets (the p_index layout)
//   a3 k_scatter        counting-sort scatter of (point idx | sign) into bucket order
//   a4 k_accum          equal-work chunks of the sorted entries, XYZZ madd hot loop, points
//                       staged in shared memory by cp.async
//   a5 k_merge_bucket   sum of each bucket's chunk-boundary partials; k_heavy_* for skewed
//                       buckets (log-depth tree)
//   a6 k_reduce_seg/_win   bucket reduction sum_j j*B_j by running sums
//   a7 k_tail           window combination sum_t 2^(ct) W_t (Horner)
//   a8 k_tail/k_combine normalise XYZZ -> canonical affine
#pragma once
#include <cuda_runtime.h>

#include "ec.cuh"
#include "coop_smem.cuh"

#ifndef GZKP_COOP_SMEM
#define GZKP_COOP_SMEM 1   // serial chains on CoopS (shared-memory slots) for N >= 12; 0: CoopEC everywhere
#endif

namespace gzkp {

constexpr uint32_t VAL_NEG = 0x80000000u;    // entry / digit-code flag: negative digit
constexpr int MERGE_QMAX = 64;               // partials summed serially per bucket

// ---------------------------------------------------------------- digits
// Booth-style signed recoding: d_t = v_t + k_{ct-1} - 2^c * k_{ct+c-1}, with
// v_t = bits [ct, ct+c) of k.  Each digit depends only on c+1 bits, so windows
// are independent; d_t in [-2^(c-1), 2^(c-1)] and sum_t d_t 2^(ct) = k when
// k < 2^(cW-1), i.e. W = ceil((b+1)/c) (reading R7).
// `word(w)` returns scalar word w (0 beyond the scalar).
template <class WordFn>
GZ_DEV int booth_digit(WordFn word, int t, int c) {
  const int pos = t * c - 1;
  uint32_t x;
  if (pos < 0) {
    x = word(0) << 1;
  } else {
    const int w = pos >> 5, off = pos & 31;
    x = __funnelshift_r(word(w), word(w + 1), off);
  }
  x &= (c >= 31) ? 0xffffffffu : ((2u << c) - 1u);
  return (int)(x >> 1) + (int)(x & 1u) - (int)(((x >> c) & 1u) << c);
}

// digit code: 0 for a zero digit, else |d| | (d < 0) << 31; bucket key = |d| - 1
GZ_DEV uint32_t digit_code(int d) { return d ? ((uint32_t)abs(d) | (d < 0 ? VAL_NEG : 0u)) : 0u; }

// ------------------------------------------------------------ a1 to_mont
template <class C>
__global__ void __launch_bounds__(256) k_to_mont(const uint32_t* __restrict__ in, uint32_t* __restrict__ out, size_t n,
                                                 const uint32_t* __restrict__ sc) {
  // sc (optional): the call's scalars.  A point whose scalar is 0 is never
  // gathered by the accumulation, so its conversion is skipped (half the
  // points of the sparse witness; the conversion is IMAD-bound).
  // Each warp compacts the non-zero points of a 256-point tile into a shared
  // list first, so the products run on full warps instead of diverged ones.
  using Fp = Field<C>;
  using E = EC<C>;
  constexpr int N = C::N;
  constexpr int TILE = 256;
  __shared__ uint32_t s_list[8][TILE];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint32_t* list = s_list[warp & 7];
  const size_t wid = (blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5;
  const size_t nwarps = ((size_t)gridDim.x * blockDim.x) >> 5;
  for (size_t base = wid * TILE; base < n; base += nwarps * TILE) {
    int cnt = 0;
    for (int q = 0; q < TILE; q += 32) {
      const size_t i = base + q + lane;
      bool live = i < n;
      if (live && sc) {
        uint32_t any = 0;
#pragma unroll
        for (int w = 0; w < C::NS; ++w) any |= __ldg(sc + i * C::NS + w);
        live = any != 0;
      }
      const unsigned m = __ballot_sync(0xffffffffu, live);
      if (live) list[cnt + __popc(m & ((1u << lane) - 1u))] = (uint32_t)(q + lane);
      cnt += __popc(m);
    }
    __syncwarp();
    for (int e = lane; e < cnt; e += 32) {
      const size_t i = base + list[e];
      uint32_t x[N], y[N];
      E::ld(x, in + i * 2 * N);
      E::ld(y, in + i * 2 * N + N);
      Fp::to_mont(x, x);
      Fp::to_mont(y, y);
      E::st(out + i * 2 * N, x);
      E::st(out + i * 2 * N + N, y);
    }
    __syncwarp();
  }
}

// ------------------------------------------- zero-scalar compaction (a1)
// A zero scalar contributes nothing (half of the sparse
// witness's scalars are 0).  k_compact keeps the points with a non-zero
// scalar: their scalars go to sc_c and their indices to idx (block-level
// ballot scan, one atomic per block), so the digit codes, the sort and the
// point conversion only see the n' <= n live points (n' in *count).  The
// order of the blocks is unspecified; the sum does not depend on it.  A bucket
// entry then names the compacted point j; k_to_mont_c writes the Montgomery
// form of point idx[j] to pts_c[j], full warps (no idle lanes on zero scalars).
// Scalars below 2^(c-1) ("small": the 1s of the sparse witness) have one
// non-zero signed digit, in window 0, so they are packed at the END of the
// compacted arrays, [n - n_small, n), and the digit and scatter kernels run
// every window over the "big" range [0, n_big) but only window 0 over the
// small range.  count[0] = n_big, count[1] = n_small.
// ones (may be null): the indices of the points whose scalar is exactly 1 go
// to ones[0 .. count[6]) instead of the small range (k_ones_sum adds them).
template <class C>
__global__ void __launch_bounds__(256) k_compact(const uint32_t* __restrict__ sc, size_t n, int c,
                                                 uint32_t* __restrict__ sc_c, uint32_t* __restrict__ idx,
                                                 uint32_t* __restrict__ count, uint32_t* __restrict__ ones) {
  constexpr int NS = C::NS;
  __shared__ uint32_t s_warp[8], s_wsm[8], s_won[8], s_base, s_sbase, s_obase;
  const size_t i = (size_t)blockIdx.x * 256 + threadIdx.x;
  uint32_t k[NS];
  bool nz = false, small = false;
  if (i < n) {
    if constexpr (NS % 4 == 0) {
      const uint4* src = reinterpret_cast<const uint4*>(sc + i * NS);
#pragma unroll
      for (int q = 0; q < NS / 4; ++q) {
        const uint4 v = __ldg(src + q);
        k[4 * q] = v.x; k[4 * q + 1] = v.y; k[4 * q + 2] = v.z; k[4 * q + 3] = v.w;
      }
    } else {
#pragma unroll
      for (int q = 0; q < NS; ++q) k[q] = __ldg(sc + i * NS + q);
    }
    uint32_t any = 0, high = 0;
#pragma unroll
    for (int q = 0; q < NS; ++q) any |= k[q];
#pragma unroll
    for (int q = 1; q < NS; ++q) high |= k[q];
    nz = any != 0;
    small = nz && high == 0 && k[0] < (1u << (c - 1));
  }
  const bool one = ones && small && k[0] == 1u;
  small = small && !one;
  const bool big = nz && !small && !one;
  const unsigned m = __ballot_sync(0xffffffffu, big), ms = __ballot_sync(0xffffffffu, small);
  const unsigned mo = __ballot_sync(0xffffffffu, one);
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (lane == 0) { s_warp[w] = __popc(m); s_wsm[w] = __popc(ms); s_won[w] = __popc(mo); }
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t tot = 0, tots = 0, toto = 0;
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const uint32_t cb = s_warp[q], cs = s_wsm[q], co = s_won[q];
      s_warp[q] = tot; tot += cb;
      s_wsm[q] = tots; tots += cs;
      s_won[q] = toto; toto += co;
    }
    s_base = tot ? atomicAdd(count, tot) : 0u;
    s_sbase = tots ? atomicAdd(count + 1, tots) : 0u;
    s_obase = toto ? atomicAdd(count + 6, toto) : 0u;
  }
  __syncthreads();
  if (one) ones[s_obase + s_won[w] + __popc(mo & ((1u << lane) - 1u))] = (uint32_t)i;
  if (nz && !one) {
    const uint32_t pos = big ? s_base + s_warp[w] + __popc(m & ((1u << lane) - 1u))
                             : (uint32_t)(n - 1 - (s_sbase + s_wsm[w] + __popc(ms & ((1u << lane) - 1u))));
    if constexpr (NS % 4 == 0) {
      uint4* dst = reinterpret_cast<uint4*>(sc_c + (size_t)pos * NS);
#pragma unroll
      for (int q = 0; q < NS / 4; ++q) dst[q] = make_uint4(k[4 * q], k[4 * q + 1], k[4 * q + 2], k[4 * q + 3]);
    } else {
#pragma unroll
      for (int q = 0; q < NS; ++q) sc_c[(size_t)pos * NS + q] = k[q];
    }
    idx[pos] = (uint32_t)i;
  }
}

// rng = {0, n_big, n - n_small, n}: the big and the small ranges
static __global__ void k_compact_ranges(const uint32_t* __restrict__ count, uint32_t n, uint32_t* __restrict__ rng) {
  rng[0] = 0;
  rng[1] = count[0];
  rng[2] = n - count[1];
  rng[3] = n;
}

template <class C>
__global__ void __launch_bounds__(256) k_to_mont_c(const uint32_t* __restrict__ in, const uint32_t* __restrict__ idx,
                                                   const uint32_t* __restrict__ rng, uint32_t* __restrict__ out) {
  using Fp = Field<C>;
  using E = EC<C>;
  constexpr int N = C::N;
  const uint32_t nb = rng[1], s0 = rng[2], n = nb + (rng[3] - s0);
  for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
    const uint32_t j = v < nb ? v : s0 + (v - nb);
    const size_t i = __ldg(idx + j);
    uint32_t x[N], y[N];
    E::ld(x, in + i * 2 * N);
    E::ld(y, in + i * 2 * N + N);
    Fp::to_mont(x, x);
    Fp::to_mont(y, y);
    E::st(out + (size_t)j * 2 * N, x);
    E::st(out + (size_t)j * 2 * N + N, y);
  }
}

// ------------------------------------------ block-level hot-key aggregation
// Skewed scalars (the sparse witness: 40 % of the scalars are 1)
// send one bucket a large share of all entries.  Warp aggregation leaves one
// global atomic per warp on that bucket's counter, and same-address atomics
// serialise in one L2 slice (ncu r01: the sort of the 2^26 sparse MSM spent
// ~8 ms there).  A warp whose key is shared by >= HOT_MIN lanes therefore adds
// into a small shared-memory table first (open addressing on the key), and the
// block issues one global atomic per hot key.
constexpr int HOT_SLOTS = 32;
constexpr uint32_t HOT_MIN = 4;
constexpr uint32_t HOT_EMPTY = 0xffffffffu;

GZ_DEV int hot_slot(uint32_t* s_key, uint32_t key) {
  int h = (int)((key * 2654435761u) >> 27);            // 5 bits: HOT_SLOTS = 32
#pragma unroll 1
  for (int q = 0; q < HOT_SLOTS; ++q, h = (h + 1) & (HOT_SLOTS - 1)) {
    const uint32_t old = atomicCAS(&s_key[h], HOT_EMPTY, key);
    if (old == HOT_EMPTY || old == key) return h;
  }
  return -1;                                          // table full: global atomic
}

// ----------------------------------------------- a2 digits + histogram
// One thread per point.  The block stages its scalars in shared memory
// (coalesced 16-B loads; [word][thread] layout, conflict-free), each thread
// derives all W digits and writes the digit codes window-major (codes[t*n + i],
// coalesced).  Counting: warp match (match.any) is an MIO instruction with low
// throughput and ncu r02 showed k_digits / k_scatter MIO-bound, so it is used
// only where keys repeat: small digits |d| <= DIG_SMALL (the 0 / 1 / small-
// integer skew of the paper's witness) count into a shared-memory
// table flushed once per block; other keys go straight to a global RED unless
// the warp sees a key equal to its lane^1 or lane^2 neighbour's (repeated large
// digits, e.g. equal scalars), which takes the warp-aggregated path.
constexpr int DIGIT_THREADS = 256;
constexpr uint32_t DIG_SMALL = 16;
constexpr int DIG_SMALL_WIN = 64;             // small table: W <= 64 windows
// Bucket set of window t: t mod Mi (Mi = W: one set per window, standard;
// Mi = M: the checkpoint interval of GZKP's Algorithm 1, weighted points).
template <class C>
__global__ void __launch_bounds__(DIGIT_THREADS) k_digits(const uint32_t* __restrict__ sc, size_t n, int c, int W,
                                                          uint32_t B, uint32_t Mi, uint32_t* __restrict__ codes,
                                                          uint32_t* __restrict__ counts,
                                                          const uint32_t* __restrict__ rng) {
  // n: the codes' row stride; rng (device, may be null = [0, n)): the point
  // range [rng[0], rng[1]) this launch covers; W: the windows it writes (1
  // for the small-scalar range of the compaction)
  constexpr int NS = C::NS;
  __shared__ uint32_t s_sc[NS * DIGIT_THREADS];
  __shared__ uint32_t s_key[HOT_SLOTS], s_cnt[HOT_SLOTS];
  __shared__ uint32_t s_small[DIG_SMALL_WIN * DIG_SMALL];
  const size_t lo = rng ? (size_t)rng[0] : 0, hi = rng ? (size_t)rng[1] : n;
  const size_t base = lo + (size_t)blockIdx.x * DIGIT_THREADS;
  if (base >= hi) return;
  const size_t left = hi - base;
  const int rows = left < (size_t)DIGIT_THREADS ? (int)left : DIGIT_THREADS;
  const bool use_small = W <= DIG_SMALL_WIN;
  if (threadIdx.x < HOT_SLOTS) { s_key[threadIdx.x] = HOT_EMPTY; s_cnt[threadIdx.x] = 0; }
  for (int q = threadIdx.x; q < DIG_SMALL_WIN * (int)DIG_SMALL; q += DIGIT_THREADS) s_small[q] = 0;
  // coalesced staging: the block's scalars are rows*NS contiguous words
  for (int q = threadIdx.x; q < rows * NS; q += DIGIT_THREADS) {
    const int r = q / NS, w = q % NS;
    s_sc[w * DIGIT_THREADS + r] = __ldg(sc + base * NS + q);
  }
  __syncthreads();
  const int tid = threadIdx.x;
  const bool live = tid < rows;
  const size_t i = base + tid;
  auto word = [&](int w) -> uint32_t { return w < NS ? s_sc[w * DIGIT_THREADS + tid] : 0u; };
  const int lane = tid & 31;
  uint32_t tr = 0;                                     // t mod Mi
  for (int t = 0; t < W; ++t, tr = tr + 1 == Mi ? 0u : tr + 1) {
    const uint32_t code = live ? digit_code(booth_digit(word, t, c)) : 0u;
    if (live) codes[(size_t)t * n + i] = code;
    const uint32_t mag = code & ~VAL_NEG;
    const uint32_t key = tr * B + mag - 1u;
    const bool small = code && use_small && mag <= DIG_SMALL;
    if (__any_sync(0xffffffffu, small) && small) {       // skewed inputs: many lanes share a small digit
      const unsigned peers = __match_any_sync(__activemask(), mag);
      if (lane == __ffs(peers) - 1) atomicAdd(&s_small[t * DIG_SMALL + mag - 1], (uint32_t)__popc(peers));
    }
    const bool big = code && !small;
    const uint32_t k_or = big ? key : 0xffffffffu - (uint32_t)lane;    // distinct sentinels
    const uint32_t nb1 = __shfl_xor_sync(0xffffffffu, k_or, 1);   // every lane shuffles
    const uint32_t nb2 = __shfl_xor_sync(0xffffffffu, k_or, 2);
    const bool rep = big && (k_or == nb1 || k_or == nb2);
    if (__any_sync(0xffffffffu, rep)) {
      if (big) {
        const unsigned peers = __match_any_sync(__activemask(), key);
        if (lane == __ffs(peers) - 1) {
          const uint32_t cnt = (uint32_t)__popc(peers);
          const int h = cnt >= HOT_MIN ? hot_slot(s_key, key) : -1;
          if (h >= 0) atomicAdd(&s_cnt[h], cnt);
          else atomicAdd(&counts[key], cnt);
        }
      }
    } else if (big) {
      atomicAdd(&counts[key], 1u);
    }
  }
  __syncthreads();
  if (tid < HOT_SLOTS && s_key[tid] != HOT_EMPTY) atomicAdd(&counts[s_key[tid]], s_cnt[tid]);
  if (use_small)
    for (int q = tid; q < W * (int)DIG_SMALL; q += DIGIT_THREADS)
      if (s_small[q]) atomicAdd(&counts[(uint32_t)(q / DIG_SMALL) % Mi * B + q % DIG_SMALL], s_small[q]);
}

// Cross-window consolidation (§4.1, Algorithm 1; NEXT-1):
// with checkpoints P_{i,j} = 2^(c M j) P_i stored as table[j*n + i] (interval
// M), window t = M j + r uses checkpoint j and bucket set r: key = r B + |d| - 1,
// val = j n + i (val_stride = n).  M = 1 is the full weighted table (one
// bucket set); the standard pipeline is Mi = W, val_stride = 0.
// ------------------------------------------------------ a3 scatter (sort)
// Window-major 1-D grid (block b covers window b / bpw) so the blocks in
// flight write into one or two windows' 4n-byte ranges, which stay resident in
// L2 until their sectors are complete.  Positions come from the bucket cursors
// (offsets copy) with warp-aggregated atomics: one atomic per distinct bucket
// per warp, and one per block for hot keys (the block's run is reserved after
// a barrier); the order inside a bucket is irrelevant (exact abelian sum,
// DESIGN.md reading R11).
constexpr int SCATTER_THREADS = 256;
constexpr int SCATTER_PER_THREAD = 4;        // consecutive points of one window per thread (one 16-B load)
constexpr int SCATTER_TILE = SCATTER_THREADS * SCATTER_PER_THREAD;
// A key is "hot" (hotbits, set by k_scan_tiles from the exact histogram) when
// its bucket holds more than HOT_COUNT entries: only hot keys take the warp
// match + block reservation path; every other entry reserves its slot with
// one returning atomic (same-address contention <= HOT_COUNT per key).
constexpr uint32_t HOT_COUNT = 1024;
static __global__ void __launch_bounds__(SCATTER_THREADS) k_scatter(const uint32_t* __restrict__ codes, size_t n,
                                                             uint32_t bpw, uint32_t B, uint32_t Mi, uint32_t val_stride,
                                                             const uint32_t* __restrict__ hotbits,
                                                             uint32_t* __restrict__ cursor, uint32_t* __restrict__ vals,
                                                             const uint32_t* __restrict__ rng,
                                                             const uint32_t* __restrict__ remap) {
  // remap (may be null): entry value = remap[i] (the compacted point's
  // original index, for the canonical-input hot loop) instead of i
  // codes exist for i in [lo, hi) (rng, device; null = [0, n)), row stride n
  __shared__ uint32_t s_key[HOT_SLOTS], s_cnt[HOT_SLOTS], s_base[HOT_SLOTS];
  const int tid = threadIdx.x;
  const size_t lo = rng ? (size_t)rng[0] : 0, hi = rng ? (size_t)rng[1] : n;
  if (lo + (size_t)(blockIdx.x % bpw) * SCATTER_TILE >= hi) return;   // whole block past the range
  if (tid < HOT_SLOTS) { s_key[tid] = HOT_EMPTY; s_cnt[tid] = 0; }
  __syncthreads();
  const uint32_t t = blockIdx.x / bpw;
  const uint32_t kbase = t % Mi * B, vbase = t / Mi * val_stride;
  const size_t i0 = lo + (size_t)(blockIdx.x % bpw) * SCATTER_TILE + (size_t)tid * SCATTER_PER_THREAD;
  const uint32_t* crow = codes + (size_t)t * n;
  uint32_t code[SCATTER_PER_THREAD];
  if (i0 + SCATTER_PER_THREAD <= hi && (n % 4) == 0 && (i0 & 3) == 0) {
    const uint4 v = *reinterpret_cast<const uint4*>(crow + i0);
    code[0] = v.x; code[1] = v.y; code[2] = v.z; code[3] = v.w;
  } else {
#pragma unroll
    for (int q = 0; q < SCATTER_PER_THREAD; ++q) code[q] = i0 + q < hi ? crow[i0 + q] : 0u;
  }
  const int lane = tid & 31;
  unsigned peers[SCATTER_PER_THREAD];
  int leader[SCATTER_PER_THREAD], h[SCATTER_PER_THREAD];
  uint32_t pos[SCATTER_PER_THREAD];
  bool hot[SCATTER_PER_THREAD];
  bool any_hot = false;
#pragma unroll
  for (int q = 0; q < SCATTER_PER_THREAD; ++q) {
    peers[q] = 0; leader[q] = 0; h[q] = -1; pos[q] = 0;
    const uint32_t key = kbase + (code[q] & ~VAL_NEG) - 1u;
    hot[q] = code[q] && ((__ldg(hotbits + (key >> 5)) >> (key & 31)) & 1u);
    if (code[q] && !hot[q]) pos[q] = atomicAdd(&cursor[key], 1u);
    any_hot |= hot[q];
  }
  if (__syncthreads_or(any_hot)) {
#pragma unroll
    for (int q = 0; q < SCATTER_PER_THREAD; ++q) {
      const uint32_t key = kbase + (code[q] & ~VAL_NEG) - 1u;
      if (!__any_sync(0xffffffffu, hot[q])) continue;
      if (hot[q]) {
        peers[q] = __match_any_sync(__activemask(), key);
        leader[q] = __ffs(peers[q]) - 1;
        if (lane == leader[q]) {
          const uint32_t cnt = (uint32_t)__popc(peers[q]);
          h[q] = cnt >= HOT_MIN ? hot_slot(s_key, key) : -1;
          if (h[q] >= 0) pos[q] = atomicAdd(&s_cnt[h[q]], cnt);     // offset inside the block's run
          else pos[q] = atomicAdd(&cursor[key], cnt);
        }
      }
    }
    __syncthreads();
    if (tid < HOT_SLOTS && s_key[tid] != HOT_EMPTY) s_base[tid] = atomicAdd(&cursor[s_key[tid]], s_cnt[tid]);
    __syncthreads();
  }
#pragma unroll
  for (int q = 0; q < SCATTER_PER_THREAD; ++q) {
    if (code[q]) {
      uint32_t p = pos[q];
      if (hot[q]) {
        if (lane == leader[q] && h[q] >= 0) p += s_base[h[q]];
        p = __shfl_sync(peers[q], p, leader[q]) + __popc(peers[q] & ((1u << lane) - 1u));
      }
      const uint32_t pi = remap ? __ldg(remap + i0 + q) : (uint32_t)(i0 + q);
      vals[p] = (vbase + pi) | (code[q] & VAL_NEG);
    }
  }
}

// ----------------------------------------------------- scan (exclusive)
constexpr int SCAN_THREADS = 1024;
constexpr int SCAN_PER_THREAD = 4;
constexpr int SCAN_TILE = SCAN_THREADS * SCAN_PER_THREAD;

GZ_DEV uint32_t block_exclusive_scan(uint32_t v, uint32_t* warp_sums, uint32_t* total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) warp_sums[wid] = x;
  __syncthreads();
  if (wid == 0) {
    uint32_t s = lane < (int)(blockDim.x >> 5) ? warp_sums[lane] : 0u;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    warp_sums[lane] = s;    // inclusive
  }
  __syncthreads();
  const uint32_t base = wid ? warp_sums[wid - 1] : 0u;
  if (total) *total = warp_sums[(blockDim.x >> 5) - 1];
  return base + x - v;
}

static __global__ void k_scan_tiles(const uint32_t* __restrict__ in, uint32_t* __restrict__ out, uint32_t M,
                             uint32_t* __restrict__ tile_sums, uint32_t* __restrict__ hotbits) {
  __shared__ uint32_t ws[32];
  const size_t base = (size_t)blockIdx.x * SCAN_TILE + threadIdx.x * SCAN_PER_THREAD;
  uint32_t v[SCAN_PER_THREAD], s = 0;
#pragma unroll
  for (int k = 0; k < SCAN_PER_THREAD; ++k) {
    v[k] = (base + k < M) ? in[base + k] : 0u;
    s += v[k];
    if (hotbits && v[k] > HOT_COUNT) atomicOr(&hotbits[(base + k) >> 5], 1u << ((base + k) & 31));   // zeroed by the host
  }
  uint32_t total;
  uint32_t ex = block_exclusive_scan(s, ws, &total);
#pragma unroll
  for (int k = 0; k < SCAN_PER_THREAD; ++k) {
    if (base + k < M) out[base + k] = ex;
    ex += v[k];
  }
  if (threadIdx.x == 0) tile_sums[blockIdx.x] = total;
}

// single block: exclusive scan of tile sums (<= SCAN_TILE tiles), writes total to out_total
static __global__ void k_scan_top(uint32_t* __restrict__ tile_sums, uint32_t ntiles, uint32_t* __restrict__ out_total) {
  __shared__ uint32_t ws[32];
  const uint32_t base = threadIdx.x * SCAN_PER_THREAD;
  uint32_t v[SCAN_PER_THREAD], s = 0;
#pragma unroll
  for (int k = 0; k < SCAN_PER_THREAD; ++k) {
    v[k] = (base + k < ntiles) ? tile_sums[base + k] : 0u;
    s += v[k];
  }
  uint32_t total;
  uint32_t ex = block_exclusive_scan(s, ws, &total);
#pragma unroll
  for (int k = 0; k < SCAN_PER_THREAD; ++k) {
    if (base + k < ntiles) tile_sums[base + k] = ex;
    ex += v[k];
  }
  if (threadIdx.x == 0) *out_total = total;
}

static __global__ void k_scan_add(uint32_t* __restrict__ out, uint32_t* __restrict__ cursor, uint32_t M,
                           const uint32_t* __restrict__ tile_sums) {
  const uint32_t add = tile_sums[blockIdx.x];
  const size_t base = (size_t)blockIdx.x * SCAN_TILE;
  for (uint32_t k = threadIdx.x; k < SCAN_TILE; k += blockDim.x) {
    if (base + k < M) {
      const uint32_t v = out[base + k] + add;
      out[base + k] = v;
      if (cursor) cursor[base + k] = v;
    }
  }
}

// ---------------------------------------------------------- cp.async glue
GZ_DEV void cp_async16(void* smem, const void* gmem) {
  const uint32_t s = (uint32_t)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem) : "memory");
}
GZ_DEV void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int K>
GZ_DEV void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(K) : "memory"); }

template <class C>
struct Stage {
  static constexpr int N = C::N;
  static constexpr int PT_WORDS = 2 * N;                 // one affine point
  static constexpr int SLOT_WORDS = 2 * PT_WORDS + 4;    // double buffer + 16 B pad (bank spread)
  static constexpr int PT_CHUNKS = PT_WORDS / 4;         // 16-B pieces per point
  GZ_DEV static void fetch(uint32_t* slot_buf, const uint32_t* __restrict__ pts, uint32_t idx) {
    const uint32_t* src = pts + (size_t)idx * PT_WORDS;
#pragma unroll
    for (int q = 0; q < PT_CHUNKS; ++q) cp_async16(slot_buf + 4 * q, src + 4 * q);
  }
};

// -------------------------------------------------- a4 bucket accumulation
// Persistent grid-stride loop over chunks of S consecutive sorted entries
// (equal work per thread whatever the bucket sizes: PAPER.md:247-255's load
// balancing by construction).  Buckets are recovered from the offsets array
// (bucket k owns entries [off[k], off[k+1])).  A run of one bucket that lies
// wholly inside the chunk is written straight to the bucket; a run touching a
// chunk boundary (its bucket continues next door) becomes a boundary partial:
// the chunk's first run, continuing from the left, goes to slot 2*chunk, the
// last run, continuing to the right, to slot 2*chunk+1.  A bucket spanning
// chunks t0..t1 therefore has its partials at slot 2*t0+1 and the head slots
// 2*t of t0 < t <= t1 (k_merge_bucket relies on this).
// One window group of the pipeline (host-planned): bucket keys
// [key_lo, key_hi) own the sorted entries [off[key_lo], off[key_hi]); the
// group's chunks are numbered from 0 and its boundary partials live in slots
// 2*(chunk_base + j) (head) and 2*(chunk_base + j) + 1 (tail).
struct Group {
  uint32_t key_lo, key_hi, chunk_base;
};

// largest k in [lo, hi) with off[k] <= pos  (off non-decreasing, off[lo] <= pos < off[hi])
GZ_DEV uint32_t find_bucket(const uint32_t* __restrict__ off, uint32_t lo, uint32_t hi, uint32_t pos) {
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (__ldg(off + mid) <= pos) lo = mid; else hi = mid;
  }
  return lo;
}

// ---- canonical input points in the hot loop (no Montgomery conversion pass;
// GZKP_CANON=1 experiment, off: the per-run products below run on divergent
// lanes and cost more than the conversion pass saves)
// The affine input (x2, y2) enters madd only through U2 = x2 ZZ1 and
// S2 = y2 ZZZ1.  If the accumulator keeps ZZ and ZZZ "primed" -- the
// Montgomery representation of ZZ R and ZZZ R instead of ZZ and ZZZ -- then
// the Montgomery product of the raw canonical x2 with the primed ZZ1 is
// x2 ZZ1 R R / R = (x2 ZZ1) R, the ordinary Montgomery form of U2, and the
// products ZZ3 = ZZ1 PP, ZZZ3 = ZZZ1 PPP stay primed; X and Y are ordinary.
// A run starts from the representative with Z = lambda = 2^(-16N) (lambda^2 =
// 1/R): X = x (raw), Y = mont(y, K) = y lambda, ZZ' = R mod p (ONE),
// ZZZ' = lambda R mod p = K, K = 2^(16N) mod p -- one product per run instead
// of two conversions per point.  flush() returns ZZ, ZZZ to ordinary form
// (one REDC each), so buckets and partials leave in the usual XYZZ form.
template <class C>
struct Canon {
  static constexpr int N = C::N;
  static constexpr bool ON = std::is_same<Field<C>, F<C>>::value;   // G1 (F_p) curves
  GZ_DEV static void k_const(uint32_t k[N]) {
#pragma unroll
    for (int i = 0; i < N; ++i) k[i] = 0;
    if constexpr (16 * N < C::P_BITS) {
      k[(16 * N) / 32] = 1u << ((16 * N) % 32);
    } else {                            // the toy curves: p < 2^32, N = 2
      static_assert(N == 2, "canonical start constant");
      const uint64_t p = (uint64_t)C::P(0) | ((uint64_t)C::P(1) << 32);
      const uint64_t w = (1ull << 32) % p;                     // 2^(16N), 16N = 32
      k[0] = (uint32_t)w;
      k[1] = (uint32_t)(w >> 32);
    }
  }
  // run start: the affine canonical point (x, y) as a primed XYZZ point
  GZ_DEV static void start(typename EC<C>::Xyzz& A, const uint32_t x[N], const uint32_t y[N]) {
    using Fp = F<C>;
    uint32_t k[N];
    k_const(k);
    Fp::copy(A.X, x);
    Fp::mul(A.Y, y, k);
#pragma unroll
    for (int i = 0; i < N; ++i) { A.ZZ[i] = C::ONE(i); A.ZZZ[i] = k[i]; }
  }
  // primed <-> ordinary ZZ, ZZZ
  GZ_DEV static void unprime(typename EC<C>::Xyzz& A) {
    using Fp = F<C>;
    Fp::from_mont(A.ZZ, A.ZZ);
    Fp::from_mont(A.ZZZ, A.ZZZ);
  }
  GZ_DEV static void prime(typename EC<C>::Xyzz& A) {
    using Fp = F<C>;
    Fp::to_mont(A.ZZ, A.ZZ);
    Fp::to_mont(A.ZZZ, A.ZZZ);
  }
  // madd_nz on a primed accumulator with a canonical affine point; the
  // exceptional same-point case doubles the (equal) accumulator instead
  GZ_DEV static void madd(typename EC<C>::Xyzz& A, const uint32_t x2[N], const uint32_t y2[N]) {
    using Fp = F<C>;
    using E = EC<C>;
    uint32_t P[N], R[N], PP[N], PPP[N], t[N];
    Fp::mul(P, x2, A.ZZ);               // U2 (ordinary form, see above)
    Fp::sub(P, P, A.X);
    Fp::mul(R, y2, A.ZZZ);              // S2
    Fp::sub(R, R, A.Y);
    if (Fp::is_zero(P)) {
      if (Fp::is_zero(R)) {             // same point: 2 A = 2 (x2, y2), inline like madd_nz's mdbl
        uint32_t xm[N], ym[N];
        Fp::to_mont(xm, x2);
        Fp::to_mont(ym, y2);
        E::mdbl(A, xm, ym);
        prime(A);
      } else {
        E::set_inf(A);
      }
      return;
    }
    Fp::sqr(PP, P);
    Fp::mul(PPP, P, PP);
    Fp::mul(A.ZZ, A.ZZ, PP);            // ZZ3' = ZZ1' PP   (stays primed)
    Fp::mul(A.ZZZ, A.ZZZ, PPP);         // ZZZ3' = ZZZ1' PPP
    Fp::mul(PP, A.X, PP);               // Q = X1 PP
    Fp::sqr(t, R);
    Fp::sub(t, t, PPP);
    Fp::sub(t, t, PP);
    Fp::sub(A.X, t, PP);                // X3 = R^2 - PPP - 2Q
    Fp::sub(t, PP, A.X);
    Fp::neg(PP, A.Y);
    Fp::mul_sum(A.Y, R, t, PP, PPP);    // Y3 = R(Q - X3) - Y1 PPP
  }
};

// ---- the sparse witness's ones ("many 0s and 1s"): points
// whose scalar is exactly 1 skip the bucket pipeline.  k_compact lists them;
// k_ones_sum adds runs of ONES_RUN of them straight from the caller's
// canonical points with the primed accumulator of Canon (every thread starts
// and flushes a run at the same time, so unlike the hot loop no lane waits on
// another's conversion); k_tree_slices sums the run partials in slices of
// 512 (CoopS group trees), level by level; k_add_point adds the total to
// window 0's sum W_0, whose weight is 1.
constexpr uint32_t ONES_RUN = 64;
constexpr uint32_t TREE_SLICE = 512;
template <class C>
__global__ void __launch_bounds__(128) k_ones_sum(const uint32_t* __restrict__ pts, const uint32_t* __restrict__ ones,
                                                  const uint32_t* __restrict__ cnt_ptr, uint32_t runs,
                                                  uint32_t* __restrict__ part) {
  using Fp = F<C>;
  using E = EC<C>;
  constexpr int N = C::N;
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  const uint32_t cnt = *cnt_ptr;
  // runs past the live ones are never read (run 0 always writes, O if none)
  if (r >= runs || (r > 0 && r * ONES_RUN >= cnt)) return;
  const uint32_t lo = r * ONES_RUN, hi = min(cnt, lo + ONES_RUN);
  typename E::Xyzz acc;
  bool inf = true;
  uint32_t xn[N], yn[N];
  if (lo < hi) {
    const size_t i = __ldg(ones + lo);
    E::ld(xn, pts + i * 2 * N);
    E::ld(yn, pts + i * 2 * N + N);
  }
  for (uint32_t j = lo; j < hi; ++j) {
    uint32_t x[N], y[N];
    Fp::copy(x, xn);
    Fp::copy(y, yn);
    if (j + 1 < hi) {                   // one point ahead
      const size_t i = __ldg(ones + j + 1);
      E::ld(xn, pts + i * 2 * N);
      E::ld(yn, pts + i * 2 * N + N);
    }
    if (Fp::is_zero(x) && Fp::is_zero(y)) continue;   // identity input point
    if (inf) {
      Canon<C>::start(acc, x, y);
      inf = false;
    } else {
      Canon<C>::madd(acc, x, y);
      inf = E::is_inf(acc);
    }
  }
  if (inf) E::set_inf(acc);
  else Canon<C>::unprime(acc);
  E::store(part + (size_t)r * 4 * N, acc);
}

// out[b] = sum of v[b*TREE_SLICE .. min(cnt, (b+1)*TREE_SLICE)) (4N words
// each); v is overwritten.  128 threads = 32 CoopS groups, dynamic shared
// memory 32 x CoopS::WORDS words.
// ones_cnt (device, may be null): only the first ceil(ceil(*ones_cnt /
// ONES_RUN) / div) elements of v are live (div = TREE_SLICE^level); slices past
// them write O without work, so a dense input (no ones) costs ~nothing.
template <class C>
__global__ void __launch_bounds__(128) k_tree_slices(uint32_t* __restrict__ v, uint32_t cnt,
                                                     uint32_t* __restrict__ out, const uint32_t* __restrict__ ones_cnt,
                                                     uint32_t div) {
  constexpr int N = C::N;
  extern __shared__ __align__(16) uint32_t tree_smem[];
  const uint32_t lo = blockIdx.x * TREE_SLICE;
  if (lo >= cnt) return;                // CTA-uniform
  if (ones_cnt) {
    const uint32_t runs = (*ones_cnt + ONES_RUN - 1) / ONES_RUN;
    cnt = min(cnt, (runs + div - 1) / div);
    if (lo >= cnt) {                    // no live element in this slice: O
      typename EC<C>::Xyzz O;
      EC<C>::set_inf(O);
      if (threadIdx.x == 0) EC<C>::store(out + (size_t)blockIdx.x * 4 * N, O);
      return;
    }
  }
  uint32_t* base = v + (size_t)lo * 4 * N;
  CoopS<C>::tree_sum(base, (int)min(TREE_SLICE, cnt - lo), tree_smem, 32);
  for (int i = threadIdx.x; i < 4 * N; i += blockDim.x) out[(size_t)blockIdx.x * 4 * N + i] = base[i];
}

// dst += src (XYZZ, 4N words each) by one CoopS group
template <class C>
__global__ void __launch_bounds__(32) k_add_point(uint32_t* __restrict__ dst, const uint32_t* __restrict__ src) {
  using CS = CoopS<C>;
  __shared__ __align__(16) uint32_t gsm[CS::WORDS];
  if (threadIdx.x >= 4) return;
  CS::put_words(gsm, CS::AX, dst);
  CS::put_words(gsm, CS::BX, src);
  CS::add(gsm);
  CS::store_a(dst, gsm);
}

// CTAs per SM the hot loop is compiled for (registers: 128 / 168 / 255 per
// thread).  BN254 fits 3 CTAs in 168 registers; for BLS12-381 forcing 3 CTAs
// (166 regs) measured slower than the unconstrained 2 CTAs (85.6 % IMAD pipe).
template <class C>
struct AccumCfg {
  static constexpr int MIN_CTAS = C::N <= 8 ? 3 : 1;
  static constexpr int THREADS = 128;     // launch size (<= 128), GZKP_ACCUM_THREADS overrides
  // FP64 (DFP) products available: 48-bit limbs tile the radix and L = 8
  static constexpr bool DFP = C::HAS_DFP && (2 * C::N / 3 == 8);
  static constexpr bool DFP_DEFAULT = false;   // GZKP_DFP=1 selects the mixed hot loop
};

// One chunk per thread, non-persistent grid sized for the group's worst case
// (threads past the group's real chunk count exit): while the next group
// accumulates, finishing CTAs free slots for the high-priority side stream
// that merges / reduces / combines the previous group.
// MINB overrides the register budget (GZKP_ACCUM_MINB=3 selects 3 CTAs / SM,
// <= 168 registers, for BLS12-381; see msm_host.cuh).
// DIRECT: the entries are the points themselves (entry j = point j of `pts`,
// no index array, no sign): the residual level array of the batch-affine
// levels (affine.cuh).
// CANON: `pts` holds the canonical input points (indexed by the entries'
// original point index) instead of their Montgomery forms (Canon above).
template <class C, bool MIXED = false, int MINB = AccumCfg<C>::MIN_CTAS, bool DIRECT = false, bool CANON = false>
__global__ void __launch_bounds__(128, MINB)
    k_accum(const uint32_t* __restrict__ vals, const uint32_t* __restrict__ off, Group grp,
            const uint32_t* __restrict__ pts, int S, uint32_t* __restrict__ buckets, uint32_t* __restrict__ spay,
            uint2* __restrict__ mlist, uint32_t* __restrict__ mcnt) {
  using Fp = Field<C>;
  using EC_ = EC<C>;
  using St = Stage<C>;
  constexpr int N = C::N;
  extern __shared__ __align__(16) uint32_t stage_smem[];
  uint32_t* slot = stage_smem + threadIdx.x * St::SLOT_WORDS;

  const uint32_t G0 = __ldg(off + grp.key_lo), G1 = __ldg(off + grp.key_hi);
  const uint32_t nchunks = (G1 - G0 + S - 1) / S;
  const uint32_t chunk = blockIdx.x * blockDim.x + threadIdx.x;
  if (chunk >= nchunks) return;
  const uint32_t beg = G0 + chunk * (uint32_t)S;
  const uint32_t end = min(G1, beg + (uint32_t)S);
  const uint32_t sidx = 2 * (grp.chunk_base + chunk);
  uint32_t cur = find_bucket(off, grp.key_lo, grp.key_hi, beg);
  uint32_t nxt = __ldg(off + cur + 1);
  bool first_run = true;

  typename EC_::Xyzz acc;
  bool acc_inf = true;
  auto flush = [&](bool last_run) {
    const bool open_l = first_run && __ldg(off + cur) < beg;
    const bool open_r = last_run && nxt > end;
    if (acc_inf) EC_::set_inf(acc);
    else if constexpr (CANON) Canon<C>::unprime(acc);
    if (!open_l && !open_r) EC_::store(buckets + (size_t)cur * 4 * N, acc);
    else EC_::store(spay + (size_t)(open_l ? sidx : sidx + 1) * 4 * N, acc);
  };

  uint32_t v_next = DIRECT ? beg : vals[beg];
  St::fetch(slot, pts, v_next & ~VAL_NEG);
  cp_async_commit();
  for (uint32_t j = beg; j < end; ++j) {
    const uint32_t v = v_next;
    const int buf = (j - beg) & 1;
    if (j + 1 < end) {
      v_next = DIRECT ? j + 1 : vals[j + 1];
      St::fetch(slot + (buf ^ 1) * St::PT_WORDS, pts, v_next & ~VAL_NEG);
    }
    cp_async_commit();
    cp_async_wait<1>();
    if (j == nxt) {                       // bucket boundary: close the run
      flush(false);
      acc_inf = true;
      first_run = false;
      do { ++cur; nxt = __ldg(off + cur + 1); } while (nxt == j);   // skip empty buckets
    }
    uint32_t x[N], y[N];
    EC_::ld(x, slot + buf * St::PT_WORDS);
    EC_::ld(y, slot + buf * St::PT_WORDS + N);
    if (Fp::is_zero(x) && Fp::is_zero(y)) continue;     // identity input point
    if (v & VAL_NEG) Fp::neg(y, y);
    if (acc_inf) {
      if constexpr (CANON) Canon<C>::start(acc, x, y);
      else EC_::from_affine(acc, x, y);
      acc_inf = false;
    } else {
      if constexpr (CANON) Canon<C>::madd(acc, x, y);
      else if constexpr (MIXED) EC_::madd_nz_mixed(acc, x, y);   // IMAD + FP64 pipes (NEXT-2)
      else EC_::madd_nz(acc, x, y);
      acc_inf = EC_::is_inf(acc);
    }
  }
  cp_async_wait<0>();
  flush(true);
  // merge list: the chunk in which a spanning bucket STARTS owns its merge
  // (its last run is open to the right); one warp-aggregated append per warp
  const bool owner = nxt > end && __ldg(off + cur) >= beg;
  const unsigned act = __activemask();
  const unsigned om = __ballot_sync(act, owner);
  if (om) {
    const int lane = threadIdx.x & 31, lead = __ffs(om) - 1;
    uint32_t base = 0;
    if (lane == lead) base = atomicAdd(mcnt, (uint32_t)__popc(om));
    base = __shfl_sync(act, base, lead);
    if (owner) mlist[base + __popc(om & ((1u << lane) - 1u))] = make_uint2(cur, chunk);
  }
}

// ----------------------------------------------------------- a5 merge
// Thread per entry (k, t0) of the merge list that k_accum appended: bucket k
// starts in local chunk t0 and continues past it, up to chunk t1, so it has
// q = t1 - t0 + 1 partials (slot 2*(base+t0)+1, then head slots 2*(base+t)).
// q <= MERGE_QMAX: summed here.  Larger q (a heavy bucket of a skewed input)
// is appended to the group's heavy list (k, t0, t1) and reduced by the
// k_heavy_* kernels instead.  The compact list keeps every lane busy whatever
// the share of spanning buckets among the keys (small shards: few).
template <class C>
__global__ void __launch_bounds__(128) k_merge_bucket(const uint32_t* __restrict__ off, Group grp, int S,
                                                      const uint2* __restrict__ mlist, const uint32_t* __restrict__ mcnt,
                                                      const uint32_t* __restrict__ spay, uint32_t* __restrict__ buckets,
                                                      uint32_t* __restrict__ heavy_cnt, uint4* __restrict__ hlist,
                                                      uint32_t hmax) {
  using EC_ = EC<C>;
  constexpr int N = C::N;
  const uint32_t G0 = __ldg(off + grp.key_lo);
  const uint32_t cnt = *mcnt;
  for (uint32_t e = blockIdx.x * blockDim.x + threadIdx.x; e < cnt; e += gridDim.x * blockDim.x) {
    const uint2 m = mlist[e];
    const uint32_t k = m.x, t0 = m.y;
    const uint32_t t1 = (__ldg(off + k + 1) - 1 - G0) / S;
    if (t1 - t0 + 1 > (uint32_t)MERGE_QMAX) {
      const uint32_t h = atomicAdd(heavy_cnt, 1u);
      if (h < hmax) hlist[h] = make_uint4(k, t0, t1, 0u);   // hmax bounds every input (planner)
      continue;
    }
    typename EC_::Xyzz acc, X;
    EC_::load(acc, spay + (size_t)(2 * (grp.chunk_base + t0) + 1) * 4 * N);
    for (uint32_t t = t0 + 1; t <= t1; ++t) {
      EC_::load(X, spay + (size_t)(2 * (grp.chunk_base + t)) * 4 * N);
      ec_add_hot<C>(acc, X);
    }
    EC_::store(buckets + (size_t)k * 4 * N, acc);
  }
}

// Heavy buckets: the head slots of chunks t0+1 .. t1 (nheads = t1 - t0) are
// summed by a tree of fan-in HEAVY_SPAN = 1024 (one CTA of 128 threads, 8
// serial adds per thread, then a shared-memory tree).  Level l (stride
// HEAVY_SPAN^l) sums the level-(l-1) results at heads u = m * stride, job
// (h, seg) covering m in [seg SPAN, (seg+1) SPAN) and writing head seg SPAN
// stride.  job_off[l][h] = first job of bucket h at level l (k_heavy_plan), so
// a CTA maps its job to (h, seg) by binary search; no per-chunk bucket lookups.
constexpr int HEAVY_THREADS = 128;
constexpr uint32_t HEAVY_SPAN = 1024;

static __global__ void k_heavy_plan(const uint32_t* __restrict__ heavy_cnt, const uint4* __restrict__ hlist,
                                    uint32_t hmax, int levels, uint32_t* __restrict__ job_off) {
  // one block: job_off[l * (hmax + 1) + h], exclusive prefix over h (serial
  // per level on thread l: the heavy list is short -- usually 1 .. W entries)
  const uint32_t H = min(*heavy_cnt, hmax);
  const int l = threadIdx.x;
  if (l >= levels) return;
  uint64_t stride = 1;
  for (int q = 0; q < l; ++q) stride *= HEAVY_SPAN;
  uint32_t acc = 0;
  uint32_t* jo = job_off + (size_t)l * (hmax + 1);
  for (uint32_t h = 0; h < H; ++h) {
    jo[h] = acc;
    const uint4 e = hlist[h];
    const uint64_t nheads = e.z - e.y;
    const uint64_t m = (nheads + stride - 1) / stride;           // heads alive at this level
    acc += m > 1 ? (uint32_t)((m + HEAVY_SPAN - 1) / HEAVY_SPAN) : 0u;
  }
  jo[H] = acc;
}

template <class C>
__global__ void __launch_bounds__(HEAVY_THREADS) k_heavy_tree(const uint32_t* __restrict__ heavy_cnt,
                                                              const uint4* __restrict__ hlist, uint32_t hmax,
                                                              const uint32_t* __restrict__ job_off, uint64_t stride,
                                                              Group grp, uint32_t* __restrict__ spay) {
  using EC_ = EC<C>;
  constexpr int N = C::N;
  extern __shared__ __align__(16) uint32_t heavy_smem[];
  const uint32_t H = min(*heavy_cnt, hmax);
  const uint32_t jobs = job_off[H];
  for (uint32_t job = blockIdx.x; job < jobs; job += gridDim.x) {
    uint32_t lo = 0, hi = H;                 // largest h with job_off[h] <= job
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (job_off[mid] <= job) lo = mid; else hi = mid;
    }
    const uint4 e = hlist[lo];
    const uint32_t t0 = e.y;
    const uint64_t nheads = e.z - e.y;
    const uint64_t alive = (nheads + stride - 1) / stride;
    const uint64_t m0 = (uint64_t)(job - job_off[lo]) * HEAVY_SPAN;
    const uint64_t m1 = alive < m0 + HEAVY_SPAN ? alive : m0 + HEAVY_SPAN;
    auto slot = [&](uint64_t m) { return spay + (size_t)(2 * (grp.chunk_base + t0 + 1 + m * stride)) * 4 * N; };
    typename EC_::Xyzz acc, X;
    EC_::set_inf(acc);
    for (uint64_t m = m0 + threadIdx.x; m < m1; m += HEAVY_THREADS) {
      EC_::load(X, slot(m));
      ec_add_hot<C>(acc, X);
    }
    EC_::store(heavy_smem + threadIdx.x * 4 * N, acc);
    __syncthreads();
    for (int w = HEAVY_THREADS / 2; w > 0; w >>= 1) {
      if (threadIdx.x < w) {
        EC_::load(X, heavy_smem + (threadIdx.x + w) * 4 * N);
        ec_add_hot<C>(acc, X);
        EC_::store(heavy_smem + threadIdx.x * 4 * N, acc);
      }
      __syncthreads();
    }
    if (threadIdx.x == 0) EC_::store(slot(m0), acc);
    __syncthreads();
  }
}

// bucket k = tail partial of chunk t0 + the summed heads (head of chunk t0+1)
template <class C>
__global__ void __launch_bounds__(128) k_heavy_final(const uint32_t* __restrict__ heavy_cnt,
                                                     const uint4* __restrict__ hlist, uint32_t hmax, Group grp,
                                                     const uint32_t* __restrict__ spay, uint32_t* __restrict__ buckets) {
  using EC_ = EC<C>;
  constexpr int N = C::N;
  const uint32_t H = min(*heavy_cnt, hmax);
  for (uint32_t h = blockIdx.x * blockDim.x + threadIdx.x; h < H; h += gridDim.x * blockDim.x) {
    const uint4 e = hlist[h];
    typename EC_::Xyzz acc, X;
    EC_::load(acc, spay + (size_t)(2 * (grp.chunk_base + e.y) + 1) * 4 * N);
    EC_::load(X, spay + (size_t)(2 * (grp.chunk_base + e.y + 1)) * 4 * N);
    ec_add<C>(acc, X);
    EC_::store(buckets + (size_t)e.x * 4 * N, acc);
  }
}

// ------------------------------------------------- a6 bucket reduction
// W_t = sum_{j=1..B} j B_{t,j} (PAPER.md:239's prefix-sum bucket reduction),
// split so that every stage is either throughput-bound or short:
//   bucket j = g s + u + 1 (segment g < G = B/s, u < s):
//   W_t = sum_g T_g + s sum_g g R_g,   T_g = sum_u (u+1) B_{gs+u+1},  R_g = sum_u B_{gs+u+1}
//       = sum_g T_g + sum_k 2^(k + log2 s) S_k,   S_k = sum_{g : bit k of g} R_g.
// k_reduce_seg: T_g, R_g by running sums (2s adds per thread, all windows at
//   once: the only stage with real work, 2 adds per bucket).
// k_reduce_bits: the plain sums S_k (k < NB = log2 G) and A = sum_g T_g, in
//   slices of RB_PER elements per CTA (strided serial adds, then a shared-
//   memory tree).
// k_reduce_bits_fin: one warp per (set, window): sum of the slice partials
//   (lane-parallel adds + shuffle tree), then 2^(k + log2 s) by cooperative
//   doublings.
// k_reduce_bits_sum: one warp per window: W_t = sum of its NB + 1 terms.
// The per-segment scalar multiple (g s) R_g of a plain segmented running sum
// (a 15-bit double-and-add per thread) is gone; its work is now ~NB/2 adds
// per segment, all in plain sums.
// Group-local window index t (window t_lo + t); arrays are window-major.
template <class C>
__global__ void __launch_bounds__(128, 2) k_reduce_seg(const uint32_t* __restrict__ buckets,
                                                       const uint32_t* __restrict__ offsets, int t_lo, int W,
                                                       uint32_t B, int s, uint32_t* __restrict__ segT,
                                                       uint32_t* __restrict__ segR) {
  using EC_ = EC<C>;
  constexpr int N = C::N;
  const uint32_t G = B / s;
  const uint32_t total = (uint32_t)W * G;
  for (uint32_t id = blockIdx.x * blockDim.x + threadIdx.x; id < total; id += gridDim.x * blockDim.x) {
    const uint32_t t = t_lo + id / G, g = id % G;
    typename EC_::Xyzz R, T;
    EC_::set_inf(R);
    EC_::set_inf(T);
    for (int u = s - 1; u >= 0; --u) {
      const uint32_t key = t * B + g * s + u;
      if (__ldg(offsets + key + 1) != __ldg(offsets + key)) {
        typename EC_::Xyzz X;
        EC_::load(X, buckets + (size_t)key * 4 * N);
        ec_add_hot<C>(R, X);
      }
      ec_add_hot<C>(T, R);
    }
    EC_::store(segT + (size_t)id * 4 * N, T);
    EC_::store(segR + (size_t)id * 4 * N, R);
  }
}

// k_reduce_seg on 4-lane CoopS groups (N >= 12, GZKP_SEG_COOP): a segment's
// two running sums are one group's chain of cooperative adds -- ~3.5x lower
// latency per add than one thread at about the same issue cost (a level's
// four products fill the group's four lanes), so the 2s-add chains stop
// being latency-bound.  32 groups per 128-thread CTA; dynamic shared memory
// 32 x CoopS::WORDS words.  Used for small (latency-bound) reductions only:
// on million-add reductions the group's redundant field additions cost more
// issue slots than the lower latency saves (msm_host.cuh).
template <class C>
__global__ void __launch_bounds__(128) k_reduce_seg_coop(const uint32_t* __restrict__ buckets,
                                                         const uint32_t* __restrict__ offsets, int t_lo, int W,
                                                         uint32_t B, int s, uint32_t* __restrict__ segT,
                                                         uint32_t* __restrict__ segR) {
  using CS = CoopS<C>;
  constexpr int N = C::N;
  extern __shared__ __align__(16) uint32_t seg_smem[];
  uint32_t* gs = seg_smem + (threadIdx.x >> 2) * CS::WORDS;
  const uint32_t G = B / s;
  const uint32_t total = (uint32_t)W * G;
  const uint32_t gpb = blockDim.x >> 2;
  for (uint32_t id = blockIdx.x * gpb + (threadIdx.x >> 2); id < total; id += gridDim.x * gpb) {
    const uint32_t t = t_lo + id / G, g = id % G;
    CS::set_inf_a(gs, CS::AX);          // R (slots AX..)
    CS::set_inf_a(gs, CS::CX);          // T (slots CX..)
    for (int u = s - 1; u >= 0; --u) {
      const uint32_t key = t * B + g * s + u;
      if (__ldg(offsets + key + 1) != __ldg(offsets + key)) {
        CS::put_words(gs, CS::BX, buckets + (size_t)key * 4 * N);
        CS::add(gs, CS::AX, CS::BX);    // R += B_{gs+u+1}
      }
      CS::add(gs, CS::CX, CS::AX);      // T += R
    }
    CS::store_pt(segT + (size_t)id * 4 * N, gs, CS::CX);
    CS::store_pt(segR + (size_t)id * 4 * N, gs, CS::AX);
  }
}

constexpr uint32_t RB_PER = 512;          // set elements per k_reduce_bits CTA
constexpr int RB_THREADS = 128;
// the serial chains and short trees of the reduction run on CoopS groups for
// N >= 12 (GZKP_COOP_SMEM); k_reduce_bits' CTA tree uses RB_GROUPS of them
template <class C>
constexpr bool coop_tree() { return GZKP_COOP_SMEM && C::N >= 12; }
template <class C>
constexpr int rb_groups() { return C::N <= 12 ? RB_THREADS / 4 : 8; }
template <class C>
constexpr size_t rb_smem_bytes() {
  return (size_t)RB_THREADS * 4 * C::N * 4 + (coop_tree<C>() ? (size_t)rb_groups<C>() * CoopS<C>::WORDS * 4 : 0);
}

// set k < NB: the G/2 segments g with bit k set (e-th such g: insert a 1 at
// bit k of e); set NB: all G segments of segT.  The grid is exact, (slices of
// all sets, W): blockIdx.x < NB nslR are the R-set slices (set x / nslR),
// the rest the T-set's; CTA (k, slice) writes mid[((t (NB+1) + k) nsl + slice]
// (nsl = the T-set's slice count).  3 CTAs / SM so one wave holds the grid.
template <class C>
__global__ void __launch_bounds__(RB_THREADS, 3) k_reduce_bits(const uint32_t* __restrict__ segT,
                                                               const uint32_t* __restrict__ segR, uint32_t G, int NB,
                                                               uint32_t nsl, uint32_t* __restrict__ mid) {
  using EC_ = EC<C>;
  constexpr int N = C::N;
  extern __shared__ __align__(16) uint32_t red_smem[];
  const uint32_t nslR = (G / 2 + RB_PER - 1) / RB_PER;
  const uint32_t x = blockIdx.x, t = blockIdx.y;
  const bool rset = x < (uint32_t)NB * nslR;
  const uint32_t k = rset ? x / nslR : (uint32_t)NB;
  const uint32_t slice = rset ? x % nslR : x - (uint32_t)NB * nslR;
  const uint32_t size = (int)k < NB ? G / 2 : G;
  const uint32_t lo = slice * RB_PER, hi = min(size, lo + RB_PER);
  const uint32_t* src = ((int)k < NB ? segR : segT) + (size_t)t * G * 4 * N;
  typename EC_::Xyzz acc;
  EC_::set_inf(acc);
  for (uint32_t e = lo + threadIdx.x; e < hi; e += RB_THREADS) {
    const uint32_t g = (int)k < NB ? (((e >> k) << (k + 1)) | (1u << k) | (e & ((1u << k) - 1u))) : e;
    typename EC_::Xyzz X;
    EC_::load(X, src + (size_t)g * 4 * N);
    ec_add_hot<C>(acc, X);
  }
  EC_::store(red_smem + threadIdx.x * 4 * N, acc);
  __syncthreads();
  if constexpr (coop_tree<C>()) {
    CoopS<C>::tree_sum(red_smem, RB_THREADS, red_smem + RB_THREADS * 4 * N, rb_groups<C>());
    uint32_t* dst = mid + ((size_t)(t * (NB + 1) + k) * nsl + slice) * 4 * N;
    for (int i = threadIdx.x; i < 4 * N; i += RB_THREADS) dst[i] = red_smem[i];
    return;
  }
  for (uint32_t w = RB_THREADS / 2; w > 0; w >>= 1) {
    if (threadIdx.x < w) {
      typename EC_::Xyzz X;
      EC_::load(X, red_smem + (threadIdx.x + w) * 4 * N);
      ec_add_hot<C>(acc, X);
      EC_::store(red_smem + threadIdx.x * 4 * N, acc);
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) EC_::store(mid + ((size_t)(t * (NB + 1) + k) * nsl + slice) * 4 * N, acc);
}

// lane-parallel sum of a warp's points through shared memory (sm: 32 x 4N
// words): lanes < o add lane o + their index, 5 levels; lane 0 ends with the
// total.  (Shuffled operands feeding the out-of-line N >= 24 group law
// miscompile, see CoopEC::level, so the exchange goes through memory.)
template <class C>
GZ_DEV void warp_sum(typename EC<C>::Xyzz& acc, uint32_t* sm, int used = 32) {
  constexpr int N = C::N;
  const int lane = threadIdx.x & 31;
  int top = 1;                                   // levels only over the lanes that hold values
  while (top < used && top < 32) top <<= 1;
  for (int o = top >> 1; o > 0; o >>= 1) {
    EC<C>::store(sm + lane * 4 * N, acc);
    __syncwarp();
    if (lane < o) {
      typename EC<C>::Xyzz X;
      EC<C>::load(X, sm + (lane + o) * 4 * N);
      ec_add_hot<C>(acc, X);
    }
    __syncwarp();
  }
}

// <<<(NB+1, W), 32>>>: S_k (or A) from its slice partials, times 2^(k + log2 s)
template <class C>
__global__ void __launch_bounds__(32) k_reduce_bits_fin(uint32_t* __restrict__ mid, uint32_t G, int NB,
                                                        uint32_t nsl, int log_s, uint32_t* __restrict__ terms) {
  using EC_ = EC<C>;
  using CO = CoopEC<C>;
  constexpr int N = C::N;
  const uint32_t k = blockIdx.x, t = blockIdx.y;
  const uint32_t size = (int)k < NB ? G / 2 : G;
  const uint32_t used = (size + RB_PER - 1) / RB_PER;
  uint32_t* src = mid + (size_t)(t * (NB + 1) + k) * nsl * 4 * N;
  if constexpr (coop_tree<C>()) {
    // tree over the slice partials by the warp's 8 groups, then group 0
    // doubles (k + log2 s) times
    using CS = CoopS<C>;
    __shared__ __align__(16) uint32_t gsm[8 * CS::WORDS];
    CS::tree_sum(src, (int)used, gsm, 8);
    if (threadIdx.x < 4) {
      CS::put_words(gsm, CS::AX, src);
      if ((int)k < NB)
        for (int d = 0; d < (int)k + log_s; ++d) CS::dbl(gsm);
      CS::store_a(terms + (size_t)(t * (NB + 1) + k) * 4 * N, gsm);
    }
  } else {
    typename EC_::Xyzz acc;
    EC_::set_inf(acc);
    for (uint32_t q = threadIdx.x; q < used; q += 32) {
      typename EC_::Xyzz X;
      EC_::load(X, src + (size_t)q * 4 * N);
      ec_add_hot<C>(acc, X);
    }
    __shared__ __align__(16) uint32_t sm[32 * 4 * N];
    warp_sum<C>(acc, sm, (int)min(used, 32u));
    if (threadIdx.x == 0) EC_::store(sm, acc);
    __syncwarp();
    EC_::load(acc, sm);                 // every lane holds the sum (CoopEC)
    if ((int)k < NB)
      for (int d = 0; d < (int)k + log_s; ++d) CO::dbl(acc);
    if (threadIdx.x == 0) EC_::store(terms + (size_t)(t * (NB + 1) + k) * 4 * N, acc);
  }
}

// <<<W, 32>>>: W_t = sum of the window's NB + 1 terms (NB + 1 <= 32)
template <class C>
__global__ void __launch_bounds__(32) k_reduce_bits_sum(uint32_t* __restrict__ terms, int NB,
                                                        uint32_t* __restrict__ win_out) {
  using EC_ = EC<C>;
  constexpr int N = C::N;
  const uint32_t t = blockIdx.x;
  if constexpr (coop_tree<C>()) {
    using CS = CoopS<C>;
    __shared__ __align__(16) uint32_t gsm[8 * CS::WORDS];
    uint32_t* v = terms + (size_t)t * (NB + 1) * 4 * N;
    CS::tree_sum(v, NB + 1, gsm, 8);
    for (int i = threadIdx.x; i < 4 * N; i += 32) win_out[(size_t)t * 4 * N + i] = v[i];
  } else {
    typename EC_::Xyzz acc;
    EC_::set_inf(acc);
    if ((int)threadIdx.x <= NB) EC_::load(acc, terms + (size_t)(t * (NB + 1) + threadIdx.x) * 4 * N);
    __shared__ __align__(16) uint32_t sm[32 * 4 * N];
    warp_sum<C>(acc, sm, NB + 1);
    if (threadIdx.x == 0) EC_::store(win_out + (size_t)t * 4 * N, acc);
  }
}

// ----------------------------------------- a7 window combination + a8 output
// Q = sum_t 2^(ct) W_t by Horner from the top window, on ONE warp with the
// cooperative formulas (CoopEC).  Launch <<<1, 32>>>.  The pipeline calls it
// once per window group, top group first: windows t_hi down to t_lo; the
// running Q is carried in `state` (XYZZ) between groups; `first` starts from
// W_{t_hi}, `last` emits out_partial (XYZZ) and/or out_affine (canonical),
// either of which may be null.
template <class C>
__global__ void __launch_bounds__(32) k_tail(const uint32_t* __restrict__ win_out, int t_hi, int t_lo, int c,
                                             int first, int last, uint32_t* __restrict__ state,
                                             uint32_t* __restrict__ out_partial, uint32_t* __restrict__ out_affine) {
  using EC_ = EC<C>;
  using CO = CoopEC<C>;
  constexpr int N = C::N;
  if (blockIdx.x) return;
  typename EC_::Xyzz Q;
  int t = t_hi;
  if constexpr (GZKP_COOP_SMEM && N >= 12) {
    // CoopS (measured, tools/tail_bench.cu: BLS12-381 3.40 -> 3.28 us per
    // doubling, MNT4-753 13.5 -> 12.8; BN254 1.74 -> 1.77 keeps CoopEC)
    using CS = CoopS<C>;
    __shared__ __align__(16) uint32_t sm[CS::WORDS];
    if (threadIdx.x >= 4) return;                  // one 4-lane group runs the chain
    if (first) {
      CS::put_words(sm, CS::AX, win_out + (size_t)t * 4 * N);
      --t;
    } else {
      CS::put_words(sm, CS::AX, state);
    }
    for (; t >= t_lo; --t) {
      for (int k = 0; k < c; ++k) CS::dbl(sm);
      CS::put_words(sm, CS::BX, win_out + (size_t)t * 4 * N);
      CS::add(sm);
    }
    CS::get(Q, sm, CS::AX);
  } else {
    if (first) {
      EC_::load(Q, win_out + (size_t)t * 4 * N);
      --t;
    } else {
      EC_::load(Q, state);
    }
    for (; t >= t_lo; --t) {
      for (int k = 0; k < c; ++k) CO::dbl(Q);
      typename EC_::Xyzz X;
      EC_::load(X, win_out + (size_t)t * 4 * N);
      CO::add(Q, X);
    }
  }
  if (threadIdx.x) return;
  if (!last) {
    EC_::store(state, Q);
    return;
  }
  if (EC_::is_inf(Q)) EC_::set_inf(Q);
  if (out_partial) EC_::store(out_partial, Q);
  if (out_affine) {
    uint32_t x[N], y[N];
    ec_to_affine<C>(x, y, Q);
    EC_::st(out_affine, x);
    EC_::st(out_affine + N, y);
  }
}

// sum of `count` XYZZ partials in index order, normalised
template <class C>
__global__ void k_combine(const uint32_t* __restrict__ partials, int count, uint32_t* __restrict__ out_affine) {
  using EC_ = EC<C>;
  constexpr int N = C::N;
  if (threadIdx.x || blockIdx.x) return;
  typename EC_::Xyzz Q;
  EC_::set_inf(Q);
  for (int g = 0; g < count; ++g) {
    typename EC_::Xyzz X;
    EC_::load(X, partials + (size_t)g * 4 * N);
    ec_add<C>(Q, X);
  }
  uint32_t x[N], y[N];
  ec_to_affine<C>(x, y, Q);
  EC_::st(out_affine, x);
  EC_::st(out_affine + N, y);
}

// ------------------------------------ NEXT-1: weighted-point precompute
// table[t] = 2^c * table[t-1] (affine Montgomery), one thread per point: c
// doublings in XYZZ, then one inversion to return to affine.  Run once per
// point set at prepare time (the proving key is fixed).
template <class C>
__global__ void __launch_bounds__(128) k_precompute_step(const uint32_t* __restrict__ prev, uint32_t* __restrict__ next,
                                                         size_t n, int c) {
  using Fp = Field<C>;
  using EC_ = EC<C>;
  constexpr int N = C::N;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    uint32_t x[N], y[N];
    EC_::ld(x, prev + i * 2 * N);
    EC_::ld(y, prev + i * 2 * N + N);
    if (Fp::is_zero(x) && Fp::is_zero(y)) {           // O stays O
      EC_::st(next + i * 2 * N, x);
      EC_::st(next + i * 2 * N + N, y);
      continue;
    }
    typename EC_::Xyzz Q;
    EC_::from_affine(Q, x, y);
    for (int k = 0; k < c; ++k) ec_dbl<C>(Q);
    uint32_t ax[N], ay[N];
    ec_to_affine<C>(ax, ay, Q);                         // canonical, O -> (0,0)
    if (!(Fp::is_zero(ax) && Fp::is_zero(ay))) {
      Fp::to_mont(ax, ax);
      Fp::to_mont(ay, ay);
    }
    EC_::st(next + i * 2 * N, ax);
    EC_::st(next + i * 2 * N + N, ay);
  }
}

// ------------------------------------- input validation (GZKP_DEBUG_CHECKS=1)
// Off the hot path.  flags |= 1: a coordinate >= p; 2: a point off the curve
// y^2 = x^3 + a x + b; 4: a scalar >= 2^b.  b is not a product
// constant: it is recovered from the generator, b = G_y^2 - G_x^3 - a G_x.
// pts / sc may be null (validate only the other).  (0, 0) is the identity.
template <class C>
__global__ void __launch_bounds__(128) k_validate(const uint32_t* __restrict__ pts, const uint32_t* __restrict__ sc,
                                                  size_t n, uint32_t* __restrict__ flags) {
  using Fp = Field<C>;
  using EC_ = EC<C>;
  constexpr int N = C::N;
  uint32_t f = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    if (sc) {
      const uint32_t* k = sc + i * C::NS;
#pragma unroll 1
      for (int w = C::SCALAR_BITS / 32; w < C::NS; ++w) {
        const int lo = C::SCALAR_BITS - 32 * w;           // bits >= lo of word w must be 0
        const uint32_t mask = lo <= 0 ? 0xffffffffu : (lo >= 32 ? 0u : ~((1u << lo) - 1u));
        if (k[w] & mask) f |= 4u;
      }
    }
    if (!pts) continue;
    uint32_t x[N], y[N], xm[N], ym[N], t[N];
    EC_::ld(x, pts + i * 2 * N);
    EC_::ld(y, pts + i * 2 * N + N);
    if (Fp::is_zero(x) && Fp::is_zero(y)) continue;
    Fp::to_mont(xm, x);
    Fp::to_mont(ym, y);
    Fp::from_mont(t, xm);
    bool canon = Fp::eq(t, x);
    Fp::from_mont(t, ym);
    canon = canon && Fp::eq(t, y);
    if (!canon) { f |= 1u; continue; }
    // f(X, Y) = Y^2 - X^3 - a X, equal to b for every point on the curve
    auto rhs_gap = [](uint32_t r[N], const uint32_t X[N], const uint32_t Y[N]) {
      uint32_t u[N], v[N];
      Fp::sqr(r, Y);
      Fp::sqr(u, X);
      Fp::mul(u, u, X);
      Fp::sub(r, r, u);
      if constexpr (!C::A_ZERO) {
        uint32_t a[N];
#pragma unroll
        for (int q = 0; q < N; ++q) a[q] = C::A_MONT(q);
        Fp::mul(v, a, X);
        Fp::sub(r, r, v);
      }
    };
    uint32_t gx[N], gy[N], bg[N], bp[N];
#pragma unroll
    for (int q = 0; q < N; ++q) { gx[q] = C::GX(q); gy[q] = C::GY(q); }
    Fp::to_mont(gx, gx);
    Fp::to_mont(gy, gy);
    rhs_gap(bg, gx, gy);
    rhs_gap(bp, xm, ym);
    if (!Fp::eq(bg, bp)) f |= 2u;
  }
  if (f) atomicOr(flags, f);
}

// ---------------------------------------- fixed-base generator (bench inputs)
template <class C>
__global__ void __launch_bounds__(128) k_fixed_base(const uint32_t* __restrict__ sc, size_t n,
                                                    uint32_t* __restrict__ out) {
  using Fp = Field<C>;
  using EC_ = EC<C>;
  constexpr int N = C::N;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    // G in Montgomery form, rebuilt per point (2 muls; keeping it live across
    // the grid-stride loop miscompiled for the out-of-line N = 24 product)
    uint32_t gx[N], gy[N];
#pragma unroll
    for (int q = 0; q < N; ++q) { gx[q] = C::GX(q); gy[q] = C::GY(q); }
    Fp::to_mont(gx, gx);
    Fp::to_mont(gy, gy);
    const uint32_t* k = sc + i * C::NS;
    typename EC_::Xyzz Q;
    bool inf = true;
    for (int b = C::NS * 32 - 1; b >= 0; --b) {
      if (!inf) { ec_dbl<C>(Q); inf = EC_::is_inf(Q); }
      if ((__ldg(k + (b >> 5)) >> (b & 31)) & 1u) {
        if (inf) { EC_::from_affine(Q, gx, gy); inf = false; }
        else { ec_madd<C>(Q, gx, gy); inf = EC_::is_inf(Q); }
      }
    }
    if (inf) EC_::set_inf(Q);
    uint32_t x[N], y[N];
    ec_to_affine<C>(x, y, Q);
    EC_::st(out + i * 2 * N, x);
    EC_::st(out + i * 2 * N + N, y);
  }
}

// ------------------------------------------------- diagnostics (tests only)
template <class C>
__global__ void k_field_op(int op, const uint32_t* __restrict__ a, const uint32_t* __restrict__ b,
                           uint32_t* __restrict__ out, size_t n) {
  using Fp = Field<C>;
  using EC_ = EC<C>;
  constexpr int N = C::N;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    uint32_t x[N], y[N], r[N];
    EC_::ld(x, a + i * N);
    EC_::ld(y, b + i * N);
    switch (op) {
      case 0: Fp::to_mont(x, x); Fp::to_mont(y, y); Fp::mul(r, x, y); Fp::from_mont(r, r); break;
      case 1: Fp::add(r, x, y); break;
      case 2: Fp::sub(r, x, y); break;
      case 3: Fp::inv_canonical(r, x); break;
      case 7:   // constant-time binary-GCD inverse (canonical in / out), F_p curves
        if constexpr (std::is_same<Fp, F<C>>::value) Fp::inv_bingcd(r, x); else Fp::inv_canonical(r, x);
        break;
      case 5: Fp::to_mont(x, x); Fp::sqr(r, x); Fp::from_mont(r, r); break;
      case 6:   // FP64 (DFP) Montgomery product where available, else the IMAD one
        Fp::to_mont(x, x); Fp::to_mont(y, y);
        if constexpr (AccumCfg<C>::DFP) Dfp<C>::mul(r, x, y); else Fp::mul(r, x, y);
        Fp::from_mont(r, r);
        break;
      default: Fp::to_mont(r, x); Fp::from_mont(r, r); break;
    }
    EC_::st(out + i * N, r);
  }
}

// field op 8: the lane-split Montgomery product (coop_mul.cuh) on canonical
// inputs; one warp per CTA, lanes 8g .. 8g+7 multiply element base + g
template <class C>
__global__ void __launch_bounds__(32) k_coop_mul_test(const uint32_t* __restrict__ a, const uint32_t* __restrict__ b,
                                                      uint32_t* __restrict__ out, size_t n) {
  using Fp = Field<C>;
  constexpr int N = C::N;
  const int lane = threadIdx.x & 31, g = lane >> 3;
  for (size_t base = (size_t)blockIdx.x * 4; base < n; base += (size_t)gridDim.x * 4) {
    const size_t e = base + g < n ? base + g : n - 1;        // uniform control flow: clamp
    uint32_t x[N], y[N], r[N];
    EC<C>::ld(x, a + e * N);
    EC<C>::ld(y, b + e * N);
    Fp::to_mont(x, x);
    Fp::to_mont(y, y);
    if constexpr (CoopMul<C>::ON && std::is_same<Fp, F<C>>::value) CoopMul<C>::mul(r, x, y, CoopMul<C>::smem());
    else Fp::mul(r, x, y);
    Fp::from_mont(r, r);
    if ((lane & 7) == 0 && base + g < n) EC<C>::st(out + e * N, r);
  }
}

template <class C>
__global__ void k_ec_op(int op, const uint32_t* __restrict__ P, const uint32_t* __restrict__ Q,
                        uint32_t* __restrict__ out, size_t n) {
  using Fp = Field<C>;
  using EC_ = EC<C>;
  constexpr int N = C::N;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    uint32_t px[N], py[N], qx[N], qy[N];
    EC_::ld(px, P + i * 2 * N); EC_::ld(py, P + i * 2 * N + N);
    EC_::ld(qx, Q + i * 2 * N); EC_::ld(qy, Q + i * 2 * N + N);
    const bool p_inf = Fp::is_zero(px) && Fp::is_zero(py);
    const bool q_inf = Fp::is_zero(qx) && Fp::is_zero(qy);
    Fp::to_mont(px, px); Fp::to_mont(py, py); Fp::to_mont(qx, qx); Fp::to_mont(qy, qy);
    typename EC_::Xyzz A, B;
    if (p_inf) EC_::set_inf(A); else EC_::from_affine(A, px, py);
    if (q_inf) EC_::set_inf(B); else EC_::from_affine(B, qx, qy);
    // make A a genuinely projective point (ZZ != 1) by doubling twice and
    // halving back is not possible; instead scale: (X l^2, Y l^3, ZZ l^2, ZZZ l^3)
    if (!p_inf) {
      uint32_t l[N], l2[N], l3[N];
      Fp::add(l, py, px); Fp::add(l, l, px);           // some nonzero-ish lambda
      if (Fp::is_zero(l)) Fp::set_one(l);
      Fp::sqr(l2, l); Fp::mul(l3, l2, l);
      Fp::mul(A.X, A.X, l2); Fp::mul(A.ZZ, A.ZZ, l2);
      Fp::mul(A.Y, A.Y, l3); Fp::mul(A.ZZZ, A.ZZZ, l3);
    }
    switch (op) {
      case 0:
        if (q_inf) break;
        if (p_inf) EC_::from_affine(A, qx, qy); else ec_madd<C>(A, qx, qy);
        break;
      case 1: ec_add<C>(A, B); break;
      case 2: ec_dbl<C>(A); break;
      default:
        if (p_inf) EC_::set_inf(A); else ec_mdbl<C>(A, px, py);
        break;
    }
    uint32_t x[N], y[N];
    ec_to_affine<C>(x, y, A);
    EC_::st(out + i * 2 * N, x);
    EC_::st(out + i * 2 * N + N, y);
  }
}

}  // namespace gzkp

#include "affine.cuh"
