// ntt.cuh -- N-NTT over the scalar field F_r (the POLY
// stage of PAPER.md:126-138 §2.2 and §3).
//
//   a_k = sum_{i<N} A_i w_N^(ik)  (forward),   A_i = N^-1 sum_k a_k w_N^(-ik)  (inverse)
//
// Radix-2 decimation-in-frequency (Gentleman-Sande) butterflies
//   x_i, x_{i+h}  ->  x_i + x_{i+h},  (x_i - x_{i+h}) w^((i mod h) N / 2h)
// over log N iterations, grouped into passes ("batches") of up to
// B iterations that run in shared memory.  A pass touches index bits
// [s, s+B): its independent groups are the 2^B elements that differ only in
// those bits.  Like GZKP's shuffle-less design (Fig. 4) the
// vector stays in natural order in HBM across passes, and one CTA takes G
// groups whose low bits are consecutive, so for every j the G elements
// (j 2^s + lo, lo = lo0..lo0+G-1) are contiguous in HBM: the CTA loads
// 2^B runs of G elements with coalesced 16-B accesses and writes them into
// shared memory as G interleaved groups (the "internal shuffle").
//
// Elements are AoS (one 8- or 24-limb value = 32 / 96 contiguous bytes), not
// the paper's column-major words: on sm_100 a warp's 16-B loads of 32
// consecutive AoS elements are fully coalesced sectors, and one thread then
// owns whole elements in registers (same field library as the MSM).
// Values stay canonical (no Montgomery conversion): twiddles are stored in
// Montgomery form, and mont(x, w R) = x w.  The last pass (times N^-1 for the
// inverse) writes a_k to position k, i.e. the DIF bit reversal is fused into
// the final store.
#pragma once
#include <cuda_runtime.h>

#include "field.cuh"

namespace gzkp {

constexpr int NTT_THREADS = 256;
constexpr int NTT_FIRST = 1, NTT_LAST = 2, NTT_SCALE = 4;

template <class R>
struct NttCfg {
  static constexpr int L = R::N;
  static constexpr int TILE_LOG = L <= 8 ? 11 : 10;     // 2048 x 32 B = 64 KB, 1024 x 96 B = 96 KB
  // radix-4 register rounds need 6 live elements: 48 words for L = 8 (fits the
  // 85-register budget of 3 CTAs/SM), 144 for L = 24 (radix-2 only)
  static constexpr bool RADIX4 = L <= 8;
  static constexpr int MIN_CTAS = L <= 8 ? 3 : 2;       // shared memory: 3 x 64 KB / 2 x 96 KB
};

template <class R>
GZ_DEV void ntt_ld(uint32_t d[R::N], const uint32_t* s) {
  const uint4* p = reinterpret_cast<const uint4*>(s);
#pragma unroll
  for (int i = 0; i < R::N / 4; ++i) {
    const uint4 v = p[i];
    d[4 * i] = v.x; d[4 * i + 1] = v.y; d[4 * i + 2] = v.z; d[4 * i + 3] = v.w;
  }
}
template <class R>
GZ_DEV void ntt_st(uint32_t* s, const uint32_t d[R::N]) {
  uint4* p = reinterpret_cast<uint4*>(s);
#pragma unroll
  for (int i = 0; i < R::N / 4; ++i) p[i] = make_uint4(d[4 * i], d[4 * i + 1], d[4 * i + 2], d[4 * i + 3]);
}

// F_r products in the NTT kernels are always the inlined CIOS body (also for
// the 24-limb MNT4-753 field, where F<R>::mul is an out-of-line call: that
// call inside these kernels gave wrong MNT4-753 butterflies on sm_100a).
template <class R>
struct NttF {
  using Fr = F<R>;
  static constexpr int L = R::N;
  GZ_DEV static void mul(uint32_t r[L], const uint32_t a[L], const uint32_t b[L]) { Fr::mul_inline(r, a, b); }
  GZ_DEV static void sqr(uint32_t r[L], const uint32_t a[L]) { Fr::mul_inline(r, a, a); }
  GZ_DEV static void to_mont(uint32_t r[L], const uint32_t a[L]) {
    uint32_t r2[L];
#pragma unroll
    for (int i = 0; i < L; ++i) r2[i] = R::R2(i);
    Fr::mul_inline(r, a, r2);
  }
  GZ_DEV static void from_mont(uint32_t r[L], const uint32_t a[L]) {
    uint32_t one[L];
    Fr::set_zero(one);
    one[0] = 1;
    Fr::mul_inline(r, a, one);
  }
};

// Shared-memory slot layout: element `slot` occupies words [slot L, slot L + L)
// with its 16-B pieces permuted by p ^ parity(slot >> 2): the 8 threads of an
// LDS.128/STS.128 phase then hit 8 distinct 16-B bank groups both for
// consecutive slots and for the strided slots of the late iterations
// (ncu r01: 50 % of shared wavefronts were conflicts without it).
template <class R>
GZ_DEV int sm_off(int slot, int piece) {
  return slot * R::N + 4 * (piece ^ (__popc((unsigned)slot >> 2) & 1));
}
template <class R>
GZ_DEV void sm_ld(uint32_t d[R::N], const uint32_t* sm, int slot) {
#pragma unroll
  for (int i = 0; i < R::N / 4; ++i) {
    const uint4 v = *reinterpret_cast<const uint4*>(sm + sm_off<R>(slot, i));
    d[4 * i] = v.x; d[4 * i + 1] = v.y; d[4 * i + 2] = v.z; d[4 * i + 3] = v.w;
  }
}
template <class R>
GZ_DEV void sm_st(uint32_t* sm, int slot, const uint32_t d[R::N]) {
#pragma unroll
  for (int i = 0; i < R::N / 4; ++i)
    *reinterpret_cast<uint4*>(sm + sm_off<R>(slot, i)) = make_uint4(d[4 * i], d[4 * i + 1], d[4 * i + 2], d[4 * i + 3]);
}

// One pass: iterations t0 .. t0+nb-1 (bits s = log_n - t0 - nb .. s+nb-1).
// CTA b owns groups q = b G .. b G + G - 1 (q = hi 2^s + lo); element (j, g)
// of the tile (j < 2^nb, g < G) is x[hi 2^(s+nb) + j 2^s + lo] with
// q = q0 + g, kept at shared slot j G + g.
// tw[k] = w^k (Montgomery), k < N/2 (w = w_N, or w_N^-1 for the inverse).
template <class R, int MINB = NttCfg<R>::MIN_CTAS>
__global__ void __launch_bounds__(NTT_THREADS, MINB) k_ntt_pass(const uint32_t* __restrict__ src, uint32_t* __restrict__ dst,
                                                          const uint32_t* __restrict__ tw, int log_n, int t0, int nb,
                                                          int logG, int flags, const uint32_t* __restrict__ scale) {
  using Fr = F<R>;
  using NF = NttF<R>;
  constexpr int L = R::N;
  extern __shared__ __align__(16) uint32_t ntt_smem[];
  const int s = log_n - t0 - nb;
  const int G = 1 << logG;
  const int T = G << nb;
  const uint64_t q0 = (uint64_t)blockIdx.x << logG;
  const int lb = s < logG ? s : logG;               // low bits that vary fastest in HBM order
  const uint64_t smask = (1ull << s) - 1;

  // HBM order e -> (j, g): lo fastest, then j, then the hi bits inside the CTA
  auto tile_pos = [&](int e, int& j, int& g) {
    const int lo = e & ((1 << lb) - 1);
    j = (e >> lb) & ((1 << nb) - 1);
    const int hl = e >> (lb + nb);
    g = (hl << lb) | lo;
  };
  auto gidx = [&](int j, int g) -> uint64_t {
    const uint64_t q = q0 + (uint64_t)g;
    return ((q >> s) << (s + nb)) | ((uint64_t)j << s) | (q & smask);
  };

  // ---- load (coalesced 16-B pieces) -> shared.  No Montgomery conversion:
  // the butterflies run on canonical values, since the product of a value x
  // with a Montgomery twiddle w R is mont(x, w R) = x w (the NTT is linear).
  {
    constexpr int PIECES = L / 4;
    for (int f = threadIdx.x; f < T * PIECES; f += NTT_THREADS) {
      const int e = f / PIECES, pc = f % PIECES;
      int j, g;
      tile_pos(e, j, g);
      const uint4 v = reinterpret_cast<const uint4*>(src + gidx(j, g) * L)[pc];
      *reinterpret_cast<uint4*>(ntt_smem + sm_off<R>(j * G + g, pc)) = v;
    }
  }
  __syncthreads();

  // ---- nb butterfly iterations in shared memory, two per round trip
  // (radix-4: a thread loads the quad j0, j0+h2, j0+hj, j0+hj+h2, runs
  // iterations u and u+1 in registers; iteration u+1's two butterflies share
  // one twiddle), then a radix-2 iteration if nb is odd
  const uint64_t lo_mask = smask;
  int u = 0;
  for (; NttCfg<R>::RADIX4 && u + 1 < nb; u += 2) {
    const int t = t0 + u;
    const int hj = 1 << (nb - 1 - u);
    const int h2 = hj >> 1;
    const int lowb = nb - 2 - u;
    for (int b = threadIdx.x; b < (T >> 2); b += NTT_THREADS) {
      const int g = b & (G - 1);
      const int jb = b >> logG;
      const int j0 = ((jb >> lowb) << (lowb + 2)) | (jb & ((1 << lowb) - 1));
      const uint64_t lo = (q0 + (uint64_t)g) & lo_mask;
      const uint64_t ka = ((((uint64_t)(j0 & (hj - 1))) << s) | lo) << t;
      const uint64_t kb = ((((uint64_t)((j0 & (hj - 1)) + h2)) << s) | lo) << t;
      const uint64_t kc = ((((uint64_t)(j0 & (h2 - 1))) << s) | lo) << (t + 1);
      uint32_t xa[L], xb[L], xc[L], xd[L], w[L], d[L];
      sm_ld<R>(xa, ntt_smem, j0 * G + g);
      sm_ld<R>(xb, ntt_smem, (j0 + h2) * G + g);
      sm_ld<R>(xc, ntt_smem, (j0 + hj) * G + g);
      sm_ld<R>(xd, ntt_smem, (j0 + hj + h2) * G + g);
      // iteration u: (a, c), (b, d)
      ntt_ld<R>(w, tw + ka * L);
      Fr::sub(d, xa, xc);
      Fr::add(xa, xa, xc);
      NF::mul(xc, d, w);
      ntt_ld<R>(w, tw + kb * L);
      Fr::sub(d, xb, xd);
      Fr::add(xb, xb, xd);
      NF::mul(xd, d, w);
      // iteration u+1: (a, b), (c, d), one twiddle
      ntt_ld<R>(w, tw + kc * L);
      Fr::sub(d, xa, xb);
      Fr::add(xa, xa, xb);
      NF::mul(xb, d, w);
      Fr::sub(d, xc, xd);
      Fr::add(xc, xc, xd);
      NF::mul(xd, d, w);
      sm_st<R>(ntt_smem, j0 * G + g, xa);
      sm_st<R>(ntt_smem, (j0 + h2) * G + g, xb);
      sm_st<R>(ntt_smem, (j0 + hj) * G + g, xc);
      sm_st<R>(ntt_smem, (j0 + hj + h2) * G + g, xd);
    }
    __syncthreads();
  }
  for (; u < nb; ++u) {                            // radix-2 iterations
    const int t = t0 + u;
    const int hj = 1 << (nb - 1 - u);
    for (int b = threadIdx.x; b < (T >> 1); b += NTT_THREADS) {
      const int g = b & (G - 1);
      const int jb = b >> logG;
      const int j1 = ((jb >> (nb - 1 - u)) << (nb - u)) | (jb & (hj - 1));
      const uint64_t lo = (q0 + (uint64_t)g) & lo_mask;
      const uint64_t k = ((((uint64_t)(j1 & (hj - 1))) << s) | lo) << t;
      uint32_t w[L], x1[L], x2[L], d[L];
      ntt_ld<R>(w, tw + k * L);
      sm_ld<R>(x1, ntt_smem, j1 * G + g);
      sm_ld<R>(x2, ntt_smem, (j1 + hj) * G + g);
      Fr::sub(d, x1, x2);
      Fr::add(x1, x1, x2);
      NF::mul(x2, d, w);
      sm_st<R>(ntt_smem, j1 * G + g, x1);
      sm_st<R>(ntt_smem, (j1 + hj) * G + g, x2);
    }
    __syncthreads();
  }

  // ---- store: natural order or, on the last pass, a_k at k = bitrev(i),
  // times N^-1 for the inverse (scale = N^-1 R: mont(x, N^-1 R) = x N^-1)
  if (flags & NTT_LAST) {
    const bool scaled = flags & NTT_SCALE;
    uint32_t c[L];
    if (scaled) ntt_ld<R>(c, scale);
    for (int e = threadIdx.x; e < T; e += NTT_THREADS) {
      int j, g;
      tile_pos(e, j, g);
      uint32_t x[L];
      sm_ld<R>(x, ntt_smem, j * G + g);
      if (scaled) NF::mul(x, x, c);
      const uint64_t i = gidx(j, g);
      const uint64_t k = __brevll(i) >> (64 - log_n);
      ntt_st<R>(dst + k * L, x);
    }
  } else {
    constexpr int PIECES = L / 4;
    for (int f = threadIdx.x; f < T * PIECES; f += NTT_THREADS) {
      const int e = f / PIECES, pc = f % PIECES;
      int j, g;
      tile_pos(e, j, g);
      reinterpret_cast<uint4*>(dst + gidx(j, g) * L)[pc] =
          *reinterpret_cast<const uint4*>(ntt_smem + sm_off<R>(j * G + g, pc));
    }
  }
}

// tw[k] = w^k for k < half (Montgomery), w = ROOT^(2^(S - log_n)), inverted when
// `inverse`; thread 0 of block 0 also writes the store scale N^-1 R =
// (1/2)^log_n R (Montgomery form; used by the inverse only).
template <class R>
__global__ void __launch_bounds__(128) k_ntt_twiddles(uint32_t* __restrict__ tw, uint64_t half, int log_n, int inverse,
                                                      uint32_t* __restrict__ scale) {
  using Fr = F<R>;
  using NF = NttF<R>;
  constexpr int L = R::N;
  constexpr int CH = 32;                               // consecutive powers per thread
  uint32_t w[L];
#pragma unroll
  for (int q = 0; q < L; ++q) w[q] = R::ROOT(q);
  NF::to_mont(w, w);
  for (int i = log_n; i < R::TWO_ADICITY; ++i) NF::sqr(w, w);      // w_N
  if (inverse) {                                                  // w_N^-1 = w_N^(N-1)
    uint32_t acc[L], b[L];
    Fr::set_one(acc);
    Fr::copy(b, w);
    for (int i = 0; i < log_n; ++i) {                             // N - 1 = 2^log_n - 1: all ones
      NF::mul(acc, acc, b);
      NF::sqr(b, b);
    }
    Fr::copy(w, acc);
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    uint32_t c[L], h[L];
#pragma unroll
    for (int q = 0; q < L; ++q) h[q] = R::HALF(q);
    NF::to_mont(h, h);
    Fr::set_one(c);
    for (int i = 0; i < log_n; ++i) NF::mul(c, c, h);
    ntt_st<R>(scale, c);
  }
  for (uint64_t k0 = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) * CH; k0 < half;
       k0 += (uint64_t)gridDim.x * blockDim.x * CH) {
    uint32_t acc[L], b[L];                 // w^k0 by square-and-multiply
    Fr::set_one(acc);
    Fr::copy(b, w);
    for (uint64_t e = k0; e; e >>= 1) {
      if (e & 1) NF::mul(acc, acc, b);
      NF::sqr(b, b);
    }
    for (int q = 0; q < CH && k0 + q < half; ++q) {
      ntt_st<R>(tw + (k0 + q) * L, acc);
      NF::mul(acc, acc, w);
    }
  }
}

}  // namespace gzkp
