// affine.cuh -- batch-affine bucket accumulation (a4), the first levels of a
// pairwise tree inside every bucket.
//
// The bucket sums B_{t,j} ("summing up all the points in bucket
// j", §4.1 point-merging) need E - #buckets additions.  An XYZZ mixed
// addition costs 8M + 2S (ec.cuh); an AFFINE addition P + Q costs
//   lambda = (y_Q - y_P) / (x_Q - x_P),  x = lambda^2 - x_P - x_Q,
//   y = lambda (x_P - x) - y_P                       (2M + 1S + one inversion)
// and Montgomery's simultaneous-inversion trick replaces BL inversions by one
// inversion and 3 (BL - 1) products.  Additions that do not depend on each
// other are needed for that, so one level adds the bucket's entries in
// disjoint pairs (2j, 2j+1) and halves every bucket: level l reads the bucket-
// ordered array A_l (level 0: the sorted entries `vals`, gathered from the
// point table with the digit's sign) with offsets off_l and writes A_{l+1},
// off_{l+1}[k] = sum_{k' < k} ceil(cnt_l(k') / 2).  A thread owns BL
// consecutive outputs:
//   forward:  d_q = x_B - x_A (2 y_A for a doubling, 1 for a copy), prefix
//             products p_q = d_0 ... d_q (1M each) into a scratch array;
//   one inversion of p_{BL-1} (F::inv_bingcd: branch-free, so the 32 lanes
//             of a warp invert 32 batches at the cost of one);
//   backward: 1/d_q = inv p_{q-1}, inv <- inv d_q (2M), then the addition (2M + 1S).
// 5M + 1S + (inversion)/BL per addition instead of 8M + 2S.  Exceptional
// pairs are explicit: x_A == x_B and y_A == y_B doubles (lambda = (3x^2 + a) /
// 2y), x_A == x_B otherwise gives O, and O operands (the identity input (0,0)
// or a cancelled pair) copy the other operand.  The last levels (few entries
// per bucket) are summed by the XYZZ hot loop (k_accum, DIRECT mode).
#pragma once
#include <cuda_runtime.h>

#include <type_traits>

namespace gzkp {

template <class C>
struct AffineCfg {
  // F_p curves only (the F_p^2 inverse of the G2 curves is not branch-free)
  static constexpr bool ON = std::is_same<Field<C>, F<C>>::value;
  static constexpr int BL = C::N >= 24 ? 16 : 32;    // additions per inversion
  static constexpr int MINB = 3;                     // CTAs per SM (register budget)
  static constexpr int THREADS = 128;
  static constexpr bool DEFAULT_ON = false;          // GZKP_AFFINE_LEVELS=L selects L levels
};

enum : uint32_t { AFF_ADD = 0, AFF_DBL = 1, AFF_COPY_A = 2, AFF_COPY_B = 3, AFF_ZERO = 4 };

// per bucket k with c = ceil(cnt_in(k) / 2) outputs at this level:
// cnt_out[k] = c (every output, for the thread distribution) and
// cnt_next[k] = c if c >= 2 else 0 (a bucket left with ONE element is final:
// the level writes it to the bucket array and drops it from the next level)
static __global__ void k_level_counts(const uint32_t* __restrict__ off_in, uint32_t M, uint32_t* __restrict__ cnt_out,
                                      uint32_t* __restrict__ cnt_next) {
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < M; k += gridDim.x * blockDim.x) {
    const uint32_t c = (off_in[k + 1] - off_in[k] + 1) >> 1;
    cnt_out[k] = c;
    cnt_next[k] = c >= 2 ? c : 0u;
  }
}

// Pair staging: element e of a level's input array is a point (x, y)
// (Montgomery, O = (0, 0)); level 0 gathers it through vals[e] (index | sign),
// later levels read A_l[e].  cp.async copies into a per-thread shared-memory
// slot, double buffered so the next pair's loads overlap this pair's products.
template <class C, bool FIRST>
struct AffineIn {
  static constexpr int N = C::N;
  static constexpr int PAIR_WORDS = 4 * N;            // x_A | y_A | x_B | y_B
  static constexpr int SLOT_WORDS = 2 * PAIR_WORDS + 4;
  GZ_DEV static const uint32_t* src(const uint32_t* __restrict__ vals, const uint32_t* __restrict__ pts,
                                    uint32_t e, uint32_t& sign) {
    if constexpr (FIRST) {
      const uint32_t v = __ldg(vals + e);
      sign = v & 0x80000000u;
      return pts + (size_t)(v & ~0x80000000u) * 2 * N;
    } else {
      sign = 0;
      return pts + (size_t)e * 2 * N;
    }
  }
  // stage x (and y when `full`) of element e into dst (x at dst, y at dst + N)
  GZ_DEV static void stage(uint32_t* dst, const uint32_t* __restrict__ vals, const uint32_t* __restrict__ pts,
                           uint32_t e, bool full, uint32_t& sign) {
    const uint32_t* g = src(vals, pts, e, sign);
    if constexpr (N % 4 == 0) {
#pragma unroll
      for (int q = 0; q < N / 4; ++q) cp_async16(dst + 4 * q, g + 4 * q);
      if (full) {
#pragma unroll
        for (int q = 0; q < N / 4; ++q) cp_async16(dst + N + 4 * q, g + N + 4 * q);
      }
    } else {                      // the 2-limb toy curves: plain copies
#pragma unroll
      for (int q = 0; q < N; ++q) dst[q] = __ldg(g + q);
      if (full) {
#pragma unroll
        for (int q = 0; q < N; ++q) dst[N + q] = __ldg(g + N + q);
      }
    }
  }
};

// one level of the pairwise tree.  Persistent grid (T resident threads, the
// prefix-product scratch holds T x BL x N words, L2-resident); thread tid
// takes the batches of BL outputs tid, tid + T, ...
template <class C, bool FIRST>
__global__ void __launch_bounds__(AffineCfg<C>::THREADS, AffineCfg<C>::MINB)
    k_affine_level(const uint32_t* __restrict__ vals, const uint32_t* __restrict__ pts,
                   const uint32_t* __restrict__ off_in, const uint32_t* __restrict__ off_out,
                   const uint32_t* __restrict__ off_next, uint32_t M, uint32_t* __restrict__ out,
                   uint32_t* __restrict__ buckets, uint32_t* __restrict__ scratch) {
  using Fp = F<C>;
  using In = AffineIn<C, FIRST>;
  constexpr int N = C::N;
  constexpr int BL = AffineCfg<C>::BL;
  constexpr int PW = In::PAIR_WORDS;
  extern __shared__ __align__(16) uint32_t aff_smem[];
  uint32_t* slot = aff_smem + threadIdx.x * In::SLOT_WORDS;
  const uint32_t T = gridDim.x * blockDim.x;
  const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
  const uint32_t E_out = __ldg(off_out + M);
  auto scr = [&](int i, int w) -> uint32_t& { return scratch[((size_t)i * N + w) * T + tid]; };
  uint32_t r3[N];                 // R^3 mod p (Montgomery inverse fix-up)
  {
    uint32_t r2[N];
#pragma unroll
    for (int w = 0; w < N; ++w) r2[w] = C::R2(w);
    Fp::mul(r3, r2, r2);
  }
  // input pair of output q (bucket k): A = e, B = e + 1 if inside the bucket
  struct Pair { uint32_t e; bool pair; };
  auto pair_of = [&](uint32_t q, uint32_t k) -> Pair {
    const uint32_t e = __ldg(off_in + k) + 2 * (q - __ldg(off_out + k));
    return {e, e + 1 < __ldg(off_in + k + 1)};
  };
  for (uint64_t b0 = (uint64_t)tid * BL; b0 < E_out; b0 += (uint64_t)T * BL) {
    const uint32_t q0 = (uint32_t)b0;
    const uint32_t q1 = min(E_out, q0 + BL);
    uint32_t lo = 0, hi = M;            // bucket of q0: largest k with off_out[k] <= q0
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (__ldg(off_out + mid) <= q0) lo = mid; else hi = mid;
    }
    // ---- forward: classes and prefix products of the denominators (x only
    // staged; y is read only for the rare x == 0 / x_A == x_B cases)
    uint32_t acc[N];
    Fp::set_one(acc);
    uint64_t classes[(BL + 20) / 21] = {};   // 3 bits per output
    uint64_t signs = 0;                // level 0: digit signs, 2 bits per output
    uint32_t k = lo, kn = lo;
    auto fwd_stage = [&](uint32_t q, uint32_t& kk, uint32_t* dst) {
      while (__ldg(off_out + kk + 1) <= q) ++kk;
      const Pair pr = pair_of(q, kk);
      uint32_t sa, sb = 0;
      In::stage(dst, vals, pts, pr.e, false, sa);
      if (pr.pair) In::stage(dst + 2 * N, vals, pts, pr.e + 1, false, sb);
      signs |= (uint64_t)((sa >> 31) | ((sb >> 31) << 1)) << (2 * (q - q0));
    };
    fwd_stage(q0, kn, slot);
    cp_async_commit();
    for (uint32_t q = q0; q < q1; ++q) {
      uint32_t* cur = slot + ((q - q0) & 1) * PW;
      if (q + 1 < q1) fwd_stage(q + 1, kn, slot + ((q + 1 - q0) & 1) * PW);
      cp_async_commit();
      cp_async_wait<1>();
      while (__ldg(off_out + k + 1) <= q) ++k;
      const Pair pr = pair_of(q, k);
      uint32_t xa[N], xb[N], d[N];
#pragma unroll
      for (int w = 0; w < N; ++w) { xa[w] = cur[w]; xb[w] = pr.pair ? cur[2 * N + w] : 0u; }
      uint32_t cls;
      const bool xa0 = Fp::is_zero(xa), xb0 = Fp::is_zero(xb);
      if (xa0 || xb0 || Fp::eq(xa, xb)) {          // rare: needs the y coordinates
        uint32_t ya[N], yb[N], sg;
        EC<C>::ld(ya, In::src(vals, pts, pr.e, sg) + N);
        if (sg && !(xa0 && Fp::is_zero(ya))) Fp::neg(ya, ya);
        if (pr.pair) {
          EC<C>::ld(yb, In::src(vals, pts, pr.e + 1, sg) + N);
          if (sg && !(xb0 && Fp::is_zero(yb))) Fp::neg(yb, yb);
        } else {
          Fp::set_zero(yb);
        }
        const bool a_inf = xa0 && Fp::is_zero(ya);
        const bool b_inf = !pr.pair || (xb0 && Fp::is_zero(yb));
        if (b_inf) cls = a_inf ? AFF_ZERO : AFF_COPY_A;
        else if (a_inf) cls = AFF_COPY_B;
        else if (Fp::eq(xa, xb)) cls = (Fp::eq(ya, yb) && !Fp::is_zero(ya)) ? AFF_DBL : AFF_ZERO;
        else cls = AFF_ADD;
        if (cls == AFF_DBL) Fp::dbl(d, ya);
        else if (cls == AFF_ADD) Fp::sub(d, xb, xa);
        else Fp::set_one(d);
      } else {
        cls = AFF_ADD;
        Fp::sub(d, xb, xa);
      }
      classes[(q - q0) / 21] |= (uint64_t)cls << (3 * ((q - q0) % 21));
      Fp::mul(acc, acc, d);
#pragma unroll
      for (int w = 0; w < N; ++w) scr(q - q0, w) = acc[w];
    }
    cp_async_wait<0>();
    // ---- one inversion: acc = aR -> (aR)^-1 = a^-1 R^-1 (binary GCD), x R^3 R^-1 = a^-1 R
    uint32_t inv[N];
    {
      uint32_t t[N];
      Fp::inv_bingcd(t, acc);
      Fp::mul(inv, t, r3);
    }
    // ---- backward: per output its 1/d, then the addition (full pairs staged)
    auto bwd_stage = [&](uint32_t q, uint32_t& kk, uint32_t* dst) {
      while (__ldg(off_out + kk) > q) --kk;
      const Pair pr = pair_of(q, kk);
      uint32_t sg;
      In::stage(dst, vals, pts, pr.e, true, sg);
      if (pr.pair) In::stage(dst + 2 * N, vals, pts, pr.e + 1, true, sg);
    };
    kn = k;
    bwd_stage(q1 - 1, kn, slot);
    cp_async_commit();
    for (uint32_t q = q1; q-- > q0;) {
      uint32_t* cur = slot + ((q1 - 1 - q) & 1) * PW;
      if (q > q0) bwd_stage(q - 1, kn, slot + ((q1 - q) & 1) * PW);
      cp_async_commit();
      cp_async_wait<1>();
      while (__ldg(off_out + k) > q) --k;
      const Pair pr = pair_of(q, k);
      const uint32_t cls = (uint32_t)(classes[(q - q0) / 21] >> (3 * ((q - q0) % 21))) & 7u;
      const uint32_t sg = (uint32_t)(signs >> (2 * (q - q0)));
      uint32_t xa[N], ya[N], xb[N], yb[N], dinv[N];
#pragma unroll
      for (int w = 0; w < N; ++w) {
        xa[w] = cur[w];
        ya[w] = cur[N + w];
        xb[w] = pr.pair ? cur[2 * N + w] : 0u;
        yb[w] = pr.pair ? cur[3 * N + w] : 0u;
      }
      if constexpr (FIRST) {
        if ((sg & 1u) && !(Fp::is_zero(xa) && Fp::is_zero(ya))) Fp::neg(ya, ya);
        if ((sg & 2u) && !(Fp::is_zero(xb) && Fp::is_zero(yb))) Fp::neg(yb, yb);
      }
      if (q > q0) {
        uint32_t d[N], pre[N];
        if (cls == AFF_ADD) Fp::sub(d, xb, xa);
        else if (cls == AFF_DBL) Fp::dbl(d, ya);
        else Fp::set_one(d);
#pragma unroll
        for (int w = 0; w < N; ++w) pre[w] = scr(q - q0 - 1, w);
        Fp::mul(dinv, inv, pre);
        Fp::mul(inv, inv, d);
      } else {
        Fp::copy(dinv, inv);
      }
      // a bucket with one output is final (XYZZ, ZZ = ZZZ = 1; O: ZZ = 0)
      const uint32_t ko = __ldg(off_out + k);
      const bool fin = __ldg(off_out + k + 1) - ko == 1;
      uint32_t* o = fin ? nullptr : out + (size_t)(__ldg(off_next + k) + (q - ko)) * 2 * N;
      uint32_t* bk = buckets + (size_t)k * 4 * N;
      auto emit = [&](const uint32_t* x, const uint32_t* y, bool inf) {
        if (fin) {
          typename EC<C>::Xyzz P;
          if (inf) EC<C>::set_inf(P);
          else EC<C>::from_affine(P, x, y);
          EC<C>::store(bk, P);
        } else {
          EC<C>::st(o, x);
          EC<C>::st(o + N, y);
        }
      };
      if (cls == AFF_ADD || cls == AFF_DBL) {
        uint32_t lam[N], num[N], x3[N], y3[N];
        if (cls == AFF_ADD) Fp::sub(num, yb, ya);
        else EC<C>::tangent_m(num, xa, nullptr);     // 3 x^2 + a
        Fp::mul(lam, num, dinv);
        Fp::sqr(x3, lam);
        Fp::sub(x3, x3, xa);
        Fp::sub(x3, x3, cls == AFF_ADD ? xb : xa);
        Fp::sub(y3, xa, x3);
        Fp::mul(y3, lam, y3);
        Fp::sub(y3, y3, ya);
        emit(x3, y3, false);
      } else if (cls == AFF_COPY_A) {
        emit(xa, ya, false);
      } else if (cls == AFF_COPY_B) {
        emit(xb, yb, false);
      } else {                                   // O: (0, 0) in a level array
        Fp::set_zero(xa);
        emit(xa, xa, true);
      }
    }
    cp_async_wait<0>();
  }
}

}  // namespace gzkp
