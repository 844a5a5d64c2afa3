// field.cuh -- multi-limb Montgomery arithmetic over F_p on 32-bit IMAD carry chains.
//
// The paper's finite-field library (§4.3) multiplies big
// integers with "modular multiplications [52]" (Montgomery) on
// 64-bit words split across cooperating threads, plus a DFP/FP64 path.  On
// sm_100 there is no 64-bit integer multiplier: the native unit is the 32-bit
// IMAD (lo / hi halves, with hardware carry-in/out), so one thread holds one
// element as N little-endian u32 limbs in registers (N = 8 / 12 / 24) and the
// product uses the CIOS schedule with the multiplicand split into even and odd
// limbs: a[2j]*b_i lands on limb pairs (2j, 2j+1) and a[2j+1]*b_i on
// (2j+1, 2j+2), so each half is ONE unbroken mad.lo.cc / madc.hi.cc chain.
// Two independent chains per row give the scheduler ILP.  The accumulators swap
// roles each row so the shift by one limb costs no moves
// (tools/emulate_mont.py checks the sequence carry-exactly).
//
// Cost: mont_mul = N(4N+1) IMAD (264 / 588 / 2328 for N = 8 / 12 / 24).
// Values are kept fully reduced in [0, p): the group law's equality tests
// (madd's U2 == X1) need canonical representatives.
#pragma once
#include <cstdint>

#ifndef GZKP_MUL_SOS
#define GZKP_MUL_SOS 0         // 1: separated-operand-scanning products everywhere (experiment)
#endif

#ifndef GZKP_MUL_KARATSUBA
#define GZKP_MUL_KARATSUBA 0   // 1: one-level Karatsuba products (N % 4 == 0; measured slower, see mul_kara)
#endif

namespace gzkp {

#define GZ_DEV __device__ __forceinline__

// ---------------------------------------------------------------- PTX glue
// Each helper is one instruction; the carry flag (CC) flows between
// consecutive asm volatile statements exactly as written.
GZ_DEV uint32_t mul_lo(uint32_t a, uint32_t b) { uint32_t r; asm("mul.lo.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b)); return r; }
GZ_DEV uint32_t mul_hi(uint32_t a, uint32_t b) { uint32_t r; asm("mul.hi.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b)); return r; }

#define MAD_LO_CC(d, a, b, c)   asm volatile("mad.lo.cc.u32 %0, %1, %2, %3;"  : "=r"(d) : "r"(a), "r"(b), "r"(c))
#define MADC_LO_CC(d, a, b, c)  asm volatile("madc.lo.cc.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c))
#define MADC_HI_CC(d, a, b, c)  asm volatile("madc.hi.cc.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c))
#define MADC_HI(d, a, b, c)     asm volatile("madc.hi.u32 %0, %1, %2, %3;"    : "=r"(d) : "r"(a), "r"(b), "r"(c))
#define ADD_CC(d, a, b)         asm volatile("add.cc.u32 %0, %1, %2;"  : "=r"(d) : "r"(a), "r"(b))
#define ADDC_CC(d, a, b)        asm volatile("addc.cc.u32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b))
#define ADDC(d, a, b)           asm volatile("addc.u32 %0, %1, %2;"    : "=r"(d) : "r"(a), "r"(b))
#define SUB_CC(d, a, b)         asm volatile("sub.cc.u32 %0, %1, %2;"  : "=r"(d) : "r"(a), "r"(b))
#define SUBC_CC(d, a, b)        asm volatile("subc.cc.u32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b))
#define SUBC(d, a, b)           asm volatile("subc.u32 %0, %1, %2;"    : "=r"(d) : "r"(a), "r"(b))

// ------------------------------------------------------- F_p element ops
// All functions take/return arrays of C::N u32 limbs (registers after unroll).

template <class C>
struct F {
  static constexpr int N = C::N;

  GZ_DEV static void copy(uint32_t r[N], const uint32_t a[N]) {
#pragma unroll
    for (int i = 0; i < N; ++i) r[i] = a[i];
  }
  GZ_DEV static void set_zero(uint32_t r[N]) {
#pragma unroll
    for (int i = 0; i < N; ++i) r[i] = 0;
  }
  GZ_DEV static void set_one(uint32_t r[N]) {   // Montgomery 1 = R mod p
#pragma unroll
    for (int i = 0; i < N; ++i) r[i] = C::ONE(i);
  }
  GZ_DEV static bool is_zero(const uint32_t a[N]) {
    uint32_t t = a[0];
#pragma unroll
    for (int i = 1; i < N; ++i) t |= a[i];
    return t == 0;
  }
  GZ_DEV static bool eq(const uint32_t a[N], const uint32_t b[N]) {
    uint32_t t = a[0] ^ b[0];
#pragma unroll
    for (int i = 1; i < N; ++i) t |= a[i] ^ b[i];
    return t == 0;
  }

  // r = a - p if a >= p (a < 2p, and a fits in N limbs: p has spare bits)
  GZ_DEV static void reduce_once(uint32_t a[N]) {
    uint32_t t[N], borrow;
    SUB_CC(t[0], a[0], C::P(0));
#pragma unroll
    for (int i = 1; i < N; ++i) SUBC_CC(t[i], a[i], C::P(i));
    SUBC(borrow, 0u, 0u);          // 0 if a >= p, 0xffffffff otherwise
#pragma unroll
    for (int i = 0; i < N; ++i) a[i] = borrow ? a[i] : t[i];
  }

  // r = a + b mod p
  GZ_DEV static void add(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) {
    ADD_CC(r[0], a[0], b[0]);
#pragma unroll
    for (int i = 1; i < N - 1; ++i) ADDC_CC(r[i], a[i], b[i]);
    ADDC(r[N - 1], a[N - 1], b[N - 1]);   // no overflow: p < 2^(32N - 1)
    reduce_once(r);
  }

  // r = a - b mod p
  GZ_DEV static void sub(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) {
    uint32_t borrow, t[N];
    SUB_CC(r[0], a[0], b[0]);
#pragma unroll
    for (int i = 1; i < N; ++i) SUBC_CC(r[i], a[i], b[i]);
    SUBC(borrow, 0u, 0u);          // 0xffffffff if a < b
#pragma unroll
    for (int i = 0; i < N; ++i) t[i] = C::P(i) & borrow;
    ADD_CC(r[0], r[0], t[0]);
#pragma unroll
    for (int i = 1; i < N - 1; ++i) ADDC_CC(r[i], r[i], t[i]);
    ADDC(r[N - 1], r[N - 1], t[N - 1]);
  }

  GZ_DEV static void dbl(uint32_t r[N], const uint32_t a[N]) { add(r, a, a); }

  // r = -a mod p
  GZ_DEV static void neg(uint32_t r[N], const uint32_t a[N]) {
    uint32_t z[N];
    set_zero(z);
    sub(r, z, a);
  }

  // ---- Montgomery product r = a * b * R^-1 mod p (even/odd CIOS) ----
  // E holds limbs at positions 0..N-1, O at positions 1..N (one limb up).
  // For N >= 24 (MNT4-753) the product is an out-of-line call: a fully inlined
  // 2328-IMAD body at every call site makes the kernels too large to compile.
  GZ_DEV static void mul(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) {
    if constexpr (N >= 24) mul_ni(r, a, b);
    else mul_inline(r, a, b);
  }
  __device__ __noinline__ static void mul_ni(uint32_t* r, const uint32_t* a, const uint32_t* b) {
    uint32_t x[N], y[N], z[N];
#pragma unroll
    for (int i = 0; i < N; ++i) { x[i] = a[i]; y[i] = b[i]; }
    mul_inline(z, x, y);
#pragma unroll
    for (int i = 0; i < N; ++i) r[i] = z[i];
  }
  // separated operand scanning: the full product (prod<N>, parity-split
  // chains) then sos_reduce; the same 2N^2 + N(2N + 1) IMAD as CIOS, a
  // different dependency structure (GZKP_MUL_SOS experiment)
  GZ_DEV static void mul_sos(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) {
    uint32_t T[2 * N];
    prod<N>(T, a, b);
    sos_reduce(r, T);
  }
  GZ_DEV static void mul_inline(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) {
#if GZKP_MUL_SOS
    if constexpr (N >= 8) {
      mul_sos(r, a, b);
      return;
    }
#endif
#if GZKP_MUL_KARATSUBA
    if constexpr (N >= 8 && N % 4 == 0) {
      mul_kara(r, a, b);
      return;
    }
#endif
    mul_cios(r, a, b);
  }
  GZ_DEV static void mul_cios(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) {
    uint32_t e[N], o[N];
    uint32_t* E = e;
    uint32_t* O = o;
    // row 0: plain products
    {
      const uint32_t bi = b[0];
#pragma unroll
      for (int j = 0; j < N; j += 2) {
        E[j] = mul_lo(a[j], bi);
        E[j + 1] = mul_hi(a[j], bi);
        O[j] = mul_lo(a[j + 1], bi);
        O[j + 1] = mul_hi(a[j + 1], bi);
      }
      redc_step(E, O);
    }
#pragma unroll
    for (int i = 1; i < N; ++i) {
      uint32_t* t = E; E = O; O = t;      // roles swap (compile-time after unroll)
      const uint32_t bi = b[i];
      // E[0] += O_old_shifted[1]; carry flows into the O chain at position 1
      ADD_CC(E[0], E[0], O[1]);
      // O_new[k] = a_odd * bi + O_old[k + 2]   (the one-limb shift)
#pragma unroll
      for (int j = 0; j < N - 2; j += 2) {
        MADC_LO_CC(O[j], a[j + 1], bi, O[j + 2]);
        MADC_HI_CC(O[j + 1], a[j + 1], bi, O[j + 3]);
      }
      MADC_LO_CC(O[N - 2], a[N - 1], bi, 0u);
      MADC_HI(O[N - 1], a[N - 1], bi, 0u);
      // E += a_even * bi, top carry into O[N-1] (position N)
      MAD_LO_CC(E[0], a[0], bi, E[0]);
      MADC_HI_CC(E[1], a[0], bi, E[1]);
#pragma unroll
      for (int j = 2; j < N; j += 2) {
        MADC_LO_CC(E[j], a[j], bi, E[j]);
        MADC_HI_CC(E[j + 1], a[j], bi, E[j + 1]);
      }
      ADDC(O[N - 1], O[N - 1], 0u);
      redc_step(E, O);
    }
    // r = (E >> 32) + O
    ADD_CC(r[0], E[1], O[0]);
#pragma unroll
    for (int k = 1; k < N - 1; ++k) ADDC_CC(r[k], E[k + 1], O[k]);
    ADDC(r[N - 1], O[N - 1], 0u);
    reduce_once(r);
  }

  // ---- two independent products with their rows interleaved (mul2): each
  // row of the even/odd CIOS is a self-contained carry sequence (its chains
  // start with a .cc op and end in a consuming op), so rows of two products
  // may alternate in the PTX stream; ptxas then has four independent carry
  // chains to overlap instead of two.  r1 may alias a1 / b1 (and r2 a2 / b2):
  // results are written after their last read.
  GZ_DEV static void cios_row0(uint32_t* E, uint32_t* O, const uint32_t a[N], uint32_t bi) {
#pragma unroll
    for (int j = 0; j < N; j += 2) {
      E[j] = mul_lo(a[j], bi);
      E[j + 1] = mul_hi(a[j], bi);
      O[j] = mul_lo(a[j + 1], bi);
      O[j + 1] = mul_hi(a[j + 1], bi);
    }
    redc_step(E, O);
  }
  GZ_DEV static void cios_row(uint32_t* E, uint32_t* O, const uint32_t a[N], uint32_t bi) {
    ADD_CC(E[0], E[0], O[1]);
#pragma unroll
    for (int j = 0; j < N - 2; j += 2) {
      MADC_LO_CC(O[j], a[j + 1], bi, O[j + 2]);
      MADC_HI_CC(O[j + 1], a[j + 1], bi, O[j + 3]);
    }
    MADC_LO_CC(O[N - 2], a[N - 1], bi, 0u);
    MADC_HI(O[N - 1], a[N - 1], bi, 0u);
    MAD_LO_CC(E[0], a[0], bi, E[0]);
    MADC_HI_CC(E[1], a[0], bi, E[1]);
#pragma unroll
    for (int j = 2; j < N; j += 2) {
      MADC_LO_CC(E[j], a[j], bi, E[j]);
      MADC_HI_CC(E[j + 1], a[j], bi, E[j + 1]);
    }
    ADDC(O[N - 1], O[N - 1], 0u);
    redc_step(E, O);
  }
  GZ_DEV static void cios_final(uint32_t r[N], const uint32_t* E, const uint32_t* O) {
    ADD_CC(r[0], E[1], O[0]);
#pragma unroll
    for (int k = 1; k < N - 1; ++k) ADDC_CC(r[k], E[k + 1], O[k]);
    ADDC(r[N - 1], O[N - 1], 0u);
    reduce_once(r);
  }
  GZ_DEV static void mul2(uint32_t r1[N], const uint32_t a1[N], const uint32_t b1[N], uint32_t r2[N],
                          const uint32_t a2[N], const uint32_t b2[N]) {
    uint32_t e1[N], o1[N], e2[N], o2[N];
    uint32_t *E1 = e1, *O1 = o1, *E2 = e2, *O2 = o2;
    cios_row0(E1, O1, a1, b1[0]);
    cios_row0(E2, O2, a2, b2[0]);
#pragma unroll
    for (int i = 1; i < N; ++i) {
      { uint32_t* t = E1; E1 = O1; O1 = t; }
      { uint32_t* t = E2; E2 = O2; O2 = t; }
      cios_row(E1, O1, a1, b1[i]);
      cios_row(E2, O2, a2, b2[i]);
    }
    uint32_t s1[N];
    cios_final(s1, E1, O1);
    cios_final(r2, E2, O2);
#pragma unroll
    for (int i = 0; i < N; ++i) r1[i] = s1[i];
  }

  // m = E[0] * n0; E += m * p_even; O += m * p_odd  (makes E[0] == 0)
  GZ_DEV static void redc_step(uint32_t* E, uint32_t* O) {
    const uint32_t m = E[0] * C::N0;
    MAD_LO_CC(O[0], C::P(1), m, O[0]);
    MADC_HI_CC(O[1], C::P(1), m, O[1]);
#pragma unroll
    for (int j = 2; j < N - 2; j += 2) {
      MADC_LO_CC(O[j], C::P(j + 1), m, O[j]);
      MADC_HI_CC(O[j + 1], C::P(j + 1), m, O[j + 1]);
    }
    if (N > 2) {
      MADC_LO_CC(O[N - 2], C::P(N - 1), m, O[N - 2]);
      MADC_HI(O[N - 1], C::P(N - 1), m, O[N - 1]);
    }
    MAD_LO_CC(E[0], C::P(0), m, E[0]);
    MADC_HI_CC(E[1], C::P(0), m, E[1]);
#pragma unroll
    for (int j = 2; j < N; j += 2) {
      MADC_LO_CC(E[j], C::P(j), m, E[j]);
      MADC_HI_CC(E[j + 1], C::P(j), m, E[j + 1]);
    }
    ADDC(O[N - 1], O[N - 1], 0u);
  }

  // ---- Montgomery square r = a^2 R^-1 mod p (tools/emulate_sqr.py checks the
  // sequence carry-exactly).  Off-diagonal products once (triangular rows,
  // split by column parity into two accumulators so each row is two unbroken
  // carry chains), doubled by a funnel shift, plus the diagonal; then a
  // separated-operand (SOS) reduction whose chain carries are deferred into
  // C[N..2N+1] (they only ever land at positions >= N, so the m_i = T[i] n0
  // sequence never needs them).  N(N-1)/2 + N + N^2 + N IMAD(.WIDE) against
  // the product's 2N^2 + N: 234 vs 300 for N = 12.
  // (MNT4-753: the out-of-line square measured slower than the out-of-line
  // product, 85 vs 78 ms accumulation at 2^20, so N >= 24 squares via mul.)
  GZ_DEV static void sqr(uint32_t r[N], const uint32_t a[N]) {
    if constexpr (N >= 24) mul(r, a, a);
    else sqr_inline(r, a);
  }
  __device__ __noinline__ static void sqr_ni(uint32_t* r, const uint32_t* a) {
    uint32_t x[N], z[N];
#pragma unroll
    for (int i = 0; i < N; ++i) x[i] = a[i];
    sqr_inline(z, x);
#pragma unroll
    for (int i = 0; i < N; ++i) r[i] = z[i];
  }
  GZ_DEV static void sqr_inline(uint32_t r[N], const uint32_t a[N]) {
    uint32_t EV[2 * N + 2], OD[2 * N + 2];
#pragma unroll
    for (int k = 0; k < 2 * N + 2; ++k) { EV[k] = 0; OD[k] = 0; }
    // triangular product: row i, a_i * a_{i+1+k} at position 2i+1+k
#pragma unroll
    for (int i = 0; i < N - 1; ++i) {
      // k even -> OD (pairs start at odd positions)
#pragma unroll
      for (int k = 0; k < N - 1 - i; k += 2) {
        const int pos = 2 * i + 1 + k;
        if (k == 0) { MAD_LO_CC(OD[pos], a[i], a[i + 1 + k], OD[pos]); }
        else { MADC_LO_CC(OD[pos], a[i], a[i + 1 + k], OD[pos]); }
        MADC_HI_CC(OD[pos + 1], a[i], a[i + 1 + k], OD[pos + 1]);
      }
      {
        const int kl = ((N - 2 - i) / 2) * 2;           // last even k
        ADDC(OD[2 * i + 3 + kl], OD[2 * i + 3 + kl], 0u);
      }
      // k odd -> EV (pairs start at even positions)
      if (N - 1 - i > 1) {
#pragma unroll
        for (int k = 1; k < N - 1 - i; k += 2) {
          const int pos = 2 * i + 1 + k;
          if (k == 1) { MAD_LO_CC(EV[pos], a[i], a[i + 1 + k], EV[pos]); }
          else { MADC_LO_CC(EV[pos], a[i], a[i + 1 + k], EV[pos]); }
          MADC_HI_CC(EV[pos + 1], a[i], a[i + 1 + k], EV[pos + 1]);
        }
        const int kl = ((N - 3 - i) / 2) * 2 + 1;       // last odd k
        ADDC(EV[2 * i + 3 + kl], EV[2 * i + 3 + kl], 0u);
      }
    }
    // V = OD + EV (V[2N] == 0), T = 2 V
    uint32_t T[2 * N];
    ADD_CC(EV[0], OD[0], EV[0]);
#pragma unroll
    for (int k = 1; k < 2 * N - 1; ++k) ADDC_CC(EV[k], OD[k], EV[k]);
    ADDC(EV[2 * N - 1], OD[2 * N - 1], EV[2 * N - 1]);
#pragma unroll
    for (int k = 2 * N - 1; k > 0; --k) T[k] = __funnelshift_l(EV[k - 1], EV[k], 1);
    T[0] = EV[0] << 1;
    // + diagonal a_i^2 at (2i, 2i+1)
    MAD_LO_CC(T[0], a[0], a[0], T[0]);
    MADC_HI_CC(T[1], a[0], a[0], T[1]);
#pragma unroll
    for (int i = 1; i < N - 1; ++i) {
      MADC_LO_CC(T[2 * i], a[i], a[i], T[2 * i]);
      MADC_HI_CC(T[2 * i + 1], a[i], a[i], T[2 * i + 1]);
    }
    MADC_LO_CC(T[2 * N - 2], a[N - 1], a[N - 1], T[2 * N - 2]);
    MADC_HI(T[2 * N - 1], a[N - 1], a[N - 1], T[2 * N - 1]);
    sos_reduce(r, T);
  }

  // ---- Montgomery reduction of a 2N-limb T < p R (separated-operand
  // scanning): r = T R^-1 mod p.  The row chains' carries are deferred into
  // Cc[pos - N] (they only ever land at positions >= N, so the m_i = T[i] n0
  // sequence never needs them).  N (2N + 1) IMAD(.WIDE).
  GZ_DEV static void sos_reduce(uint32_t r[N], uint32_t T[2 * N]) {
    uint32_t Cc[N + 2];
#pragma unroll
    for (int k = 0; k < N + 2; ++k) Cc[k] = 0;
#pragma unroll
    for (int i = 0; i < N; ++i) {
      const uint32_t m = T[i] * C::N0;
#pragma unroll
      for (int par = 0; par < 2; ++par) {
#pragma unroll
        for (int k = 0; k < N / 2; ++k) {
          const int j = 2 * k + par, pos = i + j;
          if (k == 0) { MAD_LO_CC(T[pos], C::P(j), m, T[pos]); }
          else { MADC_LO_CC(T[pos], C::P(j), m, T[pos]); }
          if (pos + 1 < 2 * N) { MADC_HI_CC(T[pos + 1], C::P(j), m, T[pos + 1]); }
        }
        ADDC(Cc[i + par], Cc[i + par], 0u);
      }
    }
    ADD_CC(r[0], T[N], Cc[0]);
#pragma unroll
    for (int k = 1; k < N - 1; ++k) ADDC_CC(r[k], T[N + k], Cc[k]);
    ADDC(r[N - 1], T[2 * N - 1], Cc[N - 1]);
    reduce_once(r);
  }

  // ---- schoolbook H x H -> 2H product z = x y.  Row i adds x_i y_k at
  // position i + k; the products of one row are split by the parity of k into
  // two unbroken mad.lo.cc / madc.hi.cc chains that land in the accumulator of
  // their position's parity (EV / OD), and each accumulator stays below the
  // running partial product, so a chain's final carry is absorbed by the limb
  // just above it.  z = EV + OD.  2 H^2 IMAD(.WIDE).
  template <int H>
  GZ_DEV static void prod(uint32_t z[2 * H], const uint32_t x[H], const uint32_t y[H]) {
    uint32_t EV[2 * H + 2], OD[2 * H + 2];
#pragma unroll
    for (int k = 0; k < 2 * H + 2; ++k) { EV[k] = 0; OD[k] = 0; }
#pragma unroll
    for (int i = 0; i < H; ++i) {
      uint32_t* A = (i & 1) ? OD : EV;      // positions i + even k
      uint32_t* B = (i & 1) ? EV : OD;      // positions i + odd k
#pragma unroll
      for (int k = 0; k < H; k += 2) {
        if (k == 0) { MAD_LO_CC(A[i + k], x[i], y[k], A[i + k]); }
        else { MADC_LO_CC(A[i + k], x[i], y[k], A[i + k]); }
        MADC_HI_CC(A[i + k + 1], x[i], y[k], A[i + k + 1]);
      }
      ADDC(A[i + H], A[i + H], 0u);
#pragma unroll
      for (int k = 1; k < H; k += 2) {
        if (k == 1) { MAD_LO_CC(B[i + k], x[i], y[k], B[i + k]); }
        else { MADC_LO_CC(B[i + k], x[i], y[k], B[i + k]); }
        MADC_HI_CC(B[i + k + 1], x[i], y[k], B[i + k + 1]);
      }
      ADDC(B[i + H + 1], B[i + H + 1], 0u);
    }
    ADD_CC(z[0], EV[0], OD[0]);
#pragma unroll
    for (int k = 1; k < 2 * H - 1; ++k) ADDC_CC(z[k], EV[k], OD[k]);
    ADDC(z[2 * H - 1], EV[2 * H - 1], OD[2 * H - 1]);
  }

  // ---- sum of two Montgomery products with ONE reduction:
  //   r = (a b + c d) R^-1 mod p.
  // Both 2N-limb products (prod<N>, 2 N^2 IMAD each) are added, then one SOS
  // reduction (N (2N + 1)): 876 IMAD for N = 12 instead of 2 x 588.  The
  // group law's Y3 = R (Q - X3) - Y1 PPP is such a sum (with -Y1 = p - Y1).
  // Bound: a, b, c, d < p gives T < 2 p^2 < p R (p < R / 2 for every curve
  // here), which is sos_reduce's precondition (result < 2p, one subtraction).
  // N >= 24 (MNT4-753) keeps its out-of-line products.
  GZ_DEV static void mul_sum(uint32_t r[N], const uint32_t a[N], const uint32_t b[N], const uint32_t c[N],
                             const uint32_t d[N]) {
    if constexpr (N >= 24) {
      uint32_t t[N];
      mul(t, c, d);
      mul(r, a, b);
      add(r, r, t);
    } else {
      uint32_t T[2 * N], U[2 * N];
      prod<N>(T, a, b);
      prod<N>(U, c, d);
      ADD_CC(T[0], T[0], U[0]);
#pragma unroll
      for (int k = 1; k < 2 * N - 1; ++k) ADDC_CC(T[k], T[k], U[k]);
      ADDC(T[2 * N - 1], T[2 * N - 1], U[2 * N - 1]);
      sos_reduce(r, T);
    }
  }

  // ---- Montgomery product with a one-level Karatsuba product (H = N/2):
  //   a b = z0 + z1 2^(32H) + z2 2^(64H),  z0 = a0 b0,  z2 = a1 b1,
  //   z1 = (a0 + a1)(b0 + b1) - z0 - z2 = a0 b1 + a1 b0  (2H + 1 limbs),
  // where the H-limb sums carry one bit each (ca, cb), applied as masked
  // additions.  3 x 2 H^2 = 1.5 N^2 IMAD for the product instead of 2 N^2,
  // then the SOS reduction: 3.5 N^2 + N in all (504 vs 588 for N = 12,
  // 232 vs 264 for N = 8); the extra work is IADD3/LOP3 on the ALU pipe.
  GZ_DEV static void mul_kara(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) {
    constexpr int H = N / 2;
    uint32_t sa[H], sb[H], ca, cb;
    ADD_CC(sa[0], a[0], a[H]);
#pragma unroll
    for (int k = 1; k < H; ++k) ADDC_CC(sa[k], a[k], a[H + k]);
    ADDC(ca, 0u, 0u);
    ADD_CC(sb[0], b[0], b[H]);
#pragma unroll
    for (int k = 1; k < H; ++k) ADDC_CC(sb[k], b[k], b[H + k]);
    ADDC(cb, 0u, 0u);
    uint32_t T[2 * N], M[2 * H + 1];
    prod<H>(T, a, b);                       // z0 -> T[0, 2H)
    prod<H>(T + 2 * H, a + H, b + H);       // z2 -> T[2H, 4H)
    prod<H>(M, sa, sb);
    M[2 * H] = ca & cb;
    {
      const uint32_t ma = 0u - ca, mb = 0u - cb;
      ADD_CC(M[H], M[H], sb[0] & ma);
#pragma unroll
      for (int k = 1; k < H; ++k) ADDC_CC(M[H + k], M[H + k], sb[k] & ma);
      ADDC(M[2 * H], M[2 * H], 0u);
      ADD_CC(M[H], M[H], sa[0] & mb);
#pragma unroll
      for (int k = 1; k < H; ++k) ADDC_CC(M[H + k], M[H + k], sa[k] & mb);
      ADDC(M[2 * H], M[2 * H], 0u);
    }
    SUB_CC(M[0], M[0], T[0]);
#pragma unroll
    for (int k = 1; k < 2 * H; ++k) SUBC_CC(M[k], M[k], T[k]);
    SUBC(M[2 * H], M[2 * H], 0u);
    SUB_CC(M[0], M[0], T[2 * H]);
#pragma unroll
    for (int k = 1; k < 2 * H; ++k) SUBC_CC(M[k], M[k], T[2 * H + k]);
    SUBC(M[2 * H], M[2 * H], 0u);
    // T[H, 3H] += M, carry through T[4H - 1]
    ADD_CC(T[H], T[H], M[0]);
#pragma unroll
    for (int k = 1; k <= 2 * H; ++k) ADDC_CC(T[H + k], T[H + k], M[k]);
#pragma unroll
    for (int k = 3 * H + 1; k < 4 * H - 1; ++k) ADDC_CC(T[k], T[k], 0u);
    ADDC(T[4 * H - 1], T[4 * H - 1], 0u);
    sos_reduce(r, T);
  }

  GZ_DEV static void to_mont(uint32_t r[N], const uint32_t a[N]) {
    uint32_t r2[N];
#pragma unroll
    for (int i = 0; i < N; ++i) r2[i] = C::R2(i);
    mul(r, a, r2);
  }
  GZ_DEV static void from_mont(uint32_t r[N], const uint32_t a[N]) {
    uint32_t one[N];
    set_zero(one);
    one[0] = 1;
    mul(r, a, one);
  }

  // ---- inverse of a CANONICAL (non-Montgomery) value by binary extended
  // Euclid; a != 0.  Latency ~2*bits iterations of N-limb shifts/subtracts,
  // far shorter than Fermat's ~1.5*bits serial multiplications.
  GZ_DEV static void shr1(uint32_t x[N], uint32_t top) {
#pragma unroll
    for (int i = 0; i < N - 1; ++i) x[i] = __funnelshift_r(x[i], x[i + 1], 1);
    x[N - 1] = (x[N - 1] >> 1) | (top << 31);
  }
  GZ_DEV static void half_mod(uint32_t x[N]) {   // x/2 mod p for x in [0, p)
    if (x[0] & 1) {
      uint32_t c;
      ADD_CC(x[0], x[0], C::P(0));
#pragma unroll
      for (int i = 1; i < N; ++i) ADDC_CC(x[i], x[i], C::P(i));
      ADDC(c, 0u, 0u);
      shr1(x, c);
    } else {
      shr1(x, 0);
    }
  }
  GZ_DEV static bool is_one_int(const uint32_t a[N]) {
    uint32_t t = a[0] ^ 1u;
#pragma unroll
    for (int i = 1; i < N; ++i) t |= a[i];
    return t == 0;
  }
  // returns borrow (a < b) and r = a - b (integer)
  GZ_DEV static bool sub_int(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) {
    uint32_t borrow;
    SUB_CC(r[0], a[0], b[0]);
#pragma unroll
    for (int i = 1; i < N; ++i) SUBC_CC(r[i], a[i], b[i]);
    SUBC(borrow, 0u, 0u);
    return borrow != 0;
  }
  GZ_DEV static void inv_canonical(uint32_t r[N], const uint32_t a[N]) {
    uint32_t u[N], v[N], x1[N], x2[N], t[N];
    copy(u, a);
#pragma unroll
    for (int i = 0; i < N; ++i) v[i] = C::P(i);
    set_zero(x1);
    x1[0] = 1;
    set_zero(x2);
    if (is_zero(a)) { set_zero(r); return; }   // no inverse; never loop forever
    // each outer pass strips >= 1 bit from u or v: <= 2 * 32N passes
    for (int guard = 0; guard < 64 * N + 8 && !is_one_int(u) && !is_one_int(v); ++guard) {
      while (!(u[0] & 1)) { shr1(u, 0); half_mod(x1); }
      while (!(v[0] & 1)) { shr1(v, 0); half_mod(x2); }
      if (!sub_int(t, u, v)) {       // u >= v
        copy(u, t);
        sub(x1, x1, x2);
      } else {
        sub_int(v, v, u);
        sub(x2, x2, x1);
      }
    }
    if (is_one_int(u)) copy(r, x1); else copy(r, x2);
  }
  // ---- constant-time inverse by the optimised binary GCD (Pornin, "Optimized
  // Binary GCD for Modular Inversion", 2020; tools/emulate_bingcd.py is the
  // bit-exact model): r = x^-1 mod p for a canonical x (x = 0 gives 0).
  // T = ceil((2 bits(p) - 1) / 31) outer iterations; each runs 31 divsteps on
  // 64-bit approximations of (a, b) (31 low + 33 top bits), then applies the
  // accumulated 2x2 matrix (|f|, |g| <= 2^31) to the full values and, with a
  // Montgomery division by 2^31, to the Bezout coefficients (u, v), keeping
  // a = u x and b = v x (mod p) exact.  No data-dependent branch: every lane
  // of a warp runs the same instruction stream, so a warp inverts 32 values
  // at the cost of one (the batch-affine accumulation relies on this).
  static constexpr int BG_OUTER = (2 * C::P_BITS - 1 + 30) / 31;
  static constexpr int BG_L = N + 2;          // signed working width (limbs)

  // r = |m| * a  (N + 1 limbs) for a u32 magnitude
  GZ_DEV static void mul_small(uint32_t r[N + 1], const uint32_t a[N], uint32_t m) {
    r[0] = a[0] * m;
    uint32_t t = mul_hi(a[0], m);
#pragma unroll
    for (int i = 1; i < N; ++i) {
      MAD_LO_CC(r[i], a[i], m, t);
      MADC_HI(t, a[i], m, 0u);
    }
    r[N] = t;
  }
  // z = a f + b g, signed, BG_L limbs two's complement (|f|, |g| <= 2^31)
  GZ_DEV static void lincomb(uint32_t z[BG_L], const uint32_t a[N], int64_t f, const uint32_t b[N], int64_t g) {
    uint32_t x[N + 1], y[N + 1];
    const uint32_t fm = (uint32_t)(f < 0 ? -f : f), gm = (uint32_t)(g < 0 ? -g : g);
    const uint32_t fs = f < 0 ? 0xffffffffu : 0u, gs = g < 0 ? 0xffffffffu : 0u;
    mul_small(x, a, fm);
    mul_small(y, b, gm);
    // two's complement negation of a magnitude: (x ^ s) + (s & 1)
    uint32_t xs[BG_L], ys[BG_L];
#pragma unroll
    for (int i = 0; i <= N; ++i) { xs[i] = x[i] ^ fs; ys[i] = y[i] ^ gs; }
    xs[N + 1] = fs;
    ys[N + 1] = gs;
    ADD_CC(z[0], xs[0], ys[0]);
#pragma unroll
    for (int i = 1; i < BG_L; ++i) ADDC_CC(z[i], xs[i], ys[i]);
    // + (fs & 1) + (gs & 1): add the two's-complement corrections
    uint32_t corr = (fs & 1u) + (gs & 1u);
    ADD_CC(z[0], z[0], corr);
#pragma unroll
    for (int i = 1; i < BG_L - 1; ++i) ADDC_CC(z[i], z[i], 0u);
    ADDC(z[BG_L - 1], z[BG_L - 1], 0u);
  }
  // arithmetic shift right by 31 of a BG_L-limb signed value, to N + 1 limbs
  GZ_DEV static void sar31(uint32_t r[N + 1], const uint32_t z[BG_L]) {
#pragma unroll
    for (int i = 0; i <= N; ++i) r[i] = __funnelshift_r(z[i], z[i + 1], 31);
  }
  GZ_DEV static void neg_n1(uint32_t r[N + 1], uint32_t s) {   // r = s ? -r : r
#pragma unroll
    for (int i = 0; i <= N; ++i) r[i] ^= s;
    ADD_CC(r[0], r[0], s & 1u);
#pragma unroll
    for (int i = 1; i < N; ++i) ADDC_CC(r[i], r[i], 0u);
    ADDC(r[N], r[N], 0u);
  }
  // r (N + 1 limbs, signed, |r| < 3p)  ->  canonical in [0, p)
  GZ_DEV static void normalize_signed(uint32_t out[N], uint32_t r[N + 1]) {
#pragma unroll
    for (int k = 0; k < 3; ++k) {          // add p while negative
      const uint32_t s = (uint32_t)((int32_t)r[N] >> 31);
      ADD_CC(r[0], r[0], C::P(0) & s);
#pragma unroll
      for (int i = 1; i < N; ++i) ADDC_CC(r[i], r[i], C::P(i) & s);
      ADDC(r[N], r[N], 0u);
    }
#pragma unroll
    for (int k = 0; k < 2; ++k) {          // subtract p while >= p
      uint32_t t[N + 1];
      SUB_CC(t[0], r[0], C::P(0));
#pragma unroll
      for (int i = 1; i < N; ++i) SUBC_CC(t[i], r[i], C::P(i));
      SUBC(t[N], r[N], 0u);
      const uint32_t keep = (uint32_t)((int32_t)t[N] >> 31);   // all ones: r < p
#pragma unroll
      for (int i = 0; i <= N; ++i) r[i] = keep ? r[i] : t[i];
    }
#pragma unroll
    for (int i = 0; i < N; ++i) out[i] = r[i];
  }
  // (u f + v g) / 2^31 mod p, u, v canonical
  GZ_DEV static void bezout_update(uint32_t out[N], const uint32_t u[N], int64_t f, const uint32_t v[N], int64_t g) {
    uint32_t z[BG_L], tp[N + 1];
    lincomb(z, u, f, v, g);
    const uint32_t t = (z[0] * C::N0) & 0x7fffffffu;     // z + t p = 0 mod 2^31
    uint32_t pp[N];
#pragma unroll
    for (int i = 0; i < N; ++i) pp[i] = C::P(i);
    mul_small(tp, pp, t);
    ADD_CC(z[0], z[0], tp[0]);
#pragma unroll
    for (int i = 1; i <= N; ++i) ADDC_CC(z[i], z[i], tp[i]);
    ADDC(z[N + 1], z[N + 1], 0u);
    uint32_t r[N + 1];
    sar31(r, z);
    normalize_signed(out, r);
  }
  __device__ __noinline__ static void inv_bingcd(uint32_t* r, const uint32_t* x) {
    uint32_t a[N], b[N], u[N], v[N];
#pragma unroll
    for (int i = 0; i < N; ++i) { a[i] = x[i]; b[i] = C::P(i); u[i] = 0; v[i] = 0; }
    u[0] = 1;
#pragma unroll 1
    for (int it = 0; it < BG_OUTER; ++it) {
      // n = max(len(a), len(b), 64); window [n - 33, n) of a and b
      uint32_t top = 0;
      int idx = 0;
#pragma unroll
      for (int i = 0; i < N; ++i) {
        const uint32_t o = a[i] | b[i];
        top = o ? o : top;
        idx = o ? i : idx;
      }
      int len = top ? 32 * idx + 32 - __clz(top) : 0;
      len = len < 64 ? 64 : len;
      const int s = len - 33, w = s >> 5, sh = s & 31;
      uint32_t al = 0, am = 0, ah = 0, bl = 0, bm = 0, bh = 0;
#pragma unroll
      for (int i = 0; i < N; ++i) {
        al = i == w ? a[i] : al;     am = i == w + 1 ? a[i] : am;     ah = i == w + 2 ? a[i] : ah;
        bl = i == w ? b[i] : bl;     bm = i == w + 1 ? b[i] : bm;     bh = i == w + 2 ? b[i] : bh;
      }
      const uint32_t at = __funnelshift_r(al, am, sh), atb = __funnelshift_r(am, ah, sh) & 1u;
      const uint32_t bt = __funnelshift_r(bl, bm, sh), btb = __funnelshift_r(bm, bh, sh) & 1u;
      uint64_t xa = ((uint64_t)((atb << 31) | (at >> 1)) << 32) | ((at << 31) | (a[0] & 0x7fffffffu));
      uint64_t xb = ((uint64_t)((btb << 31) | (bt >> 1)) << 32) | ((bt << 31) | (b[0] & 0x7fffffffu));
      int64_t f0 = 1, g0 = 0, f1 = 0, g1 = 1;
#pragma unroll 1
      for (int j = 0; j < 31; ++j) {
        const uint64_t mo = 0ull - (xa & 1ull);                  // a odd
        const uint64_t ms = mo & (0ull - (uint64_t)(xa < xb));  // odd and a < b: swap
        const uint64_t tx = (xa ^ xb) & ms;
        xa ^= tx;
        xb ^= tx;
        const int64_t tf = (f0 ^ f1) & (int64_t)ms, tg = (g0 ^ g1) & (int64_t)ms;
        f0 ^= tf; f1 ^= tf;
        g0 ^= tg; g1 ^= tg;
        xa -= xb & mo;
        f0 -= f1 & (int64_t)mo;
        g0 -= g1 & (int64_t)mo;
        xa >>= 1;
        f1 += f1;
        g1 += g1;
      }
      // (a, b) <- ((a f0 + b g0) / 2^31, (a f1 + b g1) / 2^31), made non-negative
      uint32_t za[BG_L], zb[BG_L], ra[N + 1], rb[N + 1];
      lincomb(za, a, f0, b, g0);
      lincomb(zb, a, f1, b, g1);
      sar31(ra, za);
      sar31(rb, zb);
      const uint32_t sa = (uint32_t)((int32_t)za[BG_L - 1] >> 31), sb = (uint32_t)((int32_t)zb[BG_L - 1] >> 31);
      neg_n1(ra, sa);
      neg_n1(rb, sb);
      f0 = sa ? -f0 : f0;  g0 = sa ? -g0 : g0;
      f1 = sb ? -f1 : f1;  g1 = sb ? -g1 : g1;
#pragma unroll
      for (int i = 0; i < N; ++i) { a[i] = ra[i]; b[i] = rb[i]; }
      uint32_t nu[N], nv[N];
      bezout_update(nu, u, f0, v, g0);
      bezout_update(nv, u, f1, v, g1);
#pragma unroll
      for (int i = 0; i < N; ++i) { u[i] = nu[i]; v[i] = nv[i]; }
    }
    // b = gcd(x, p) = 1 for x != 0: v = x^-1; x = 0 leaves b = p, v = 0
#pragma unroll
    for (int i = 0; i < N; ++i) r[i] = v[i];
  }

  // Montgomery-domain inverse: (aR)^-1 R = from/to conversions around the
  // binary GCD (round 2, tools/tail_bench.cu, one thread: BLS12-381 72.9 ->
  // 61.4 us, MNT4-753 240.8 -> 176.9 us, BN254 39.2 -> 37.5 us against the
  // EEA inv_canonical, identical results; branch-free, so a warp of
  // independent inversions no longer diverges)
  GZ_DEV static void inv(uint32_t r[N], const uint32_t a[N]) {
    uint32_t c[N], ic[N];
    from_mont(c, a);
    inv_bingcd(ic, c);
    to_mont(r, ic);
  }
};

}  // namespace gzkp
