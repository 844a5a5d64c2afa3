// field_dfp.cuh -- Montgomery multiplication on the FP64 pipe ("DFP",
// PAPER.md:263 §4.3: "we choose base D = 2^52 ... convert them to double-
// precision floating point (DFP), followed by applying Dekker's Method ... to
// complete the DFP multiplications and additions without rounding issues").
//
// B200 runs DFMA at the IMAD rate and co-issues the two (tools/microbench.cu:
// 61.8 DFMA + 62.6 IMAD per SM per clock, 60.9 of each when interleaved), so
// products computed here occupy a pipe the IMAD carry chains leave idle.
//
// Representation: L = 2N/3 limbs of 48 bits (radix beta = 2^48), so
// beta^L = 2^(32N) = R: a DFP product of Montgomery operands is the same
// Montgomery product as F<C>::mul and the two can be mixed in one formula.
// Each 48x48-bit product is split exactly with two FMAs (the reading of the
// paper's Dekker step used here): with b' = b * 2^-48,
//     Hb' = fma_rz(a, b', Hb)      Hb biased by 2^52: adds floor(a b / beta) exactly
//     f   = fma(a, b', -(Hb' - Hb)) = frac(a b / beta), exact (48 fraction bits)
// Column sums stay below 2^53 (L <= 8), so every addition is exact.  The
// reduction is SOS with m_i = (c_i mod beta) n0' mod beta computed by the same
// split.  tools/emulate_dfp.py models every operation with exact rationals and
// asserts each exactness claim.  Only L = 8 (BLS12-381) is within the 2^53
// bound; other curves keep the IMAD product.
#pragma once
#include "field.cuh"

namespace gzkp {

template <class C>
struct Dfp {
  static constexpr int N = C::N;
  static constexpr int L = 2 * N / 3;
  static constexpr double TWO52 = 4503599627370496.0;        // 2^52
  static constexpr double BETA = 281474976710656.0;          // 2^48
  static constexpr double INV_BETA = 1.0 / 281474976710656.0;

  // 48-bit limb k of a 32N-bit little-endian u32 value, as an exact double,
  // optionally pre-scaled by 2^-48 (exponent trick: 2^52+x or 2^4+x*2^-48)
  GZ_DEV static double limb(const uint32_t a[N], int k, bool scaled) {
    const int m = k >> 1;
    uint32_t lo, hi16;
    if ((k & 1) == 0) {
      lo = a[3 * m];
      hi16 = a[3 * m + 1] & 0xffffu;
    } else {
      lo = (a[3 * m + 1] >> 16) | (a[3 * m + 2] << 16);
      hi16 = a[3 * m + 2] >> 16;
    }
    if (scaled) return __dsub_rn(__hiloint2double((int)(0x40300000u | hi16), (int)lo), 16.0);
    return __dsub_rn(__hiloint2double((int)(0x43300000u | hi16), (int)lo), TWO52);
  }

  // floor(c / beta) for an exact integer double 0 <= c < 2^53
  GZ_DEV static double floor_beta(double c) { return __dsub_rn(__fma_rz(c, INV_BETA, TWO52), TWO52); }

  // one out-of-line body shared by the call sites of the mixed hot loop (four
  // inlined copies overflowed the instruction cache: ncu stall no_instruction)
  __device__ __noinline__ static void mul_ni(uint32_t* r, const uint32_t* a, const uint32_t* b) {
    uint32_t x[N], y[N], z[N];
#pragma unroll
    for (int i = 0; i < N; ++i) { x[i] = a[i]; y[i] = b[i]; }
    mul(z, x, y);
#pragma unroll
    for (int i = 0; i < N; ++i) r[i] = z[i];
  }

  GZ_DEV static void mul(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) {
    static_assert(L == 8, "DFP product is exact for 8 limbs only");
    double A[L], Bs[L];
#pragma unroll
    for (int k = 0; k < L; ++k) {
      A[k] = limb(a, k, false);
      Bs[k] = limb(b, k, true);
    }
    // ---- product: Hb[k] biased floors, F[k] fractions (column k-1 units of beta)
    double Hb[2 * L + 1], Fr[2 * L + 1];
#pragma unroll
    for (int k = 0; k < 2 * L + 1; ++k) { Hb[k] = TWO52; Fr[k] = 0.0; }
#pragma unroll
    for (int i = 0; i < L; ++i) {
#pragma unroll
      for (int j = 0; j < L; ++j) {
        const int k = i + j + 1;
        const double old = Hb[k];
        Hb[k] = __fma_rz(A[i], Bs[j], old);
        const double d = __dsub_rn(Hb[k], old);
        Fr[k] = __dadd_rn(Fr[k], __fma_rn(A[i], Bs[j], -d));
      }
    }
    // ---- normalise product columns to limbs N_k < beta
    double Nn[2 * L + 1];
    double carry = 0.0;
#pragma unroll
    for (int k = 0; k < 2 * L; ++k) {
      const double c = __dadd_rn(__dadd_rn(__dsub_rn(Hb[k], TWO52), Fr[k + 1] * BETA), carry);
      const double q = floor_beta(c);
      Nn[k] = __fma_rn(q, -BETA, c);
      carry = q;
    }
    Nn[2 * L] = carry;
    // ---- Montgomery reduction (SOS) with fresh accumulators
#pragma unroll
    for (int k = 0; k < 2 * L + 1; ++k) { Hb[k] = TWO52; Fr[k] = 0.0; }
    carry = 0.0;
#pragma unroll
    for (int i = 0; i < L; ++i) {
      const double c = __dadd_rn(__dadd_rn(__dadd_rn(Nn[i], __dsub_rn(Hb[i], TWO52)), Fr[i + 1] * BETA), carry);
      const double q = floor_beta(c);
      const double t = __fma_rn(q, -BETA, c);                       // c mod beta
      const double h = __dsub_rn(__fma_rz(t, C::N048S, TWO52), TWO52);
      const double m = __fma_rn(t, C::N048S, -h) * BETA;           // (t n0) mod beta
#pragma unroll
      for (int j = 0; j < L; ++j) {
        const int k = i + j + 1;
        const double old = Hb[k];
        Hb[k] = __fma_rz(m, C::P48S(j), old);
        const double d = __dsub_rn(Hb[k], old);
        Fr[k] = __dadd_rn(Fr[k], __fma_rn(m, C::P48S(j), -d));
      }
      // column i is now a multiple of beta: exact division
      const double col = __dadd_rn(__dadd_rn(__dadd_rn(Nn[i], __dsub_rn(Hb[i], TWO52)), Fr[i + 1] * BETA), carry);
      carry = col * INV_BETA;
    }
    // ---- result columns L..2L-1 -> 48-bit limbs -> u32 words
    double X[L];
#pragma unroll
    for (int k = L; k < 2 * L; ++k) {
      const double c = __dadd_rn(__dadd_rn(__dadd_rn(Nn[k], __dsub_rn(Hb[k], TWO52)), Fr[k + 1] * BETA), carry);
      const double q = floor_beta(c);
      X[k - L] = __fma_rn(q, -BETA, c);
      carry = q;
    }
    // (the value is < 2p < 2^382, so the top column's carry is 0)
#pragma unroll
    for (int m = 0; m < L / 2; ++m) {
      const double e0 = __dadd_rn(X[2 * m], TWO52), e1 = __dadd_rn(X[2 * m + 1], TWO52);
      const uint32_t lo0 = (uint32_t)__double2loint(e0), hi0 = (uint32_t)__double2hiint(e0) & 0xffffu;
      const uint32_t lo1 = (uint32_t)__double2loint(e1), hi1 = (uint32_t)__double2hiint(e1) & 0xffffu;
      r[3 * m] = lo0;
      r[3 * m + 1] = hi0 | (lo1 << 16);
      r[3 * m + 2] = (lo1 >> 16) | (hi1 << 16);
    }
    F<C>::reduce_once(r);
  }
};

}  // namespace gzkp
