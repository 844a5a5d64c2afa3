// field2.cuh -- F_p^2 = F_p[u]/(u^2 + 1) on top of the F_p Montgomery library,
// for G2 coordinates (GZKP's MSM
// optimisations "apply to both G1 and G2").
//
// An element is c0 + c1 u, stored as 2 NB words c0 || c1 (each NB-limb F_p value
// in Montgomery form, fully reduced).  The product is Karatsuba (3 F_p products
// + 5 additions), the square the complex-squaring form (2 products):
//   (a0 + a1 u)(b0 + b1 u) = (a0 b0 - a1 b1) + ((a0 + a1)(b0 + b1) - a0 b0 - a1 b1) u
//   (a0 + a1 u)^2          = (a0 + a1)(a0 - a1) + 2 a0 a1 u
// (The test oracle multiplies schoolbook instead; the two share no code.)
//
// F2<B> has the same static interface as F<C>, so the group law (ec.cuh) and the
// whole Pippenger pipeline instantiate unchanged for a G2 "curve" struct that
// names its base field (`using Base = ...`, curves.cuh).
#pragma once
#include <type_traits>

#include "field.cuh"

namespace gzkp {

template <class B>
struct F2 {
  using Fp = F<B>;
  static constexpr int NB = B::N;
  static constexpr int N = 2 * NB;

  GZ_DEV static void copy(uint32_t r[N], const uint32_t a[N]) {
#pragma unroll
    for (int i = 0; i < N; ++i) r[i] = a[i];
  }
  GZ_DEV static void set_zero(uint32_t r[N]) {
#pragma unroll
    for (int i = 0; i < N; ++i) r[i] = 0;
  }
  GZ_DEV static void set_one(uint32_t r[N]) {
    Fp::set_one(r);
    Fp::set_zero(r + NB);
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
  GZ_DEV static void add(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) {
    Fp::add(r, a, b);
    Fp::add(r + NB, a + NB, b + NB);
  }
  GZ_DEV static void sub(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) {
    Fp::sub(r, a, b);
    Fp::sub(r + NB, a + NB, b + NB);
  }
  GZ_DEV static void dbl(uint32_t r[N], const uint32_t a[N]) { add(r, a, a); }
  GZ_DEV static void neg(uint32_t r[N], const uint32_t a[N]) {
    Fp::neg(r, a);
    Fp::neg(r + NB, a + NB);
  }

  // every read of a and b precedes the first write of r (r may alias either)
  GZ_DEV static void mul(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) {
    uint32_t t0[NB], t1[NB], sa[NB], sb[NB];
    Fp::add(sa, a, a + NB);
    Fp::add(sb, b, b + NB);
    Fp::mul(t0, a, b);                  // a0 b0
    Fp::mul(t1, a + NB, b + NB);        // a1 b1
    Fp::mul(sa, sa, sb);                // (a0 + a1)(b0 + b1)
    Fp::sub(r, t0, t1);
    Fp::sub(sa, sa, t0);
    Fp::sub(r + NB, sa, t1);
  }
  GZ_DEV static void mul_inline(uint32_t r[N], const uint32_t a[N], const uint32_t b[N]) { mul(r, a, b); }
  // r = a b + c d (no shared reduction over F_p^2: two Karatsuba products)
  GZ_DEV static void mul_sum(uint32_t r[N], const uint32_t a[N], const uint32_t b[N], const uint32_t c[N],
                             const uint32_t d[N]) {
    uint32_t t[N];
    mul(t, c, d);
    mul(r, a, b);
    add(r, r, t);
  }

  GZ_DEV static void sqr(uint32_t r[N], const uint32_t a[N]) {
    uint32_t s[NB], d[NB], m[NB];
    Fp::add(s, a, a + NB);
    Fp::sub(d, a, a + NB);
    Fp::mul(m, a, a + NB);              // a0 a1
    Fp::mul(r, s, d);                   // a0^2 - a1^2
    Fp::add(r + NB, m, m);              // 2 a0 a1
  }

  GZ_DEV static void to_mont(uint32_t r[N], const uint32_t a[N]) {
    Fp::to_mont(r, a);
    Fp::to_mont(r + NB, a + NB);
  }
  GZ_DEV static void from_mont(uint32_t r[N], const uint32_t a[N]) {
    Fp::from_mont(r, a);
    Fp::from_mont(r + NB, a + NB);
  }

  // Montgomery-domain inverse: (a0 - a1 u) / (a0^2 + a1^2), one F_p inversion
  GZ_DEV static void inv(uint32_t r[N], const uint32_t a[N]) {
    uint32_t n0[NB], n1[NB], ni[NB];
    Fp::sqr(n0, a);
    Fp::sqr(n1, a + NB);
    Fp::add(n0, n0, n1);                // the norm, in F_p
    Fp::inv(ni, n0);
    Fp::mul(n1, a + NB, ni);
    Fp::mul(r, a, ni);
    Fp::neg(r + NB, n1);
  }
  // inverse of a canonical (non-Montgomery) element; a != 0
  GZ_DEV static void inv_canonical(uint32_t r[N], const uint32_t a[N]) {
    uint32_t m[N];
    to_mont(m, a);
    inv(m, m);
    from_mont(r, m);
  }
};

// The field of a curve struct: F_p for G1 curves, F_p^2 for a G2 struct that
// declares `using Base = <G1 curve>`.
template <class C, class = void>
struct FieldSel {
  using type = F<C>;
};
template <class C>
struct FieldSel<C, std::void_t<typename C::Base>> {
  using type = F2<typename C::Base>;
};
template <class C>
using Field = typename FieldSel<C>::type;

}  // namespace gzkp
