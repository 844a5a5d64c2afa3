// coop_smem.cuh -- warp-cooperative group law with the operands in shared
// memory, for the latency-bound serial chains (window combination Horner,
// the bucket reduction's doublings).
//
// Same schedule as CoopEC (ec.cuh): each dependency level of dbl-2008-s-1 /
// add-2008-s has up to 4 independent products, lane q = lane & 3 computes the
// q-th (a cooperative group parallelises the operations of
// one PADD).  What differs is where the values live: the point and every
// intermediate sit in a per-warp shared-memory slot array, a lane loads its
// two operands by slot index (LDS.128) and lanes 0..k-1 store their products
// back.  CoopEC instead kept the point in every lane's registers, blended the
// operands with LOP3/SEL per limb and broadcast each product with N shuffles;
// at N = 24 (MNT4-753) that state did not fit the register file.
// A GROUP of 4 consecutive lanes (lane & ~3) runs one point operation on its
// own slot array, so a warp can run up to 8 independent operations at once
// (e.g. the levels of a tree sum); control flow is uniform within a group and
// __syncwarp over the group's 4 lanes orders its slot traffic.  Lanes of a
// warp that are not in an active group must not call in.
#pragma once
#include "ec.cuh"

#ifndef GZKP_COOPS_SQR
#define GZKP_COOPS_SQR 1    // all-square levels use the triangular square (N <= 12)
#endif

namespace gzkp {

template <class C>
struct CoopS {
  static constexpr int N = C::N;
  using Fp = Field<C>;
  using E = EC<C>;
  using Xyzz = typename E::Xyzz;

  // slots (N words each); the accumulator is A, an addend B
  enum : int {
    AX, AY, AZZ, AZZZ, BX, BY, BZZ, BZZZ,
    U, V, XX, W, S, MM, M, T, R, PP, PPP, Q, T1, T2, S1, Z4,
    CX, CY, CZZ, CZZZ,            // a third point (k_reduce_seg's running sum T)
    NSLOT
  };
  static constexpr int WORDS = NSLOT * N;      // per warp

  GZ_DEV static uint32_t* at(uint32_t* sm, int s) { return sm + s * N; }
  GZ_DEV static int lane() { return threadIdx.x & 3; }        // lane within the group
  GZ_DEV static unsigned gmask() { return 0xFu << (threadIdx.x & 28); }
  GZ_DEV static void sync() { __syncwarp(gmask()); }
  GZ_DEV static int sel4(int q, int a, int b, int c, int d) { return q == 0 ? a : q == 1 ? b : q == 2 ? c : d; }

  GZ_DEV static void put(uint32_t* sm, const Xyzz& P, int base) {
    if (lane() == 0) {
      E::st(at(sm, base), P.X); E::st(at(sm, base + 1), P.Y);
      E::st(at(sm, base + 2), P.ZZ); E::st(at(sm, base + 3), P.ZZZ);
    }
    sync();
  }
  GZ_DEV static void get(Xyzz& P, uint32_t* sm, int base) {
    E::ld(P.X, at(sm, base)); E::ld(P.Y, at(sm, base + 1));
    E::ld(P.ZZ, at(sm, base + 2)); E::ld(P.ZZZ, at(sm, base + 3));
  }
  // 4N words (an XYZZ point) from memory into slots base..base+3 (contiguous)
  GZ_DEV static void put_words(uint32_t* sm, int base, const uint32_t* src) {
    for (int i = lane(); i < 4 * N; i += 4) sm[base * N + i] = src[i];
    sync();
  }

  // one level: lane q < k computes slot d_q = slot a_q * slot b_q
  // (SQ: every product of the level is a square, b_q == a_q)
  template <int K, bool SQ = false>
  GZ_DEV static void level(uint32_t* sm, int d0, int a0, int b0, int d1, int a1, int b1, int d2 = 0, int a2 = 0,
                           int b2 = 0, int d3 = 0, int a3 = 0, int b3 = 0) {
    const int q = lane();
    const int sa = sel4(q, a0, a1, a2, a3), sb = sel4(q, b0, b1, b2, b3), sd = sel4(q, d0, d1, d2, d3);
    uint32_t x[N], y[N], r[N];
    E::ld(x, at(sm, sa));
    if constexpr (SQ && GZKP_COOPS_SQR && std::is_same<Fp, F<C>>::value && N <= 12) {
      Fp::sqr_inline(r, x);
    } else {
      E::ld(y, at(sm, sb));
      Fp::mul_inline(r, x, y);
    }
    sync();
    if (lane() < K) E::st(at(sm, sd), r);
    sync();
  }

  // every lane computes the same linear combination; lane 0 stores
  GZ_DEV static void store0(uint32_t* sm, int d, const uint32_t v[N]) {
    if (lane() == 0) E::st(at(sm, d), v);
  }

  // A = 2A (slots a .. a+3) (dbl-2008-s-1, general a)
  GZ_DEV static void dbl(uint32_t* sm, int a = AX) {
    const int aX = a, aY = a + 1, aZZ = a + 2, aZZZ = a + 3;
    {
      uint32_t y[N], u[N];
      E::ld(y, at(sm, aY));
      Fp::dbl(u, y);
      store0(sm, U, u);
      sync();
    }
    // V = U^2, XX = X^2 (, Z4 = ZZ^2)
    if constexpr (C::A_ZERO) level<2, true>(sm, V, U, U, XX, aX, aX);
    else level<3, true>(sm, V, U, U, XX, aX, aX, Z4, aZZ, aZZ);
    {
      uint32_t xx[N], m[N];
      E::ld(xx, at(sm, XX));
      Fp::add(m, xx, xx);
      Fp::add(m, m, xx);
      if constexpr (!C::A_ZERO) {
        uint32_t z4[N], t[N];
        E::ld(z4, at(sm, Z4));
        if constexpr (C::A_SMALL == 2) {
          Fp::dbl(t, z4);
        } else {
          uint32_t a[N];
#pragma unroll
          for (int i = 0; i < N; ++i) a[i] = C::A_MONT(i);
          Fp::mul(t, z4, a);
        }
        Fp::add(m, m, t);
      }
      store0(sm, M, m);
      sync();
    }
    // W = U V, S = X V, MM = M^2, ZZ3 = V ZZ
    level<4>(sm, W, U, V, S, aX, V, MM, M, M, aZZ, V, aZZ);
    {
      uint32_t mm[N], s[N], x3[N], t[N];
      E::ld(mm, at(sm, MM));
      E::ld(s, at(sm, S));
      Fp::sub(t, mm, s);
      Fp::sub(x3, t, s);                // X3 = M^2 - 2S
      Fp::sub(t, s, x3);
      store0(sm, aX, x3);
      store0(sm, T, t);
      sync();
    }
    // T = M (S - X3), S = W Y, ZZZ3 = W ZZZ
    level<3>(sm, T, M, T, S, W, aY, aZZZ, W, aZZZ);
    {
      uint32_t a[N], b[N], y3[N];
      E::ld(a, at(sm, T));
      E::ld(b, at(sm, S));
      Fp::sub(y3, a, b);                // Y3 = M(S - X3) - W Y
      store0(sm, aY, y3);
      sync();
    }
  }

  GZ_DEV static bool is_zero_slot(uint32_t* sm, int s) {
    uint32_t v[N];
    E::ld(v, at(sm, s));
    return Fp::is_zero(v);
  }
  GZ_DEV static void copy_slot(uint32_t* sm, int d, int s) {
    for (int i = lane(); i < N; i += 4) sm[d * N + i] = sm[s * N + i];
    sync();
  }
  GZ_DEV static void set_inf_a(uint32_t* sm, int a = AX) {
    if (lane() == 0) {
      Xyzz O;
      E::set_inf(O);
      E::st(at(sm, a), O.X); E::st(at(sm, a + 1), O.Y); E::st(at(sm, a + 2), O.ZZ); E::st(at(sm, a + 3), O.ZZZ);
    }
    sync();
  }

  // A += B (add-2008-s), all cases; A in slots a .. a+3, B in b .. b+3
  GZ_DEV static void add(uint32_t* sm, int a = AX, int b = BX) {
    const int aX = a, aY = a + 1, aZZ = a + 2, aZZZ = a + 3;
    const int bX = b, bY = b + 1, bZZ = b + 2, bZZZ = b + 3;
    if (is_zero_slot(sm, bZZ)) return;
    if (is_zero_slot(sm, aZZ)) {
      for (int s = 0; s < 4; ++s) copy_slot(sm, aX + s, bX + s);
      return;
    }
    // U1 = X1 ZZ2, U2 = X2 ZZ1, S1 = Y1 ZZZ2, S2 = Y2 ZZZ1
    level<4>(sm, U, aX, bZZ, PP, bX, aZZ, S1, aY, bZZZ, R, bY, aZZZ);
    bool pz, rz;
    {
      uint32_t u1[N], u2[N], s1[N], s2[N], p[N], r[N];
      E::ld(u1, at(sm, U)); E::ld(u2, at(sm, PP));
      E::ld(s1, at(sm, S1)); E::ld(s2, at(sm, R));
      Fp::sub(p, u2, u1);
      Fp::sub(r, s2, s1);
      pz = Fp::is_zero(p);
      rz = Fp::is_zero(r);
      store0(sm, V, p);                 // P
      store0(sm, R, r);
      sync();
    }
    if (pz) {
      if (rz) dbl(sm, aX);
      else set_inf_a(sm, aX);
      return;
    }
    // PP = P^2, RR = R^2 (-> MM), T1 = ZZ1 ZZ2, T2 = ZZZ1 ZZZ2
    level<4>(sm, PP, V, V, MM, R, R, T1, aZZ, bZZ, T2, aZZZ, bZZZ);
    // PPP = P PP, Q = U1 PP, ZZ3 = T1 PP
    level<3>(sm, PPP, V, PP, Q, U, PP, aZZ, T1, PP);
    {
      uint32_t rr[N], ppp[N], q[N], t[N], x3[N];
      E::ld(rr, at(sm, MM)); E::ld(ppp, at(sm, PPP)); E::ld(q, at(sm, Q));
      Fp::sub(t, rr, ppp);
      Fp::sub(t, t, q);
      Fp::sub(x3, t, q);                // X3 = R^2 - PPP - 2Q
      Fp::sub(t, q, x3);
      store0(sm, aX, x3);
      store0(sm, T, t);
      sync();
    }
    // ZZZ3 = T2 PPP, S1 PPP, R (Q - X3)
    level<3>(sm, aZZZ, T2, PPP, S1, S1, PPP, T, R, T);
    {
      uint32_t a[N], b[N], y3[N];
      E::ld(a, at(sm, T));
      E::ld(b, at(sm, S1));
      Fp::sub(y3, a, b);                // Y3 = R(Q - X3) - S1 PPP
      store0(sm, aY, y3);
      sync();
    }
  }

  // slots base .. base+3 (a point) back to memory (4 lanes)
  GZ_DEV static void store_pt(uint32_t* dst, uint32_t* sm, int base) {
    for (int i = lane(); i < 4 * N; i += 4) dst[i] = sm[base * N + i];
    sync();
  }
  // A <- the group's sum slots back to memory (4 lanes)
  GZ_DEV static void store_a(uint32_t* dst, uint32_t* sm) {
    for (int i = lane(); i < 4 * N; i += 4) dst[i] = sm[AX * N + i];
    sync();
  }

  // In-place tree sum of cnt XYZZ points v[0], v[4N], ... (global or shared
  // memory) into v[0] by the first ng 4-lane groups of the CTA (group g =
  // threadIdx.x / 4 uses the slot array sm + g WORDS).  Level "step" adds
  // v[i + step] into v[i] for i = 0, 2 step, ...: a pair's left element is
  // only ever written by the group that reads it, so one barrier per level
  // suffices.  Every thread of the CTA must call (it contains __syncthreads).
  // Depth ceil(log2 cnt) cooperative adds instead of single-thread adds:
  // ~3.5x lower latency per level for the reductions' short trees.
  GZ_DEV static void tree_sum(uint32_t* v, int cnt, uint32_t* sm, int ng) {
    const int g = threadIdx.x >> 2;
    uint32_t* gs = sm + g * WORDS;
    for (int step = 1; step < cnt; step <<= 1) {
      if (g < ng) {
        for (int i = g * 2 * step; i + step < cnt; i += ng * 2 * step) {
          put_words(gs, AX, v + (size_t)i * 4 * N);
          put_words(gs, BX, v + (size_t)(i + step) * 4 * N);
          add(gs);
          store_a(v + (size_t)i * 4 * N, gs);
        }
      }
      __syncthreads();
    }
  }
};

}  // namespace gzkp
