// ec.cuh -- G1 group law in XYZZ coordinates (x = X/ZZ, y = Y/ZZZ, ZZ^3 = ZZZ^2).
//
// The paper's PADD ("point-addition ... including point doubling",
// PAPER.md:116 fn. 2, §2.1) on E: y^2 = x^3 + a x + b.  The paper
// does not fix a coordinate system (reading R6); XYZZ is chosen because
// the bucket hot loop is a mixed add (affine input point) and XYZZ's madd costs
// 8M + 2S with no inversion:
//   madd-2008-s : XYZZ + affine        8M + 2S
//   add-2008-s  : XYZZ + XYZZ         12M + 2S
//   dbl-2008-s-1: 2 * XYZZ (general a)  6M + 3S (+1S +1M when a != 0)
//   mdbl-2008-s-1: 2 * affine
// Exceptional cases are explicit: the identity O is ZZ = ZZZ = 0 (tracked by a
// flag in the hot loop), P == Q takes the doubling path, P == -Q gives O.  Every
// field value is canonical, so the P == Q tests are exact limb comparisons.
#pragma once
#include "field.cuh"
#include "field2.cuh"
#include "field_dfp.cuh"
#include "coop_mul.cuh"

#ifndef GZKP_ADD2
// ec_add_hot (N <= 12): paired products (EC::add2).  Measured: k_reduce_seg
// 610 -> 620 us (BLS12-381 2^19), and madd_nz2 in the hot loop 0.99x
// (tools/madd_bench.cu): ptxas already overlaps what the carry flag allows.
#define GZKP_ADD2 0
#endif

#ifndef GZKP_MADD2_SQR
#define GZKP_MADD2_SQR 1    // madd_nz2: the two squares as squares (1) or as one paired product (0)
#endif

#ifndef GZKP_COOP_SOS
#define GZKP_COOP_SOS 0     // 1: separated-operand-scanning products in the cooperative chains
#endif

#ifndef GZKP_COOP_SPLIT
#define GZKP_COOP_SPLIT 0   // 1: lane-split products (coop_mul.cuh) in the cooperative chains
#endif

#ifndef GZKP_COOP_KARATSUBA
#define GZKP_COOP_KARATSUBA 0   // 1: Karatsuba products in the cooperative chains (measured slower: BLS12-381 tail 1.01 -> 1.20 ms)
#endif

namespace gzkp {

template <class C>
struct EC {
  static constexpr int N = C::N;
  using Fp = Field<C>;

  struct Xyzz {
    uint32_t X[N], Y[N], ZZ[N], ZZZ[N];
  };

  GZ_DEV static void set_inf(Xyzz& P) {
    Fp::set_zero(P.X); Fp::set_one(P.Y); Fp::set_zero(P.ZZ); Fp::set_zero(P.ZZZ);
  }
  GZ_DEV static bool is_inf(const Xyzz& P) { return Fp::is_zero(P.ZZ); }

  GZ_DEV static void from_affine(Xyzz& R, const uint32_t x[N], const uint32_t y[N]) {
    Fp::copy(R.X, x); Fp::copy(R.Y, y); Fp::set_one(R.ZZ); Fp::set_one(R.ZZZ);
  }

  // M = 3 x^2 + a zz^2   (zz == nullptr means zz = 1)
  GZ_DEV static void tangent_m(uint32_t M[N], const uint32_t X[N], const uint32_t* ZZ) {
    uint32_t t[N];
    Fp::sqr(t, X);
    Fp::add(M, t, t);
    Fp::add(M, M, t);
    if constexpr (!C::A_ZERO) {
      uint32_t a[N];
#pragma unroll
      for (int i = 0; i < N; ++i) a[i] = C::A_MONT(i);
      if (ZZ) {
        uint32_t z2[N];
        Fp::sqr(z2, ZZ);
        Fp::mul(t, z2, a);
        Fp::add(M, M, t);
      } else {
        Fp::add(M, M, a);
      }
    }
  }

  // R = 2 * (x, y) for an affine point (mdbl-2008-s-1); y == 0 gives O.
  GZ_DEV static void mdbl(Xyzz& R, const uint32_t x[N], const uint32_t y[N]) {
    uint32_t U[N], V[N], W[N], S[N], M[N], t[N];
    Fp::dbl(U, y);
    Fp::sqr(V, U);
    Fp::mul(W, U, V);
    Fp::mul(S, x, V);
    tangent_m(M, x, nullptr);
    Fp::sqr(t, M);
    Fp::sub(t, t, S);
    Fp::sub(R.X, t, S);                 // X3 = M^2 - 2S
    Fp::sub(t, S, R.X);
    Fp::neg(S, y);
    Fp::mul_sum(R.Y, M, t, W, S);       // Y3 = M(S - X3) - W y (one reduction)
    Fp::copy(R.ZZ, V);
    Fp::copy(R.ZZZ, W);
  }

  // P = 2P (dbl-2008-s-1, general a).  O and 2-torsion map to O (V = 0).
  GZ_DEV static void dbl(Xyzz& P) {
    uint32_t U[N], V[N], W[N], S[N], M[N], t[N];
    Fp::dbl(U, P.Y);
    Fp::sqr(V, U);
    Fp::mul(W, U, V);
    Fp::mul(S, P.X, V);
    tangent_m(M, P.X, P.ZZ);
    Fp::sqr(t, M);
    Fp::sub(t, t, S);
    Fp::sub(P.X, t, S);                 // X3 = M^2 - 2S
    Fp::sub(t, S, P.X);
    Fp::neg(S, P.Y);
    Fp::mul_sum(P.Y, M, t, W, S);       // Y3 = M(S - X3) - W Y1 (one reduction)
    Fp::mul(P.ZZ, V, P.ZZ);
    Fp::mul(P.ZZZ, W, P.ZZZ);
  }

  // acc += (x2, y2) affine, acc not O (madd-2008-s).  Exceptional cases explicit.
  GZ_DEV static void madd_nz(Xyzz& A, const uint32_t x2[N], const uint32_t y2[N]) {
    uint32_t P[N], R[N], PP[N], PPP[N], t[N];
    Fp::mul(P, x2, A.ZZ);               // U2
    Fp::sub(P, P, A.X);                 // P = U2 - X1
    Fp::mul(R, y2, A.ZZZ);              // S2
    Fp::sub(R, R, A.Y);                 // R = S2 - Y1
    if (Fp::is_zero(P)) {
      if (Fp::is_zero(R)) mdbl(A, x2, y2);   // same point
      else set_inf(A);                       // inverse points
      return;
    }
    Fp::sqr(PP, P);
    Fp::mul(PPP, P, PP);
    Fp::mul(A.ZZ, A.ZZ, PP);            // ZZ3 = ZZ1 PP
    Fp::mul(A.ZZZ, A.ZZZ, PPP);         // ZZZ3 = ZZZ1 PPP
    Fp::mul(PP, A.X, PP);               // Q = X1 PP
    Fp::sqr(t, R);
    Fp::sub(t, t, PPP);
    Fp::sub(t, t, PP);
    Fp::sub(A.X, t, PP);                // X3 = R^2 - PPP - 2Q
    Fp::sub(t, PP, A.X);
    Fp::neg(PP, A.Y);
    Fp::mul_sum(A.Y, R, t, PP, PPP);    // Y3 = R(Q - X3) - Y1 PPP (one reduction)
  }

  // madd_nz with its independent products paired (F::mul2: rows of two
  // products interleaved, four carry chains in flight instead of two)
  GZ_DEV static void madd_nz2(Xyzz& A, const uint32_t x2[N], const uint32_t y2[N]) {
    uint32_t P[N], R[N], PP[N], PPP[N], t[N];
    Fp::mul2(P, x2, A.ZZ, R, y2, A.ZZZ);    // U2, S2
    Fp::sub(P, P, A.X);                 // P = U2 - X1
    Fp::sub(R, R, A.Y);                 // R = S2 - Y1
    if (Fp::is_zero(P)) {
      if (Fp::is_zero(R)) mdbl(A, x2, y2);
      else set_inf(A);
      return;
    }
#if GZKP_MADD2_SQR
    Fp::sqr(PP, P);
    Fp::sqr(t, R);
#else
    Fp::mul2(PP, P, P, t, R, R);        // PP = P^2, t = R^2
#endif
    Fp::mul2(PPP, P, PP, A.ZZ, A.ZZ, PP);     // PPP = P PP, ZZ3 = ZZ1 PP
    Fp::mul2(A.ZZZ, A.ZZZ, PPP, PP, A.X, PP); // ZZZ3 = ZZZ1 PPP, Q = X1 PP
    Fp::sub(t, t, PPP);
    Fp::sub(t, t, PP);
    Fp::sub(A.X, t, PP);                // X3 = R^2 - PPP - 2Q
    Fp::sub(t, PP, A.X);
    Fp::neg(PP, A.Y);
    Fp::mul_sum(A.Y, R, t, PP, PPP);    // Y3 = R(Q - X3) - Y1 PPP (one reduction)
  }

  // madd_nz with 4 of its 10 products on the FP64 pipe (Dfp<C>::mul, NEXT-2):
  // one product of each dependency level that has two or more (S2, R^2, Q,
  // Y1 PPP) goes to DFP, the rest stay on IMAD, so the two pipes work
  // concurrently (§4.3's FP64 field arithmetic).
  GZ_DEV static void madd_nz_mixed(Xyzz& A, const uint32_t x2[N], const uint32_t y2[N]) {
    using D = Dfp<C>;
    uint32_t P[N], R[N], PP[N], PPP[N], t[N];
    Fp::mul(P, x2, A.ZZ);               // U2            (IMAD)
    D::mul(R, y2, A.ZZZ);               // S2            (FP64)
    Fp::sub(P, P, A.X);
    Fp::sub(R, R, A.Y);
    if (Fp::is_zero(P)) {
      if (Fp::is_zero(R)) mdbl(A, x2, y2);
      else set_inf(A);
      return;
    }
    Fp::sqr(PP, P);                     // PP            (IMAD)
    D::mul(t, R, R);                    // R^2           (FP64)
    Fp::mul(PPP, P, PP);                // PPP           (IMAD)
    D::mul(P, A.X, PP);                 // Q = X1 PP     (FP64)
    Fp::mul(A.ZZ, A.ZZ, PP);            // ZZ3           (IMAD)
    Fp::mul(A.ZZZ, A.ZZZ, PPP);         // ZZZ3          (IMAD)
    D::mul(PP, A.Y, PPP);               // Y1 PPP        (FP64)
    Fp::sub(t, t, PPP);
    Fp::sub(t, t, P);
    Fp::sub(A.X, t, P);                 // X3 = R^2 - PPP - 2Q
    Fp::sub(t, P, A.X);
    Fp::mul(t, R, t);                   // R (Q - X3)    (IMAD)
    Fp::sub(A.Y, t, PP);                // Y3 = R(Q - X3) - Y1 PPP
  }

  // acc += B (add-2008-s), all cases.
  GZ_DEV static void add(Xyzz& A, const Xyzz& B) {
    if (is_inf(B)) return;
    if (is_inf(A)) { A = B; return; }
    uint32_t U1[N], S1[N], P[N], R[N], PP[N], PPP[N], t[N];
    Fp::mul(U1, A.X, B.ZZ);
    Fp::mul(P, B.X, A.ZZ);
    Fp::sub(P, P, U1);                  // P = U2 - U1
    Fp::mul(S1, A.Y, B.ZZZ);
    Fp::mul(R, B.Y, A.ZZZ);
    Fp::sub(R, R, S1);                  // R = S2 - S1
    if (Fp::is_zero(P)) {
      if (Fp::is_zero(R)) dbl(A);
      else set_inf(A);
      return;
    }
    Fp::sqr(PP, P);
    Fp::mul(PPP, P, PP);
    Fp::mul(A.ZZ, A.ZZ, B.ZZ);
    Fp::mul(A.ZZ, A.ZZ, PP);            // ZZ3 = ZZ1 ZZ2 PP
    Fp::mul(A.ZZZ, A.ZZZ, B.ZZZ);
    Fp::mul(A.ZZZ, A.ZZZ, PPP);         // ZZZ3 = ZZZ1 ZZZ2 PPP
    Fp::mul(PP, U1, PP);                // Q = U1 PP
    Fp::sqr(t, R);
    Fp::sub(t, t, PPP);
    Fp::sub(t, t, PP);
    Fp::sub(A.X, t, PP);                // X3 = R^2 - PPP - 2Q
    Fp::sub(t, PP, A.X);
    Fp::neg(S1, S1);
    Fp::mul_sum(A.Y, R, t, S1, PPP);    // Y3 = R(Q - X3) - S1 PPP (one reduction)
  }

  // add with its independent products paired (F::mul2, four carry chains in
  // flight): for the latency-bound post-processing (segment running sums,
  // tree sums, merges) that runs few warps per SM.  Same values as add().
  GZ_DEV static void add2(Xyzz& A, const Xyzz& B) {
    if (is_inf(B)) return;
    if (is_inf(A)) { A = B; return; }
    uint32_t U1[N], S1[N], P[N], R[N], PP[N], PPP[N], t[N];
    Fp::mul2(U1, A.X, B.ZZ, P, B.X, A.ZZ);      // U1, U2
    Fp::mul2(S1, A.Y, B.ZZZ, R, B.Y, A.ZZZ);    // S1, S2
    Fp::sub(P, P, U1);                  // P = U2 - U1
    Fp::sub(R, R, S1);                  // R = S2 - S1
    if (Fp::is_zero(P)) {
      if (Fp::is_zero(R)) dbl(A);
      else set_inf(A);
      return;
    }
    Fp::mul2(A.ZZ, A.ZZ, B.ZZ, A.ZZZ, A.ZZZ, B.ZZZ);   // ZZ1 ZZ2, ZZZ1 ZZZ2
    Fp::sqr(PP, P);
    Fp::sqr(t, R);
    Fp::mul2(PPP, P, PP, A.ZZ, A.ZZ, PP);      // PPP = P PP, ZZ3 = ZZ1 ZZ2 PP
    Fp::mul2(A.ZZZ, A.ZZZ, PPP, PP, U1, PP);   // ZZZ3 = ZZZ1 ZZZ2 PPP, Q = U1 PP
    Fp::sub(t, t, PPP);
    Fp::sub(t, t, PP);
    Fp::sub(A.X, t, PP);                // X3 = R^2 - PPP - 2Q
    Fp::sub(t, PP, A.X);
    Fp::neg(S1, S1);
    Fp::mul_sum(A.Y, R, t, S1, PPP);    // Y3 = R(Q - X3) - S1 PPP (one reduction)
  }

  // XYZZ (Montgomery) -> canonical affine, O -> (0,0).
  GZ_DEV static void to_affine_canonical(uint32_t x[N], uint32_t y[N], const Xyzz& P) {
    if (is_inf(P)) { Fp::set_zero(x); Fp::set_zero(y); return; }
    uint32_t d[N], inv[N], t[N];
    Fp::mul(d, P.ZZ, P.ZZZ);
    Fp::inv(inv, d);                    // 1 / (ZZ ZZZ)
    Fp::mul(t, inv, P.ZZZ);             // 1 / ZZ
    Fp::mul(t, P.X, t);
    Fp::from_mont(x, t);
    Fp::mul(t, inv, P.ZZ);              // 1 / ZZZ
    Fp::mul(t, P.Y, t);
    Fp::from_mont(y, t);
  }

  // vectorised copies of one N-limb coordinate (16-B aligned when N % 4 == 0)
  GZ_DEV static void ld(uint32_t d[N], const uint32_t* src) {
    if constexpr (N % 4 == 0) {
      const uint4* s = reinterpret_cast<const uint4*>(src);
#pragma unroll
      for (int i = 0; i < N / 4; ++i) {
        uint4 v = s[i];
        d[4 * i] = v.x; d[4 * i + 1] = v.y; d[4 * i + 2] = v.z; d[4 * i + 3] = v.w;
      }
    } else {
      const uint2* s = reinterpret_cast<const uint2*>(src);
#pragma unroll
      for (int i = 0; i < N / 2; ++i) { uint2 v = s[i]; d[2 * i] = v.x; d[2 * i + 1] = v.y; }
    }
  }
  GZ_DEV static void st(uint32_t* dst, const uint32_t d[N]) {
    if constexpr (N % 4 == 0) {
      uint4* s = reinterpret_cast<uint4*>(dst);
#pragma unroll
      for (int i = 0; i < N / 4; ++i) s[i] = make_uint4(d[4 * i], d[4 * i + 1], d[4 * i + 2], d[4 * i + 3]);
    } else {
      uint2* s = reinterpret_cast<uint2*>(dst);
#pragma unroll
      for (int i = 0; i < N / 2; ++i) s[i] = make_uint2(d[2 * i], d[2 * i + 1]);
    }
  }
  // an XYZZ point in memory is X || Y || ZZ || ZZZ (4N u32, Montgomery form)
  GZ_DEV static void load(Xyzz& P, const uint32_t* src) {
    ld(P.X, src); ld(P.Y, src + N); ld(P.ZZ, src + 2 * N); ld(P.ZZZ, src + 3 * N);
  }
  GZ_DEV static void store(uint32_t* dst, const Xyzz& P) {
    st(dst, P.X); st(dst + N, P.Y); st(dst + 2 * N, P.ZZ); st(dst + 3 * N, P.ZZZ);
  }
};

// ---- warp-cooperative group law for latency-bound serial chains ----------
// The window combination is a chain of (W-1)c doublings on ONE point; one
// thread runs it at the latency of 9 dependent products per doubling.  Here
// every lane of a warp holds the same point and lane q = lane & 3 computes the
// q-th independent product of each dependency level of the formula, then the
// products are broadcast with shuffles (warp-uniform control flow, no
// divergence).  Critical path: 3 products per dbl-2008-s-1, 4 per add-2008-s.
// This is the paper's cooperative-group idea applied at
// the formula level instead of the limb level.
template <class C>
struct CoopEC {
  static constexpr int N = C::N;
  using Fp = Field<C>;
  using E = EC<C>;
  using Xyzz = typename E::Xyzz;

  // lane-split products (coop_mul.cuh): product q of a level is computed by
  // lanes 8q .. 8q+7 and published in shared memory; otherwise lane q
  // computes it alone and it is broadcast by shuffles
  // GZKP_COOP_SPLIT=1 (compile time): measured slower than the one-lane
  // product (BLS12-381 tail 1.00 -> 1.55 ms, MNT4-753 2^17 10.97 -> 11.19 ms;
  // profiles/r02_coop_split_experiment.md), so off by default
  static constexpr bool SPLIT = GZKP_COOP_SPLIT && CoopMul<C>::ON && std::is_same<Fp, F<C>>::value;
  GZ_DEV static void bcast(uint32_t d[N], const uint32_t s[N], int src) {
    if constexpr (SPLIT) {
      CoopMul<C>::result(d, src);
    } else {
#pragma unroll
      for (int i = 0; i < N; ++i) d[i] = __shfl_sync(0xffffffffu, s[i], src);
    }
  }
  // branch-free 4-way blend by lane (pure LOP3s: no local-memory indexing)
  GZ_DEV static void pick(uint32_t d[N], int q, const uint32_t* a0, const uint32_t* a1, const uint32_t* a2,
                          const uint32_t* a3) {
    const uint32_t m0 = 0u - (uint32_t)(q == 0), m1 = 0u - (uint32_t)(q == 1);
    const uint32_t m2 = 0u - (uint32_t)(q == 2), m3 = 0u - (uint32_t)(q == 3);
#pragma unroll
    for (int i = 0; i < N; ++i) d[i] = (a0[i] & m0) | (a1[i] & m1) | (a2[i] & m2) | (a3[i] & m3);
  }
  // one level: lane q computes r = x_q * y_q; results of lanes 0..k-1 broadcast
  GZ_DEV static void level(uint32_t r[N], const uint32_t* x0, const uint32_t* y0, const uint32_t* x1,
                           const uint32_t* y1, const uint32_t* x2, const uint32_t* y2, const uint32_t* x3,
                           const uint32_t* y3) {
    const int q = SPLIT ? (threadIdx.x & 31) >> 3 : threadIdx.x & 3;
    uint32_t x[N], y[N];
    pick(x, q, x0, x1, x2, x3);
    pick(y, q, y0, y1, y2, y3);
    if constexpr (SPLIT) {
      CoopMul<C>::mul(r, x, y, CoopMul<C>::smem());
      return;
    }
    // always inlined here (also for N = 24): per-lane operands feeding an
    // out-of-line call between warp shuffles produced wrong MNT4-753 results.
    // GZKP_COOP_KARATSUBA=1 tries the one-level Karatsuba product here (three
    // independent half products for the single warp's ILP): measured slower.
#if GZKP_COOP_KARATSUBA
    if constexpr (N >= 8 && N <= 12 && N % 4 == 0) Fp::mul_kara(r, x, y);
    else Fp::mul_inline(r, x, y);
#elif GZKP_COOP_SOS
    if constexpr (N >= 8 && std::is_same<Fp, F<C>>::value) Fp::mul_sos(r, x, y);
    else Fp::mul_inline(r, x, y);
#else
    Fp::mul_inline(r, x, y);
#endif
  }

  // P = 2P (all lanes hold P; identical result on every lane)
  GZ_DEV static void dbl(Xyzz& P) {
    uint32_t U[N], V[N], XX[N], W[N], S[N], MM[N], M[N], t[N], r[N];
    Fp::dbl(U, P.Y);
    // level 1: V = U^2, XX = X^2, (lane 2: ZZ^2 for a != 0)
    level(r, U, U, P.X, P.X, P.ZZ, P.ZZ, U, U);
    bcast(V, r, 0);
    bcast(XX, r, 1);
    Fp::add(M, XX, XX);
    Fp::add(M, M, XX);
    if constexpr (!C::A_ZERO) {
      uint32_t z2[N];
      bcast(z2, r, 2);
      if constexpr (C::A_SMALL == 2) {
        Fp::dbl(t, z2);
      } else {
        uint32_t a[N];
#pragma unroll
        for (int i = 0; i < N; ++i) a[i] = C::A_MONT(i);
        Fp::mul(t, z2, a);
      }
      Fp::add(M, M, t);
    }
    // level 2: W = U V, S = X V, MM = M^2, ZZ3 = V ZZ
    level(r, U, V, P.X, V, M, M, V, P.ZZ);
    bcast(W, r, 0);
    bcast(S, r, 1);
    bcast(MM, r, 2);
    bcast(P.ZZ, r, 3);
    Fp::sub(t, MM, S);
    Fp::sub(P.X, t, S);                 // X3 = M^2 - 2S
    Fp::sub(t, S, P.X);
    // level 3: M (S - X3), W Y, ZZZ3 = W ZZZ
    level(r, M, t, W, P.Y, W, P.ZZZ, M, t);
    bcast(t, r, 0);
    bcast(U, r, 1);
    bcast(P.ZZZ, r, 2);
    Fp::sub(P.Y, t, U);                 // Y3 = M(S - X3) - W Y
  }

  // A += B, all cases (warp-uniform branches: every lane holds the same values)
  GZ_DEV static void add(Xyzz& A, const Xyzz& B) {
    if (E::is_inf(B)) return;
    if (E::is_inf(A)) { A = B; return; }
    uint32_t U1[N], S1[N], P[N], R[N], PP[N], RR[N], T1[N], T2[N], PPP[N], Q[N], t[N], r[N];
    // level 1: U1 = X1 ZZ2, U2 = X2 ZZ1, S1 = Y1 ZZZ2, S2 = Y2 ZZZ1
    level(r, A.X, B.ZZ, B.X, A.ZZ, A.Y, B.ZZZ, B.Y, A.ZZZ);
    bcast(U1, r, 0);
    bcast(P, r, 1);
    bcast(S1, r, 2);
    bcast(R, r, 3);
    Fp::sub(P, P, U1);
    Fp::sub(R, R, S1);
    if (Fp::is_zero(P)) {
      if (Fp::is_zero(R)) dbl(A);
      else E::set_inf(A);
      return;
    }
    // level 2: PP = P^2, RR = R^2, T1 = ZZ1 ZZ2, T2 = ZZZ1 ZZZ2
    level(r, P, P, R, R, A.ZZ, B.ZZ, A.ZZZ, B.ZZZ);
    bcast(PP, r, 0);
    bcast(RR, r, 1);
    bcast(T1, r, 2);
    bcast(T2, r, 3);
    // level 3: PPP = P PP, Q = U1 PP, ZZ3 = T1 PP
    level(r, P, PP, U1, PP, T1, PP, P, PP);
    bcast(PPP, r, 0);
    bcast(Q, r, 1);
    bcast(A.ZZ, r, 2);
    Fp::sub(t, RR, PPP);
    Fp::sub(t, t, Q);
    Fp::sub(A.X, t, Q);                 // X3 = R^2 - PPP - 2Q
    Fp::sub(t, Q, A.X);
    // level 4: ZZZ3 = T2 PPP, S1 PPP, R (Q - X3)
    level(r, T2, PPP, S1, PPP, R, t, T2, PPP);
    bcast(A.ZZZ, r, 0);
    bcast(S1, r, 1);
    bcast(t, r, 2);
    Fp::sub(A.Y, t, S1);                // Y3 = R(Q - X3) - S1 PPP
  }
};

// ---- out-of-line versions for the cold kernels (merge, reduction, tail,
// generators, diagnostics): one copy of each group-law body per TU keeps the
// compile time and the instruction footprint bounded; only the bucket hot loop
// (k_accum) inlines madd.
template <class C>
__device__ __noinline__ void ec_add(typename EC<C>::Xyzz& A, const typename EC<C>::Xyzz& B) { EC<C>::add(A, B); }
template <class C>
__device__ __noinline__ void ec_dbl(typename EC<C>::Xyzz& A) { EC<C>::dbl(A); }
template <class C>
__device__ __noinline__ void ec_madd(typename EC<C>::Xyzz& A, const uint32_t* x, const uint32_t* y) {
  uint32_t xx[C::N], yy[C::N];
#pragma unroll
  for (int i = 0; i < C::N; ++i) { xx[i] = x[i]; yy[i] = y[i]; }
  EC<C>::madd_nz(A, xx, yy);
}
template <class C>
__device__ __noinline__ void ec_mdbl(typename EC<C>::Xyzz& A, const uint32_t* x, const uint32_t* y) {
  uint32_t xx[C::N], yy[C::N];
#pragma unroll
  for (int i = 0; i < C::N; ++i) { xx[i] = x[i]; yy[i] = y[i]; }
  EC<C>::mdbl(A, xx, yy);
}
template <class C>
__device__ __noinline__ void ec_to_affine(uint32_t* x, uint32_t* y, const typename EC<C>::Xyzz& P) {
  uint32_t xx[C::N], yy[C::N];
  EC<C>::to_affine_canonical(xx, yy, P);
#pragma unroll
  for (int i = 0; i < C::N; ++i) { x[i] = xx[i]; y[i] = yy[i]; }
}
// Inlined group law for the throughput-bound post-processing kernels (merge,
// bucket reduction) when N <= 12: passing XYZZ operands by reference to an
// out-of-line function keeps them in local memory (r01: k_reduce_seg had a
// 792-B frame and ran at ~28 % of IMAD peak).  N > 12 (MNT4-753 and the G2
// curves) keeps the calls.
template <class C>
GZ_DEV void ec_add_hot(typename EC<C>::Xyzz& A, const typename EC<C>::Xyzz& B) {
  if constexpr (C::N <= 12 && GZKP_ADD2) EC<C>::add2(A, B);
  else if constexpr (C::N <= 12) EC<C>::add(A, B);
  else ec_add<C>(A, B);
}
}  // namespace gzkp
