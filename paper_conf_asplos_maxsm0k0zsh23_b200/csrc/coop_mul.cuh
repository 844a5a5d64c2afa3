// coop_mul.cuh -- lane-parallel Montgomery product for the latency-bound
// serial chains (window combination, the bucket reduction's doublings).
//
// The paper splits every field operation of a PADD across the threads of a
// cooperative group (§4.1/§4.3: "threads in a warp are
// decomposed into multiple CGs ... each parallelizing individual PADD
// operations").  CoopEC (ec.cuh) already runs the independent products of one
// formula level on different lanes; here each of those products is itself
// split over a group of 8 lanes, so a warp computes up to 4 products at once,
// each at roughly a third of one thread's latency.
//
// Group of 8 lanes (lane r), N limbs, K = N / 4 output columns per lane:
//   T = x y      lane r sums the columns rK .. rK+K-1 (x from a zero-padded
//                shared-memory copy, y in registers), rows split into an even
//                and an odd carry chain; the lanes' (K+2)-word partials overlap
//                by two words and are normalised by one shuffle and a 1-bit
//                carry-lookahead over the group (ballot, an 8-bit add).
//   m = (T mod R) n' mod R    the same column product on lanes 0..3 with the
//                constant n' = -p^-1 mod R (curves.cuh NP).
//   V = T + m p  the column product with the constant p, accumulated on top of
//                T, normalised; V / R (lanes 4..7) < 2p.
//   r = V / R - p if that does not borrow (borrow lookahead over lanes 4..7).
// The result is left in shared memory (res[g]) for the group-to-warp broadcast.
// Everything is warp-synchronous (__syncwarp); control flow is uniform.
#pragma once
#include <cstdint>

namespace gzkp {

template <class C>
struct CoopMul {
  static constexpr int N = C::N;
  static constexpr int K = N / 4;              // columns per lane (8 lanes, 2N columns)
  static constexpr int ZB = 3 * N;             // zero-padded operand window
  static constexpr bool ON = (N == 8 || N == 12 || N == 24);
  // per group: operand window ZB words + result N words
  static constexpr int GROUP_WORDS = ZB + N;
  static constexpr int WARP_WORDS = 4 * GROUP_WORDS;

  // 1-bit carry lookahead over the 8 lanes of the group: lane r generates g
  // (carry out regardless of carry in) or propagates p (all ones: carry in ->
  // carry out); returns the carry into lane r.
  GZ_DEV static uint32_t lookahead(bool g, bool p) {
    const int lane = threadIdx.x & 31, r = lane & 7, sh = lane & ~7;
    const uint32_t G = (__ballot_sync(0xffffffffu, g) >> sh) & 0xffu;
    const uint32_t P = (__ballot_sync(0xffffffffu, p) >> sh) & 0xffu;
    const uint32_t a = G | P;
    const uint32_t c = ((a + G) ^ a ^ G);     // bit r: carry into position r
    return (c >> r) & 1u;
  }

  // A[0..K+1] += sum over the rows j of xw[c - j + N - 1] * Y(j) at column c,
  // c < K (lane-local columns).  Y(j) is a functor (registers or constants).
  template <class Yf>
  GZ_DEV static void columns(uint32_t A[K + 2], const uint32_t xw[N + K - 1], Yf Y) {
    uint32_t EV[K + 2], OD[K + 2];
#pragma unroll
    for (int q = 0; q < K + 2; ++q) { EV[q] = A[q]; OD[q] = 0; }
#pragma unroll
    for (int j = 0; j < N; ++j) {
      const uint32_t yj = Y(j);
      // even columns c: pairs (c, c+1) do not overlap -> one carry chain
#pragma unroll
      for (int c = 0; c < K; c += 2) {
        const uint32_t xv = xw[c - j + N - 1];
        if (c == 0) { MAD_LO_CC(EV[c], xv, yj, EV[c]); }
        else { MADC_LO_CC(EV[c], xv, yj, EV[c]); }
        MADC_HI_CC(EV[c + 1], xv, yj, EV[c + 1]);
      }
      {
        constexpr int ce = ((K - 1) / 2) * 2 + 2;      // first word above the even chain
#pragma unroll
        for (int q = ce; q < K + 1; ++q) ADDC_CC(EV[q], EV[q], 0u);
        ADDC(EV[K + 1], EV[K + 1], 0u);
      }
      if (K > 1) {
#pragma unroll
        for (int c = 1; c < K; c += 2) {
          const uint32_t xv = xw[c - j + N - 1];
          if (c == 1) { MAD_LO_CC(OD[c], xv, yj, OD[c]); }
          else { MADC_LO_CC(OD[c], xv, yj, OD[c]); }
          MADC_HI_CC(OD[c + 1], xv, yj, OD[c + 1]);
        }
        constexpr int co = ((K - 2) / 2) * 2 + 3;      // first word above the odd chain
#pragma unroll
        for (int q = co; q < K + 1; ++q) ADDC_CC(OD[q], OD[q], 0u);
        ADDC(OD[K + 1], OD[K + 1], 0u);
      }
    }
    ADD_CC(A[0], EV[0], OD[0]);
#pragma unroll
    for (int q = 1; q < K + 1; ++q) ADDC_CC(A[q], EV[q], OD[q]);
    ADDC(A[K + 1], EV[K + 1], OD[K + 1]);
  }

  // lane partials A (K+2 words at word offset rK) -> S (K words of the sum)
  GZ_DEV static void normalize(uint32_t S[K], const uint32_t A[K + 2]) {
    const int r = threadIdx.x & 7;
    uint32_t h0 = __shfl_up_sync(0xffffffffu, A[K], 1);
    uint32_t h1 = __shfl_up_sync(0xffffffffu, A[K + 1], 1);
    if (r == 0) { h0 = 0; h1 = 0; }
    uint32_t g;
    ADD_CC(S[0], A[0], h0);
    if (K > 1) {
      ADDC_CC(S[1], A[1], h1);
#pragma unroll
      for (int q = 2; q < K; ++q) ADDC_CC(S[q], A[q], 0u);
      ADDC(g, 0u, 0u);
    } else {
      ADDC(g, 0u, 0u);      // K == 1 is not used (N >= 8)
    }
    uint32_t all = S[0];
#pragma unroll
    for (int q = 1; q < K; ++q) all &= S[q];
    const uint32_t cin = lookahead(g != 0, all == 0xffffffffu);
    ADD_CC(S[0], S[0], cin);
#pragma unroll
    for (int q = 1; q < K - 1; ++q) ADDC_CC(S[q], S[q], 0u);
    if (K > 1) ADDC(S[K - 1], S[K - 1], 0u);
  }

  // load the lane's operand window from the group's zero-padded buffer
  GZ_DEV static void window(uint32_t xw[N + K - 1], const uint32_t* zb) {
    const int r = threadIdx.x & 7;
#pragma unroll
    for (int t = 0; t < N + K - 1; ++t) xw[t] = zb[r * K + t];
  }

  // the warp's shared buffer (CoopEC kernels run one warp per CTA)
  GZ_DEV static uint32_t* smem() {
    __shared__ __align__(16) uint32_t buf[WARP_WORDS];
    return buf;
  }
  // group g's last product (valid after mul() on every lane of the warp)
  GZ_DEV static void result(uint32_t d[N], int g) {
    const uint32_t* res = smem() + g * GROUP_WORDS + ZB;
#pragma unroll
    for (int q = 0; q < N; ++q) d[q] = res[q];
  }
  // r = x y R^-1 mod p; x, y: this lane's group operands (uniform in the
  // group); smem: WARP_WORDS words of this warp.  Leaves the result in the
  // group's res area and returns it in r on every lane of the group.
  GZ_DEV static void mul(uint32_t out[N], const uint32_t x[N], const uint32_t y[N], uint32_t* smem) {
    const int lane = threadIdx.x & 31, g = lane >> 3, r = lane & 7;
    uint32_t* zb = smem + g * GROUP_WORDS;
    uint32_t* res = zb + ZB;
    // zero padding + x in the middle: logical index i at zb[i + N - 1]
    __syncwarp();                                      // previous readers of zb / res are done
#pragma unroll
    for (int q = 0; q < N - 1; ++q)
      if ((q & 7) == r) zb[q] = 0u;
#pragma unroll
    for (int j = 0; j < N; ++j)
      if ((j & 7) == r) zb[N - 1 + j] = x[j];
#pragma unroll
    for (int q = 2 * N - 1; q < ZB; ++q)
      if ((q & 7) == r) zb[q] = 0u;
    __syncwarp();
    uint32_t xw[N + K - 1], A[K + 2], T[K], S[K];
    window(xw, zb);
#pragma unroll
    for (int q = 0; q < K + 2; ++q) A[q] = 0;
    columns(A, xw, [&](int j) { return y[j]; });
    normalize(T, A);                                   // T words rK .. rK+K-1
    // m = (T mod R) n' mod R : T_lo lives on lanes 0..3
    __syncwarp();
    if (r < 4) {
#pragma unroll
      for (int c = 0; c < K; ++c) zb[N - 1 + r * K + c] = T[c];
    }
    __syncwarp();
    window(xw, zb);
#pragma unroll
    for (int q = 0; q < K + 2; ++q) A[q] = 0;
    columns(A, xw, [](int j) { return C::NP(j); });
    normalize(S, A);                                   // m words on lanes 0..3
    __syncwarp();
    if (r < 4) {
#pragma unroll
      for (int c = 0; c < K; ++c) zb[N - 1 + r * K + c] = S[c];
    }
    __syncwarp();
    window(xw, zb);
    // V = T + m p
#pragma unroll
    for (int c = 0; c < K; ++c) A[c] = T[c];
    A[K] = 0;
    A[K + 1] = 0;
    columns(A, xw, [](int j) { return C::P(j); });
    normalize(S, A);                                   // V; V / R on lanes 4..7
    // conditional subtraction of p over lanes 4..7 (lanes 0..3: V mod R = 0)
    uint32_t pw[K];
#pragma unroll
    for (int c = 0; c < K; ++c) {
      const uint32_t p0 = C::P(c), p1 = C::P(K + c), p2 = C::P(2 * K + c), p3 = C::P(3 * K + c);
      pw[c] = r == 4 ? p0 : r == 5 ? p1 : r == 6 ? p2 : r == 7 ? p3 : 0u;
    }
    uint32_t D[K], bo;
    SUB_CC(D[0], S[0], pw[0]);
#pragma unroll
    for (int c = 1; c < K; ++c) SUBC_CC(D[c], S[c], pw[c]);
    SUBC(bo, 0u, 0u);                                  // borrow out (no borrow in)
    uint32_t z = D[0];
#pragma unroll
    for (int c = 1; c < K; ++c) z |= D[c];
    const uint32_t bin = lookahead(bo != 0, z == 0);    // D == 0 propagates a borrow in
    uint32_t bfin;
    SUB_CC(D[0], D[0], bin);
#pragma unroll
    for (int c = 1; c < K; ++c) SUBC_CC(D[c], D[c], 0u);
    SUBC(bfin, 0u, 0u);
    // the borrow out of lane 7 decides: V / R < p keeps V / R
    const uint32_t top_borrow = __shfl_sync(0xffffffffu, (bo | bfin) & 1u, (lane & ~7) | 7);
    if (r >= 4) {
#pragma unroll
      for (int c = 0; c < K; ++c) res[(r - 4) * K + c] = top_borrow ? S[c] : D[c];
    }
    __syncwarp();
#pragma unroll
    for (int q = 0; q < N; ++q) out[q] = res[q];
  }
};

}  // namespace gzkp
