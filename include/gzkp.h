/*
 * gzkp.h -- C ABI of libgzkp.so, a B200 (sm_100a) G1 multi-scalar
 * multiplication library.
 *
 * The operation (§2.1):   Q = s . P = sum_{i<n} s_i (x) P_i
 * over the G1 group of y^2 = x^3 + a x + b, for the curves the
 * paper evaluates: ALT-BN128 (BN254), BLS12-381, MNT4-753 (PAPER.md:279-287,
 * Table 1).  n is "typically a power of 2" but any n is accepted (PAPER.md:114
 * fn. 1).  The point vector is fixed per application, so it can
 * be prepared once (gzkp_points_prepare) and reused across MSMs.
 *
 * Method: signed-window Pippenger (§2.3 windows,
 * buckets, bucket- and window-reduction) with all sub-MSM columns consolidated
 * into one bucket set per window (§4.1), load balancing by sorting
 * entries by bucket and cutting equal-work chunks (§4.2), and
 * the bucket reduction by running sums.  Multi-GPU: each rank
 * sums its shard and one NCCL all-gather combines the partial sums
 * (§5.2, "sub-MSM tasks" per GPU).
 *
 * ENCODINGS (all little-endian u32 limbs):
 *   coordinate  gzkp_field_bytes(curve) bytes, canonical integer in [0, p)
 *               (NOT Montgomery form).  32 / 48 / 96 bytes.
 *   point       x || y  (2 coordinates).  The identity O is (0, 0); (0,0) is on
 *               none of the curves, so the encoding is unambiguous.
 *   scalar      gzkp_scalar_bytes(curve) bytes, any integer < 2^b with
 *               b = 254 / 255 / 753 (bit length of the group order r); the
 *               semantics are integer multiples (not reduced mod r).
 *   partial     gzkp_partial_bytes(curve) bytes: one point in the library's
 *               internal XYZZ Montgomery form (X||Y||ZZ||ZZZ), produced by
 *               gzkp_msm_partial and consumed by gzkp_combine_partials.
 * All device buffers must be 16-byte aligned.
 *
 * OWNERSHIP: the caller owns every input/output buffer; they must stay valid
 * until `stream` reaches the enqueued work.  The library allocates its
 * workspace stream-ordered (cudaMallocAsync) unless one is supplied (_ex).
 * Handles (prepared points, communicators) are library-owned until released.
 *
 * ERRORS: argument errors are reported synchronously (NULL with n > 0,
 * misalignment, unknown curve).  n == 0 writes (0,0).  Kernel faults surface as
 * GZKP_ERROR_CUDA from a later call or a stream synchronisation.  Inputs are
 * not validated unless the environment sets GZKP_DEBUG_CHECKS=1: then every
 * MSM / prepare entry point first checks, on the device, that each point is
 * (0,0) or has canonical coordinates (< p) satisfying y^2 = x^3 + a x + b,
 * and that each scalar is < 2^b, synchronises `stream`, and returns
 * GZKP_ERROR_INVALID_VALUE (detail in gzkp_last_error) before any MSM work.
 * No exception crosses the ABI; gzkp_last_error() gives thread-local detail.
 *
 * THREADING: calls on different streams are independent: the library keeps
 * one workspace and one pair of side streams per (device, stream) -- per
 * (device, stream, thread) for cudaStreamPerThread -- and calls on one stream
 * are ordered by it.  Per-device setup (kernel attributes, the private memory
 * pool, the stack limit) runs once per device, so one process may drive
 * several GPUs.  Release a stream's resources with gzkp_release_stream before
 * destroying it.  Two concurrent gzkp_msm_sharded calls on one communicator
 * are not allowed (NCCL ordering rule).
 *
 * WORK SKIPPED BY DEFINITION: a zero scalar contributes nothing; gzkp_msm /
 * _ex / _partial drop those points before the sort (and convert only the rest
 * to Montgomery form), so sparse scalar vectors cost in
 * proportion to their non-zero entries.
 */
#ifndef GZKP_H
#define GZKP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  GZKP_BN254 = 0,
  GZKP_BLS12_381 = 1,
  GZKP_MNT4_753 = 2,
  /* G2: the order-r subgroup of the
   * sextic twist E'(F_p^2): y^2 = x^3 + b' over F_p^2 = F_p[u]/(u^2 + 1),
   * b' = 3/(9+u) (BN254, EIP-197) and 4(1+u) (BLS12-381).  A coordinate is
   * c0 || c1 (c0 + c1 u), each an F_p value as above, so field_bytes = 64 | 96;
   * scalars are the same F_r scalars as G1. */
  GZKP_BN254_G2 = 3,
  GZKP_BLS12_381_G2 = 4,
  GZKP_TOY_A0 = 100, /* y^2 = x^3 + 3 over F_10099, prime order 9967 (tests) */
  GZKP_TOY_A2 = 101  /* y^2 = x^3 + 2x + 30 over F_10007, prime order 10091 (tests) */
} gzkp_curve;

typedef enum {
  GZKP_SUCCESS = 0,
  GZKP_ERROR_INVALID_VALUE = 1,
  GZKP_ERROR_UNSUPPORTED_CURVE = 2,
  GZKP_ERROR_OUT_OF_MEMORY = 3,
  GZKP_ERROR_CUDA = 4,
  GZKP_ERROR_NCCL = 5
} gzkp_status;

typedef void *gzkp_stream; /* a cudaStream_t; NULL = legacy default stream */

/* --- sizes ------------------------------------------------------------ */
size_t gzkp_field_bytes(int curve);   /* one coordinate: 32 | 48 | 96 (8 for toys; G2: 64 | 96) */
size_t gzkp_scalar_bytes(int curve);  /* one scalar:     32 | 32 | 96 (4 for toys) */
size_t gzkp_partial_bytes(int curve); /* one XYZZ partial: 4 * field_bytes */

/* --- single-GPU MSM ------------------------------------------------------
 * out (device, 2*field_bytes) = sum_i scalars[i] * points[i].
 * points: device, n x (2*field_bytes), canonical affine.
 * scalars: device, n x scalar_bytes.
 * Enqueued on `stream`; returns after enqueue. */
gzkp_status gzkp_msm(int curve, const void *points_affine, const void *scalars, size_t n,
                     void *out, gzkp_stream stream);

/* Same, with caller-provided device workspace of at least
 * gzkp_msm_workspace_bytes(curve, n) bytes (16-B aligned). */
size_t gzkp_msm_workspace_bytes(int curve, size_t n);
gzkp_status gzkp_msm_ex(int curve, const void *points_affine, const void *scalars, size_t n,
                        void *out, void *workspace, size_t workspace_bytes, gzkp_stream stream);

/* Same, but points/scalars/out are HOST buffers (pinned or pageable).  The
 * call copies inputs to the device, runs gzkp_msm and copies the result back;
 * it synchronises `stream` before returning. */
gzkp_status gzkp_msm_host(int curve, const void *points_affine_host, const void *scalars_host,
                          size_t n, void *out_host, gzkp_stream stream);

/* --- prepared points, PAPER.md:194 ("P ... remains unchanged for a specific
 * application", so it is preprocessed once) ------------------------------
 * weighted = M >= 1: GZKP's cross-window consolidation with checkpoint
 *   interval M (§4.1, Algorithm 1): the library stores the
 *   checkpoints 2^(c M j) P_i for j < ceil(W/M), W = ceil((b+1)/c) (that many
 *   copies of n*2*field_bytes bytes of HBM).  Window t = M j + r then uses
 *   checkpoint j and bucket set r, so the W windows accumulate into M bucket
 *   sets; the remaining weight 2^(c r) is applied once per bucket set to its
 *   reduced sum (reading R10), not per point as Alg. 1 lines 8-9 do.
 *   M = 1: the full weighted table, one bucket set, no window combination.
 *   M >= W: no table beyond the points themselves (the standard pipeline).
 *   window_bits = 0 lets the planner choose c, else 2..22; later MSMs on the
 *   handle use that c.
 * weighted = 0: Montgomery-form copy of the points only (standard pipeline);
 *   window_bits 0 (planner per call) or 2..18 (fixed c for every call).
 *   Other values: GZKP_ERROR_INVALID_VALUE.
 * gzkp_points_prepare = _ex(window_bits 0, weighted 1), falling back to
 * weighted 0 if the table does not fit.  gzkp_prepared_info reports the window
 * bits, the number of table copies (1 for weighted = 0), the interval M (0 for
 * unweighted) and the bytes held. */
gzkp_status gzkp_points_prepare_ex(int curve, const void *points_affine, size_t n, int window_bits,
                                   int weighted, void **handle, gzkp_stream stream);
gzkp_status gzkp_points_prepare(int curve, const void *points_affine, size_t n, void **handle,
                                gzkp_stream stream);
gzkp_status gzkp_prepared_info(const void *handle, int *window_bits, int *windows, int *weighted,
                               size_t *bytes);
gzkp_status gzkp_msm_prepared(const void *handle, const void *scalars, size_t n, void *out,
                              gzkp_stream stream);
/* host-buffer scalars/out with a prepared handle (copies inside, synchronises) */
gzkp_status gzkp_msm_prepared_host(const void *handle, const void *scalars_host, size_t n,
                                   void *out_host, gzkp_stream stream);
gzkp_status gzkp_points_release(void *handle);

/* --- building blocks (also used to test sharding on one GPU) ------------- */
/* partial_xyzz (device, partial_bytes) = sum over this slice, not normalised */
gzkp_status gzkp_msm_partial(int curve, const void *points_affine, const void *scalars, size_t n,
                             void *partial_xyzz, gzkp_stream stream);
/* out_affine (device) = sum of `count` partials (device, count x partial_bytes),
 * added in index order, then normalised.  count == 0 gives (0,0). */
gzkp_status gzkp_combine_partials(int curve, const void *partials_xyzz, int count,
                                  void *out_affine, gzkp_stream stream);

/* --- multi-GPU (one process per GPU) -------------------------------------- */
gzkp_status gzkp_nccl_unique_id(unsigned char id[128]);
gzkp_status gzkp_comm_init(int world, int rank, const unsigned char id[128], void **comm);
gzkp_status gzkp_comm_destroy(void *comm);
/* Collective: every rank passes its own shard (possibly n_local == 0).  Each
 * rank runs the full Pippenger on its shard, the per-rank XYZZ partials are
 * exchanged with ONE ncclAllGather, and every rank writes the same `out`. */
gzkp_status gzkp_msm_sharded(int curve, const void *points_affine, const void *scalars,
                             size_t n_local, void *out, gzkp_stream stream, void *comm);
/* Same collective on prepared points: every rank passes the handle of ITS
 * shard (gzkp_points_prepare on the local slice; weighted tables remove the
 * per-rank window combination) and its n_local <= prepared count scalars. */
gzkp_status gzkp_msm_prepared_sharded(const void *handle, const void *scalars, size_t n_local, void *out,
                                      gzkp_stream stream, void *comm);

/* --- NTT over the scalar field F_r -------------------
 * The POLY stage of the prover (§2.2, §3): for N = 2^log_n and
 * A_i in F_r of `curve` (G1 and G2 ids share F_r),
 *   inverse = 0:  out[k] = sum_i in[i] w_N^(i k)        = A(w_N^k)
 *   inverse = 1:  out[i] = N^-1 sum_k in[k] w_N^(-i k)
 * with w_N = g^((r-1)/N), g the smallest quadratic non-residue mod r
 * (reading R15; w_N^(N/2) = -1).  in/out: device, N elements of
 * gzkp_scalar_bytes(curve) bytes each, canonical (< r) little-endian, 16-B
 * aligned; in == out is allowed.  log_n <= gzkp_ntt_max_log(curve)
 * (min(2-adicity of r - 1, 30): 28 | 30 | 30).  Enqueued on `stream`; twiddle
 * tables are built on the device at the first call per (log_n, direction) and
 * kept by the library.  Inputs >= r are not detected. */
int gzkp_ntt_max_log(int curve);
gzkp_status gzkp_ntt(int curve, const void *in, void *out, int log_n, int inverse, gzkp_stream stream);
/* kernels launched by this thread's last gzkp_ntt call (benchmark bookkeeping) */
int gzkp_ntt_last_launches(void);
/* F_r element ops for the tests, same op codes as gzkp_field_op (0..5). */
gzkp_status gzkp_scalar_field_op(int curve, int op, const void *a, const void *b, void *out, size_t n,
                                 gzkp_stream stream);

/* --- benchmark/test input generation (not on the MSM path) --------------- */
/* out[i] = scalars[i] * G (canonical affine) for the curve's fixed generator G.
 * Used to build synthetic proving-key points with known discrete logs. */
gzkp_status gzkp_fixed_base_mul(int curve, const void *scalars, size_t n, void *out_affine,
                                gzkp_stream stream);

/* --- diagnostics ----------------------------------------------------------- */
/* Test hook (not on the MSM path): runs ONLY the product's digit + sort stage
 * (a2-a3: signed c-bit windows, §2.3 / Figure 3; the bucket
 * layout p_index of PAPER.md:206) for `scalars` (device, n x scalar_bytes) at
 * window bits c in 2..18, synchronises, and copies to HOST memory:
 *   offsets_host[0 .. W 2^(c-1)]: bucket key t 2^(c-1) + |d| - 1 (window t,
 *     digit d != 0) owns entries [offsets[key], offsets[key+1]);
 *   vals_host[0 .. E): point index | 0x80000000 if the digit is negative,
 *     E = offsets[W 2^(c-1)].  The order inside a bucket is unspecified.
 * offsets_cap / vals_cap are the buffers' capacities in u32 words. */
gzkp_status gzkp_debug_buckets(int curve, const void *scalars, size_t n, int window_bits,
                               uint32_t *offsets_host, size_t offsets_cap, uint32_t *vals_host,
                               size_t vals_cap, gzkp_stream stream);
/* Elementwise field ops on canonical inputs (device arrays of n elements):
 * op 0: a*b mod p, 1: a+b, 2: a-b, 3: a^-1 (a != 0), 4: round trip to/from Montgomery,
 * 5: a^2 mod p (the dedicated Montgomery squaring), 6: a*b mod p by the FP64
 * (DFP) Montgomery product, which exists for BLS12-381 only (8 x 48-bit limbs;
 * NEXT-2, measured slower than the IMAD product and off by default); every
 * other curve, MNT4-753 included, computes op 6 with the IMAD product,
 * 7: a^-1 mod p by the constant-time binary GCD (the batch-affine inverse;
 * G2 curves fall back to op 3), 8: a*b mod p by the lane-split product of the
 * cooperative chains (8 lanes per product, BN254 / BLS12-381 / MNT4-753; other
 * curves: the one-thread product).  For G2 curves the elements are F_p^2 values
 * c0 || c1. */
gzkp_status gzkp_field_op(int curve, int op, const void *a, const void *b, void *out, size_t n,
                          gzkp_stream stream);
/* Elementwise group ops on canonical affine points (device, n points each):
 * op 0: P+Q via XYZZ madd, 1: P+Q via XYZZ full add, 2: 2P via XYZZ dbl,
 * 3: 2P via mdbl. */
gzkp_status gzkp_ec_op(int curve, int op, const void *P, const void *Q, void *out, size_t n,
                       gzkp_stream stream);
/* Tunables (0 = automatic): window bits c (2..18), entries per accumulation chunk. */
gzkp_status gzkp_set_config(int window_bits, int chunk_entries);
/* Plan the window size the library would use for (curve, n). */
int gzkp_window_bits(int curve, size_t n);
/* Phase profiling (off by default; also GZKP_PROFILE=1).  When on, every MSM
 * call records CUDA events on its own stream between the phases
 *   0 digits+sort (a1-a3), 1 bucket accumulation (a4), 2 merge (a5),
 *   3 bucket reduction (a6), 4 window combination + normalise (a7-a8)
 * without synchronising.  gzkp_profile_read synchronises the recorded events
 * and returns the summed phase times (ms) over all calls since the last reset,
 * plus stats[0] = calls, stats[1] = kernels launched by the last call,
 * stats[2] = non-zero digits (bucket entries) of the last call,
 * stats[3] = window bits c of the last call. */
gzkp_status gzkp_set_profiling(int on);
gzkp_status gzkp_profile_read(double phase_ms[5], uint64_t stats[4], int reset);
/* The library keeps one grow-only workspace and one high-priority side stream
 * per (device, caller stream) so back-to-back calls do not re-allocate.  Call
 * this before destroying a stream that was passed to the library: it frees
 * that stream's workspace (stream-ordered, after the work queued on it) and
 * synchronises and destroys its side stream.  Safe on streams never used. */
gzkp_status gzkp_release_stream(gzkp_stream stream);
const char *gzkp_status_string(gzkp_status status);
const char *gzkp_last_error(void);

#ifdef __cplusplus
}
#endif

#endif /* GZKP_H */
