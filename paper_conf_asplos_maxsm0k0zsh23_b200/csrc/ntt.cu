// ntt.cu -- host side of the F_r NTT (PAPER.md:126-138,
// §3) and its extern "C" entry points (declared in include/gzkp.h).
//
// Pass plan: log N iterations split into P = ceil(log N / B_max) passes of
// near-equal size; a pass of nb iterations gives each CTA G = 2^(TILE_LOG - nb)
// groups of 2^nb elements (G >= 4 contiguous elements per HBM run, PAPER.md:178
// "G ... at 4 or higher").  Twiddle tables w^k (k < N/2) are built on the device
// on first use per (device, field, log N, direction) and cached.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <map>
#include <mutex>
#include <tuple>

#include "fr_fields.cuh"
#include "internal.h"
#include "msm_kernels.cuh"
#include "ntt.cuh"

namespace gzkp {

#define NTT_CHECK(expr)                                             \
  do {                                                              \
    cudaError_t _e = (expr);                                        \
    if (_e != cudaSuccess) return cuda_status(_e, #expr);           \
  } while (0)

struct NttTables {
  uint32_t* tw = nullptr;      // N/2 powers (Montgomery), then the store scale (canonical)
  size_t half = 0;
};

template <class R>
struct NttImpl {
  static constexpr int L = R::N;
  static constexpr int TILE_LOG = NttCfg<R>::TILE_LOG;

  static gzkp_status tables(int fid, int log_n, int inverse, cudaStream_t s, NttTables** out) {
    static std::mutex mu;
    static std::map<std::tuple<int, int, int, int>, NttTables> cache;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lock(mu);
    NttTables& t = cache[std::make_tuple(dev, fid, log_n, inverse)];
    if (!t.tw) {
      t.half = log_n ? (size_t)1 << (log_n - 1) : 0;
      const size_t bytes = (t.half + 1) * L * 4;
      NTT_CHECK(cudaMalloc(&t.tw, bytes));
      const int threads = 128;
      const uint64_t work = (t.half + 31) / 32;
      const int grid = (int)std::max<uint64_t>(1, std::min<uint64_t>((work + threads - 1) / threads,
                                                                     (uint64_t)device_sm_count() * 8));
      k_ntt_twiddles<R><<<grid, threads, 0, s>>>(t.tw, t.half, log_n, inverse, t.tw + t.half * L);
      // publish the table only once it is built: a later call on another
      // (non-blocking) stream must never read it half-written
      cudaError_t e = cudaGetLastError();
      if (e == cudaSuccess) e = cudaStreamSynchronize(s);
      if (e != cudaSuccess) {
        cudaFree(t.tw);
        t.tw = nullptr;
        return cuda_status(e, "k_ntt_twiddles");
      }
    }
    *out = &t;
    return GZKP_SUCCESS;
  }

  static gzkp_status run(int fid, const void* in, void* out, int log_n, int inverse, cudaStream_t s, int* launches) {
    const size_t n = (size_t)1 << log_n;
    const size_t bytes = n * L * 4;
    NttTables* tb = nullptr;
    if (gzkp_status st = tables(fid, log_n, inverse, s, &tb)) return st;
    const size_t smem = ((size_t)1 << TILE_LOG) * L * 4;
    // register budget: MIN_CTAS CTAs/SM (the shared-memory limit) or, with
    // GZKP_NTT_MINB=2 (8-limb fields), 2 CTAs/SM with up to 128 registers
    static const bool two = [] {
      const char* e = getenv("GZKP_NTT_MINB");
      return L <= 8 && e && atoi(e) == 2;
    }();
    auto kern = two ? k_ntt_pass<R, 2> : k_ntt_pass<R>;
    static int attr_tag;   // per device
    if (gzkp_status st = once_per_device(&attr_tag, [smem] {
          NTT_CHECK(cudaFuncSetAttribute(k_ntt_pass<R>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
          NTT_CHECK(cudaFuncSetAttribute(k_ntt_pass<R, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
          return GZKP_SUCCESS;
        }))
      return st;
    *launches = 0;
    if (log_n == 0) {   // N = 1: a_0 = A_0 (N^-1 = 1)
      if (in != out) NTT_CHECK(cudaMemcpyAsync(out, in, bytes, cudaMemcpyDeviceToDevice, s));
      return GZKP_SUCCESS;
    }
    const int nb_max = TILE_LOG - 2;
    const int P = (log_n + nb_max - 1) / nb_max;
    void* ws = nullptr;
    if (P > 1 || in == out) {
      if (gzkp_status st = stream_workspace(s, bytes, &ws)) return st;
    }
    const uint32_t* src = (const uint32_t*)in;
    if (P == 1 && in == out) {
      NTT_CHECK(cudaMemcpyAsync(ws, in, bytes, cudaMemcpyDeviceToDevice, s));
      src = (const uint32_t*)ws;
    }
    int t0 = 0;
    for (int p = 0; p < P; ++p) {
      const int nb = log_n / P + (p < log_n % P ? 1 : 0);
      const int logG = std::min(TILE_LOG - nb, log_n - nb);
      const unsigned grid = (unsigned)(n >> (nb + logG));
      const bool last = p == P - 1;
      uint32_t* dst = last ? (uint32_t*)out : (uint32_t*)ws;
      const int flags = (p == 0 ? NTT_FIRST : 0) | (last ? NTT_LAST : 0) | (last && inverse ? NTT_SCALE : 0);
      const size_t sm = ((size_t)1 << (nb + logG)) * L * 4;
      kern<<<grid, NTT_THREADS, sm, s>>>(src, dst, tb->tw, log_n, t0, nb, logG, flags, tb->tw + tb->half * L);
      NTT_CHECK(cudaGetLastError());
      ++*launches;
      src = dst;
      t0 += nb;
    }
    return GZKP_SUCCESS;
  }

  static gzkp_status field_op(int op, const void* a, const void* b, void* out, size_t n, cudaStream_t s) {
    if (!n) return GZKP_SUCCESS;
    const int threads = 128;
    const int grid = (int)std::min<size_t>((n + threads - 1) / threads, 4096);
    k_field_op<R><<<grid, threads, 0, s>>>(op, (const uint32_t*)a, (const uint32_t*)b, (uint32_t*)out, n);
    NTT_CHECK(cudaGetLastError());
    return GZKP_SUCCESS;
  }
};

static int ntt_field(int curve) {
  switch (curve) {
    case GZKP_BN254: case GZKP_BN254_G2: return 0;
    case GZKP_BLS12_381: case GZKP_BLS12_381_G2: return 1;
    case GZKP_MNT4_753: return 2;
    default: return -1;
  }
}

static int ntt_two_adicity(int fid) {
  switch (fid) {
    case 0: return FR_BN254::TWO_ADICITY;
    case 1: return FR_BLS12_381::TWO_ADICITY;
    case 2: return FR_MNT4_753::TWO_ADICITY;
    default: return -1;
  }
}

static thread_local int g_ntt_launches = 0;

}  // namespace gzkp

using namespace gzkp;

extern "C" {

int gzkp_ntt_max_log(int curve) {
  const int f = ntt_field(curve);
  return f < 0 ? -1 : std::min(ntt_two_adicity(f), 30);
}

gzkp_status gzkp_ntt(int curve, const void* in, void* out, int log_n, int inverse, gzkp_stream stream) {
  const int f = ntt_field(curve);
  if (f < 0) return set_error(GZKP_ERROR_UNSUPPORTED_CURVE, "no scalar field NTT for this curve");
  if (log_n < 0 || log_n > gzkp_ntt_max_log(curve)) return set_error(GZKP_ERROR_INVALID_VALUE, "log_n out of range");
  if (!in || !out) return set_error(GZKP_ERROR_INVALID_VALUE, "NULL buffer");
  if (((uintptr_t)in | (uintptr_t)out) & 15u) return set_error(GZKP_ERROR_INVALID_VALUE, "buffers must be 16-byte aligned");
  init_pool_once();
  cudaStream_t s = (cudaStream_t)stream;
  const int inv = inverse ? 1 : 0;
  switch (f) {
    case 0: return NttImpl<FR_BN254>::run(f, in, out, log_n, inv, s, &g_ntt_launches);
    case 1: return NttImpl<FR_BLS12_381>::run(f, in, out, log_n, inv, s, &g_ntt_launches);
    default: return NttImpl<FR_MNT4_753>::run(f, in, out, log_n, inv, s, &g_ntt_launches);
  }
}

int gzkp_ntt_last_launches(void) { return g_ntt_launches; }

gzkp_status gzkp_scalar_field_op(int curve, int op, const void* a, const void* b, void* out, size_t n,
                                 gzkp_stream stream) {
  const int f = ntt_field(curve);
  if (f < 0) return set_error(GZKP_ERROR_UNSUPPORTED_CURVE, "unknown curve");
  if (op < 0 || op > 5 || (n && (!a || !b || !out))) return set_error(GZKP_ERROR_INVALID_VALUE, "bad arguments");
  init_pool_once();
  cudaStream_t s = (cudaStream_t)stream;
  switch (f) {
    case 0: return NttImpl<FR_BN254>::field_op(op, a, b, out, n, s);
    case 1: return NttImpl<FR_BLS12_381>::field_op(op, a, b, out, n, s);
    default: return NttImpl<FR_MNT4_753>::field_op(op, a, b, out, n, s);
  }
}

}  // extern "C"
