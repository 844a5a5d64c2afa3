// microbench.cu -- B200 pipe microbenchmarks (SURVEY.md §7 build step 1).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 \
//        -I paper_conf_asplos_maxsm0k0zsh23_b200/csrc tools/microbench.cu -o /tmp/mb && /tmp/mb
//
// Prints JSON: IMAD, IMAD.WIDE, DFMA throughput per SM per clock (independent
// chains, full occupancy), IMAD+DFMA co-issue, and the single-thread latency
// of one Montgomery multiplication per curve.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#include "curves.cuh"
#include "field.cuh"

using namespace gzkp;

constexpr int CH = 8;          // independent chains per thread
constexpr int ITERS = 4096;

__global__ void k_imad(uint32_t* out, uint32_t seed) {
  uint32_t a[CH];
#pragma unroll
  for (int i = 0; i < CH; ++i) a[i] = seed + threadIdx.x * 7 + i;
  const uint32_t b = seed | 1, c = 12345u;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(a[i]) : "r"(b), "r"(c));
  }
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) s ^= a[i];
  if (s == 0xdeadbeef) out[0] = s;
}

__global__ void k_imad_wide(uint32_t* out, uint32_t seed) {
  uint64_t a[CH];
#pragma unroll
  for (int i = 0; i < CH; ++i) a[i] = seed + threadIdx.x * 7 + i;
  const uint32_t b = seed | 1;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) {
      uint32_t lo = (uint32_t)a[i];
      asm volatile("mad.wide.u32 %0, %1, %2, %0;" : "+l"(a[i]) : "r"(lo), "r"(b));
    }
  }
  uint64_t s = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) s ^= a[i];
  if (s == 0xdeadbeefull) out[0] = (uint32_t)s;
}

__global__ void k_dfma(uint32_t* out, double seed) {
  double a[CH];
#pragma unroll
  for (int i = 0; i < CH; ++i) a[i] = seed + threadIdx.x * 1e-9 + i;
  const double b = 0.999999, c = 1e-7;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) a[i] = fma(a[i], b, c);
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) s += a[i];
  if (s == 123.456) out[0] = 1;
}

// IMAD and DFMA interleaved in one instruction stream: co-issue test
__global__ void k_mix(uint32_t* out, uint32_t seed) {
  uint32_t a[CH];
  double d[CH];
#pragma unroll
  for (int i = 0; i < CH; ++i) { a[i] = seed + threadIdx.x + i; d[i] = 1.0 + i * 1e-3; }
  const uint32_t b = seed | 1, c = 777u;
  const double db = 0.999999, dc = 1e-7;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) {
      asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(a[i]) : "r"(b), "r"(c));
      d[i] = fma(d[i], db, dc);
    }
  }
  uint32_t s = 0;
  double t = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) { s ^= a[i]; t += d[i]; }
  if (s == 0xdeadbeef && t == 1.5) out[0] = 1;
}

__global__ void k_imad_hi(uint32_t* out, uint32_t seed) {
  uint32_t a[CH];
#pragma unroll
  for (int i = 0; i < CH; ++i) a[i] = seed + threadIdx.x * 7 + i;
  const uint32_t b = seed | 1, c = 12345u;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) asm volatile("mad.hi.u32 %0, %0, %1, %2;" : "+r"(a[i]) : "r"(b), "r"(c));
  }
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) s ^= a[i];
  if (s == 0xdeadbeef) out[0] = s;
}

// Montgomery-mul throughput: each thread chains CH/2 independent products
template <class C>
__global__ void k_mul_tput(uint32_t* out, int reps) {
  constexpr int N = C::N;
  uint32_t a[N], b[N], c[N];
#pragma unroll
  for (int i = 0; i < N; ++i) { a[i] = C::ONE(i) ^ threadIdx.x; b[i] = C::R2(i); c[i] = C::ONE(i) + blockIdx.x; }
  F<C>::reduce_once(a);
  F<C>::reduce_once(c);
  for (int r = 0; r < reps; ++r) {
    F<C>::mul(a, a, b);
    F<C>::mul(c, c, b);
  }
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < N; ++i) s ^= a[i] ^ c[i];
  if (s == 0x12345678) out[0] = s;
}

template <class C>
__global__ void k_mul_latency(uint32_t* out, long long* cycles, int reps) {
  constexpr int N = C::N;
  uint32_t a[N], b[N];
#pragma unroll
  for (int i = 0; i < N; ++i) { a[i] = C::ONE(i); b[i] = C::R2(i); }
  long long t0 = clock64();
  for (int r = 0; r < reps; ++r) F<C>::mul(a, a, b);
  long long t1 = clock64();
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < N; ++i) s ^= a[i];
  out[0] = s;
  cycles[0] = (t1 - t0) / reps;
}

template <class K, class... A>
static double time_kernel(K kern, int blocks, int threads, A... args) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  kern<<<blocks, threads>>>(args...);   // warm
  cudaEventRecord(e0);
  kern<<<blocks, threads>>>(args...);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  return ms;
}

int main() {
  int dev = 0, sms = 0, clk_khz = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, dev);
  uint32_t* out;
  long long* cyc;
  cudaMalloc(&out, 64);
  cudaMalloc(&cyc, 64);
  const int threads = 256, blocks = sms * 8;     // 64 warps per SM
  const double ops = (double)blocks * threads * ITERS * CH;
  // rates are reported per SM per clock at the clock the kernel ran at; the
  // clock is measured with a clock64() spin of known length below
  double ms_imad = time_kernel(k_imad, blocks, threads, out, 3u);
  double ms_wide = time_kernel(k_imad_wide, blocks, threads, out, 3u);
  double ms_dfma = time_kernel(k_dfma, blocks, threads, out, 1.0);
  double ms_mix = time_kernel(k_mix, blocks, threads, out, 3u);
  double ms_hi = time_kernel(k_imad_hi, blocks, threads, out, 3u);
  const int mreps = 256;
  const int mblocks = sms * 2, mthreads = 128;    // the accumulation kernel's occupancy (BLS)
  double ms_mbn = time_kernel(k_mul_tput<BN254>, sms * 3, mthreads, out, mreps);
  double ms_mbls = time_kernel(k_mul_tput<BLS12_381>, mblocks, mthreads, out, mreps);
  const double f_ghz0 = clk_khz / 1e6;
  const double mul_bn = (double)sms * 3 * mthreads * mreps * 2 / (ms_mbn * 1e-3) / sms / (f_ghz0 * 1e9);
  const double mul_bls = (double)mblocks * mthreads * mreps * 2 / (ms_mbls * 1e-3) / sms / (f_ghz0 * 1e9);
  printf("{\"imad_hi_per_sm_clk\": %.2f, \"mont_mul_per_sm_clk\": {\"bn254\": %.4f, \"bls12_381\": %.4f}, "
         "\"mont_mul_imad_equiv_per_sm_clk\": {\"bn254\": %.2f, \"bls12_381\": %.2f}}\n",
         (double)blocks * threads * ITERS * CH / (ms_hi * 1e-3) / sms / (f_ghz0 * 1e9), mul_bn, mul_bls,
         mul_bn * 2 * (4 * 8 * 8 + 8), mul_bls * (4 * 12 * 12 + 12));
  // effective clock: time a kernel of known cycle length
  long long h_cyc[4];
  k_mul_latency<BN254><<<1, 1>>>(out, cyc, 64);
  cudaMemcpy(h_cyc, cyc, 8, cudaMemcpyDeviceToHost);
  long long lat_bn = h_cyc[0];
  k_mul_latency<BLS12_381><<<1, 1>>>(out, cyc, 64);
  cudaMemcpy(h_cyc, cyc, 8, cudaMemcpyDeviceToHost);
  long long lat_bls = h_cyc[0];
  k_mul_latency<MNT4_753><<<1, 1>>>(out, cyc, 16);
  cudaMemcpy(h_cyc, cyc, 8, cudaMemcpyDeviceToHost);
  long long lat_mnt = h_cyc[0];
  const double f_ghz = clk_khz / 1e6;   // nominal max clock (attribute)
  auto per_sm_clk = [&](double ms) { return ops / (ms * 1e-3) / sms / (f_ghz * 1e9); };
  printf("{\"sms\": %d, \"clock_attr_ghz\": %.3f, "
         "\"imad_per_sm_clk\": %.2f, \"imad_wide_per_sm_clk\": %.2f, \"dfma_per_sm_clk\": %.2f, "
         "\"mix_imad_plus_dfma_pairs_per_sm_clk\": %.2f, "
         "\"imad_tops\": %.3f, \"dfma_tflops\": %.3f, "
         "\"mont_mul_latency_cycles\": {\"bn254\": %lld, \"bls12_381\": %lld, \"mnt4_753\": %lld}, "
         "\"note\": \"rates at the clock attribute (max); independent chains, %d warps/SM\"}\n",
         sms, f_ghz, per_sm_clk(ms_imad), per_sm_clk(ms_wide), per_sm_clk(ms_dfma), per_sm_clk(ms_mix),
         ops / (ms_imad * 1e-3) / 1e12, 2 * ops / (ms_dfma * 1e-3) / 1e12, lat_bn, lat_bls, lat_mnt,
         blocks * threads / 32 / sms);
  return 0;
}
