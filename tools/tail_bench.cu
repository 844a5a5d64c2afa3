// tail_bench.cu -- latency of the window-combination chain (c doublings + one
// XYZZ add per window, one warp) for the cooperative group-law variants:
// CoopEC (registers + shuffles) vs CoopS (shared-memory slots).  Both run the
// same formulas on canonical values, so the bytes must be identical.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo \
//        -I paper_conf_asplos_maxsm0k0zsh23_b200/csrc tools/tail_bench.cu -o /tmp/tb && /tmp/tb
#include <cstdio>
#include <cstdint>
#include <cstring>
#include <vector>
#include <random>
#include <cuda_runtime.h>

#include "curves.cuh"
#include "field.cuh"
#include "ec.cuh"
#include "coop_smem.cuh"

using namespace gzkp;

template <class C>
__global__ void __launch_bounds__(32) k_old(const uint32_t* in, uint32_t* out, int c, int H) {
  using EC_ = EC<C>;
  constexpr int N = C::N;
  typename EC_::Xyzz Q;
  EC_::load(Q, in);
  for (int h = 0; h < H; ++h) {
    for (int k = 0; k < c; ++k) CoopEC<C>::dbl(Q);
    typename EC_::Xyzz X;
    EC_::load(X, in + (size_t)(h + 1) * 4 * N);
    CoopEC<C>::add(Q, X);
  }
  if (threadIdx.x == 0) EC_::store(out, Q);
}

template <class C>
__global__ void __launch_bounds__(32) k_new(const uint32_t* in, uint32_t* out, int c, int H) {
  using CS = CoopS<C>;
  constexpr int N = C::N;
  __shared__ __align__(16) uint32_t sm[CS::WORDS];
  if (threadIdx.x >= 4) return;
  CS::put_words(sm, CS::AX, in);
  for (int h = 0; h < H; ++h) {
    for (int k = 0; k < c; ++k) CS::dbl(sm);
    CS::put_words(sm, CS::BX, in + (size_t)(h + 1) * 4 * N);
    CS::add(sm);
  }
  for (int i = threadIdx.x; i < 4 * N; i += 4) out[i] = sm[CS::AX * N + i];
}

// chain of K dependent Montgomery products on one warp (x <- x y)
template <class C>
__global__ void __launch_bounds__(32) k_mulchain(const uint32_t* in, uint32_t* out, int K) {
  using Fp = Field<C>;
  constexpr int N = C::N;
  uint32_t x[N], y[N], r[N];
  for (int i = 0; i < N; ++i) { x[i] = in[i]; y[i] = in[N + i]; }
  for (int k = 0; k < K; ++k) {
    Fp::mul_inline(r, x, y);
    for (int i = 0; i < N; ++i) x[i] = r[i];
  }
  if (threadIdx.x == 0)
    for (int i = 0; i < N; ++i) out[i] = x[i];
}

// chain of K inversions on one thread: x <- x^-1 (canonical), EEA vs binary GCD
template <class C, bool BG>
__global__ void k_inv(const uint32_t* in, uint32_t* out, int K) {
  using Fp = Field<C>;
  constexpr int N = C::N;
  if (threadIdx.x) return;
  uint32_t x[N], r[N];
  for (int i = 0; i < N; ++i) x[i] = in[i];
  for (int k = 0; k < K; ++k) {
    if constexpr (BG) Fp::inv_bingcd(r, x);
    else Fp::inv_canonical(r, x);
    for (int i = 0; i < N; ++i) x[i] = r[i];
  }
  for (int i = 0; i < N; ++i) out[i] = x[i];
}

template <class C>
void run(const char* name, int c, int H) {
  constexpr int N = C::N;
  std::mt19937 rng(7);
  std::vector<uint32_t> h((size_t)(H + 1) * 4 * N);
  for (size_t i = 0; i < h.size(); ++i) {
    uint32_t v = rng();
    if constexpr (requires { C::P(0); }) {
      if ((int)(i % N) == N - 1) v %= C::P(N - 1);
    } else {      // F_p^2: two base-field halves
      constexpr int H2 = N / 2;
      if ((int)(i % H2) == H2 - 1) v %= C::Base::P(H2 - 1);
    }
    h[i] = v;
  }
  uint32_t *din, *d1, *d2;
  cudaMalloc(&din, h.size() * 4);
  cudaMalloc(&d1, 4 * N * 4);
  cudaMalloc(&d2, 4 * N * 4);
  cudaMemcpy(din, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float t_old = 0, t_new = 0;
  for (int rep = 0; rep < 3; ++rep) {
    cudaEventRecord(e0);
    k_old<C><<<1, 32>>>(din, d1, c, H);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&t_old, e0, e1);
    cudaEventRecord(e0);
    k_new<C><<<1, 32>>>(din, d2, c, H);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&t_new, e0, e1);
  }
  float t_eea = 0, t_bg = 0;
  if constexpr (requires { C::P(0); }) {
    float t_mul = 0;
    const int KM = 2000;
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(e0);
      k_mulchain<C><<<1, 32>>>(din, d1 + 0, KM);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      cudaEventElapsedTime(&t_mul, e0, e1);
    }
    printf("{\"curve\": \"%s\", \"mul_latency_ns\": %.1f}\n", name, 1e6 * t_mul / KM);
    const int K = 8;
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(e0);
      k_inv<C, false><<<1, 32>>>(din, d1 + 0, K);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      cudaEventElapsedTime(&t_eea, e0, e1);
      cudaEventRecord(e0);
      k_inv<C, true><<<1, 32>>>(din, d2 + 0, K);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      cudaEventElapsedTime(&t_bg, e0, e1);
    }
    std::vector<uint32_t> i1(N), i2(N);
    cudaMemcpy(i1.data(), d1, N * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(i2.data(), d2, N * 4, cudaMemcpyDeviceToHost);
    printf("{\"curve\": \"%s\", \"inv_eea_us\": %.2f, \"inv_bingcd_us\": %.2f, \"identical\": %s}\n", name,
           1e3 * t_eea / K, 1e3 * t_bg / K, memcmp(i1.data(), i2.data(), N * 4) == 0 ? "true" : "false");
    // the MSM comparison below overwrites d1 / d2
    for (int rep = 0; rep < 1; ++rep) {
      k_old<C><<<1, 32>>>(din, d1, c, H);
      k_new<C><<<1, 32>>>(din, d2, c, H);
    }
  }
  cudaError_t err = cudaDeviceSynchronize();
  std::vector<uint32_t> o1(4 * N), o2(4 * N);
  cudaMemcpy(o1.data(), d1, 4 * N * 4, cudaMemcpyDeviceToHost);
  cudaMemcpy(o2.data(), d2, 4 * N * 4, cudaMemcpyDeviceToHost);
  const bool same = memcmp(o1.data(), o2.data(), 4 * N * 4) == 0;
  const int dbls = c * H, adds = H;
  printf("{\"curve\": \"%s\", \"c\": %d, \"windows\": %d, \"old_ms\": %.4f, \"new_ms\": %.4f, "
         "\"old_us_per_dbl\": %.3f, \"new_us_per_dbl\": %.3f, \"identical\": %s, \"err\": \"%s\"}\n",
         name, c, H, t_old, t_new, 1e3 * t_old / (dbls + 1.33 * adds), 1e3 * t_new / (dbls + 1.33 * adds),
         same ? "true" : "false", cudaGetErrorString(err));
  cudaFree(din);
  cudaFree(d1);
  cudaFree(d2);
}

int main() {
  run<BN254>("bn254", 16, 15);
  run<BLS12_381>("bls12_381", 16, 15);
  run<MNT4_753>("mnt4_753", 13, 8);
  run<BLS12_381_G2>("bls12_381_g2", 16, 4);
  return 0;
}
