// madd_bench.cu -- throughput of the bucket hot loop's mixed addition at the
// k_accum occupancy (2 CTAs x 128 threads per SM): EC::madd_nz (products in
// sequence) vs EC::madd_nz2 (independent products paired, F::mul2).  Points
// come from shared memory so only the arithmetic is timed; both variants
// must produce identical bytes.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo \
//        -I paper_conf_asplos_maxsm0k0zsh23_b200/csrc tools/madd_bench.cu -o tools/madd_bench
#include <cstdio>
#include <cstdint>
#include <cstring>
#include <vector>
#include <random>
#include <cuda_runtime.h>

#include "curves.cuh"
#include "field.cuh"
#include "ec.cuh"

using namespace gzkp;

constexpr int TABLE = 64;

template <class C, int V>
__global__ void __launch_bounds__(128, 2) k_madd(const uint32_t* __restrict__ pts, uint32_t* __restrict__ out, int K) {
  using E = EC<C>;
  constexpr int N = C::N;
  __shared__ __align__(16) uint32_t sp[TABLE * 2 * N];
  for (int i = threadIdx.x; i < TABLE * 2 * N; i += blockDim.x) sp[i] = pts[i];
  __syncthreads();
  const int tid = blockIdx.x * blockDim.x + threadIdx.x;
  typename E::Xyzz acc;
  {
    uint32_t x[N], y[N];
    E::ld(x, sp + (tid % TABLE) * 2 * N);
    E::ld(y, sp + (tid % TABLE) * 2 * N + N);
    E::from_affine(acc, x, y);
  }
  for (int k = 0; k < K; ++k) {
    const int j = (tid * 7 + k * 13 + 1) % TABLE;
    uint32_t x[N], y[N];
    E::ld(x, sp + j * 2 * N);
    E::ld(y, sp + j * 2 * N + N);
    if constexpr (V == 0) E::madd_nz(acc, x, y);
    else E::madd_nz2(acc, x, y);
  }
  E::store(out + (size_t)tid * 4 * N, acc);
}

template <class C>
void run(const char* name, int K) {
  constexpr int N = C::N;
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int grid = sms * 2, threads = 128, T = grid * threads;
  std::mt19937 rng(11);
  std::vector<uint32_t> h(TABLE * 2 * N);
  for (size_t i = 0; i < h.size(); ++i) {
    uint32_t v = rng();
    if ((int)(i % N) == N - 1) v %= C::P(N - 1);
    h[i] = v;
  }
  uint32_t *dp, *o0, *o1;
  cudaMalloc(&dp, h.size() * 4);
  cudaMalloc(&o0, (size_t)T * 4 * N * 4);
  cudaMalloc(&o1, (size_t)T * 4 * N * 4);
  cudaMemcpy(dp, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float t0 = 0, t1 = 0;
  for (int rep = 0; rep < 3; ++rep) {
    cudaEventRecord(e0);
    k_madd<C, 0><<<grid, threads>>>(dp, o0, K);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&t0, e0, e1);
    cudaEventRecord(e0);
    k_madd<C, 1><<<grid, threads>>>(dp, o1, K);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&t1, e0, e1);
  }
  cudaError_t err = cudaDeviceSynchronize();
  std::vector<uint32_t> a((size_t)T * 4 * N), b((size_t)T * 4 * N);
  cudaMemcpy(a.data(), o0, a.size() * 4, cudaMemcpyDeviceToHost);
  cudaMemcpy(b.data(), o1, b.size() * 4, cudaMemcpyDeviceToHost);
  const double madds = (double)T * K;
  printf("{\"curve\": \"%s\", \"madd_nz_gmadd_s\": %.3f, \"madd_nz2_gmadd_s\": %.3f, \"speedup\": %.3f, "
         "\"identical\": %s, \"err\": \"%s\"}\n",
         name, madds / t0 / 1e6, madds / t1 / 1e6, t0 / t1, memcmp(a.data(), b.data(), a.size() * 4) == 0 ? "true" : "false",
         cudaGetErrorString(err));
  cudaFree(dp);
  cudaFree(o0);
  cudaFree(o1);
}

int main() {
  run<BN254>("bn254", 2048);
  run<BLS12_381>("bls12_381", 1024);
  run<MNT4_753>("mnt4_753", 128);
  return 0;
}
