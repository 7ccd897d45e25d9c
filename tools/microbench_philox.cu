// Philox4x32-10 throughput on one B200: wide multiplies (IMAD.WIDE) vs
// umulhi + mul (IMAD.HI + IMAD), all SMs, results folded so nothing is dead.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include "../paper_conf_sosp_gonglmc0lwl23_b200/csrc/common.cuh"
using namespace gsb;

__device__ __forceinline__ U4 philox_hi(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3, const PhiloxKeys& K) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    const uint32_t hi0 = __umulhi(0xD2511F53u, c0), lo0 = 0xD2511F53u * c0;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c2), lo1 = 0xCD9E8D57u * c2;
    const uint32_t n0 = hi1 ^ c1 ^ K.k[2 * r], n2 = hi0 ^ c3 ^ K.k[2 * r + 1];
    c1 = lo1; c3 = lo0; c0 = n0; c2 = n2;
  }
  return U4{c0, c1, c2, c3};
}

template <int V>
__global__ void bench(PhiloxKeys K, int iters, uint32_t* out) {
  uint32_t acc = 0;
  const uint32_t base = blockIdx.x * blockDim.x + threadIdx.x;
  for (int i = 0; i < iters; ++i) {
    U4 r = V == 0 ? philox_k(base, (uint32_t)i, 77u, 5u, K) : philox_hi(base, (uint32_t)i, 77u, 5u, K);
    acc ^= r.x;
  }
  out[base] = acc;
}

int main() {
  PhiloxKeys K = philox_keys(0x1234567890ull);
  uint32_t* out;
  cudaMalloc(&out, 148 * 8 * 1024 * 4);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int iters = 4096;
  for (int v = 0; v < 2; ++v) {
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(a);
      if (v == 0) bench<0><<<148 * 8, 256>>>(K, iters, out);
      else bench<1><<<148 * 8, 256>>>(K, iters, out);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      const double n = 148.0 * 8 * 256 * iters;
      if (rep) printf("variant %d: %.3f ms, %.2f G philox/s, %.3f SM-cycles per philox (1.965 GHz)\n", v, ms,
                      n / ms / 1e6, 148.0 * 1.965e9 * ms * 1e-3 / n);
    }
  }
  return 0;
}
