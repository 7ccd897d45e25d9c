// microbench2.cu -- random-gather throughput vs array size / ILP / sector reuse
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}
template <int ILP>
__global__ void gath(const int* big, size_t nbig, int iters, int* out) {
  uint32_t s = hsh(blockIdx.x * blockDim.x + threadIdx.x + 777);
  int acc = 0;
  for (int it = 0; it < iters; ++it) {
    size_t idx[ILP];
#pragma unroll
    for (int i = 0; i < ILP; ++i) { s = hsh(s + i); idx[i] = ((size_t)s * 8) % nbig; }
    int v[ILP];
#pragma unroll
    for (int i = 0; i < ILP; ++i) v[i] = __ldg(big + idx[i]);
#pragma unroll
    for (int i = 0; i < ILP; ++i) acc += v[i];
  }
  if (acc == 0x1234567) out[0] = acc;
}
int main() {
  const size_t maxn = (size_t)2 << 30;  // 8 GB of int
  int* big; cudaMalloc(&big, maxn * 4); cudaMemset(big, 1, maxn * 4);
  int* out; cudaMalloc(&out, 8);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (size_t mb : {64ul, 200ul, 496ul, 2000ul, 8000ul}) {
    const size_t n = mb << 18;
    for (int cfg = 0; cfg < 3; ++cfg) {
      const int blocks = cfg == 2 ? 148 * 8 : 296, threads = 512, iters = 32;
      float ms = 0;
      for (int rep = 0; rep < 3; ++rep) {
        cudaEventRecord(e0);
        if (cfg == 0) gath<4><<<blocks, threads>>>(big, n, iters, out);
        else gath<8><<<blocks, threads>>>(big, n, iters, out);
        cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
      }
      const double ops = (double)blocks * threads * iters * (cfg == 0 ? 4 : 8);
      printf("array %5zu MB  blocks %4d ILP %d : %7.2f G sectors/s  (%.2f TB/s of 32B sectors)\n", mb, blocks,
             cfg == 0 ? 4 : 8, ops / ms / 1e6, ops * 32 / ms / 1e9);
    }
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
}
