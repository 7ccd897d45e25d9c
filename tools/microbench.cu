// microbench.cu -- latency/throughput of the primitives the node-wise kernel
// is built from, in isolation on the B200: random 4-byte gathers over a large
// array, 64-bit CAS into a small (L2-resident) table, loads of that table.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mb tools/microbench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}

template <int MODE, int ILP>
__global__ void kern(const int* big, size_t nbig, unsigned long long* tab, uint32_t tmask,
                     int iters, unsigned long long* out) {
  uint32_t s = hsh(blockIdx.x * blockDim.x + threadIdx.x + 12345);
  unsigned long long acc = 0;
  for (int it = 0; it < iters; ++it) {
    uint32_t idx[ILP];
#pragma unroll
    for (int i = 0; i < ILP; ++i) { s = hsh(s + i); idx[i] = s; }
    if (MODE == 0) {  // random gathers over the big array
      int v[ILP];
#pragma unroll
      for (int i = 0; i < ILP; ++i) v[i] = __ldg(big + (idx[i] % nbig));
#pragma unroll
      for (int i = 0; i < ILP; ++i) acc += v[i];
    } else if (MODE == 1) {  // CAS into the table
      unsigned long long o[ILP];
#pragma unroll
      for (int i = 0; i < ILP; ++i) o[i] = atomicCAS(tab + (idx[i] & tmask), ~0ull, (unsigned long long)idx[i]);
#pragma unroll
      for (int i = 0; i < ILP; ++i) acc += o[i];
    } else if (MODE == 2) {  // loads of the table (L2 hits)
      unsigned long long o[ILP];
#pragma unroll
      for (int i = 0; i < ILP; ++i) o[i] = __ldcg(tab + (idx[i] & tmask));
#pragma unroll
      for (int i = 0; i < ILP; ++i) acc += o[i];
    } else if (MODE == 3) {  // atomicMin into the table
      unsigned long long o[ILP];
#pragma unroll
      for (int i = 0; i < ILP; ++i) o[i] = atomicMin(tab + (idx[i] & tmask), (unsigned long long)idx[i]);
#pragma unroll
      for (int i = 0; i < ILP; ++i) acc += o[i];
    } else {  // fire-and-forget atomics (RED)
#pragma unroll
      for (int i = 0; i < ILP; ++i) atomicMin(tab + (idx[i] & tmask), (unsigned long long)idx[i]);
    }
  }
  if (acc == 0x123456789ull) out[0] = acc;
}

int main() {
  const size_t nbig = 124000000;  // ~PD indices
  int* big;
  cudaMalloc(&big, nbig * 4);
  cudaMemset(big, 1, nbig * 4);
  unsigned long long* tab;
  const size_t tab_entries = 16ull << 18;  // 16 tables of 2^18 entries
  cudaMalloc(&tab, tab_entries * 8);
  cudaMemset(tab, 0xFF, tab_entries * 8);
  unsigned long long* out;
  cudaMalloc(&out, 8);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int blocks = 296, threads = 512, iters = 64;
  const double ops = (double)blocks * threads * iters * 4;
  const char* names[] = {"gather 4B from 496MB", "CAS 64-bit", "ldcg 64-bit", "atomicMin (ret)", "atomicMin (no ret)"};
  for (int mode = 0; mode < 5; ++mode) {
    for (uint32_t tbits : {18u, 22u}) {
      if (mode == 0 && tbits == 22u) continue;
      const uint32_t tmask = (1u << tbits) - 1u;
      for (int rep = 0; rep < 3; ++rep) {
        cudaMemset(tab, 0xFF, tab_entries * 8);
        cudaEventRecord(e0);
        switch (mode) {
          case 0: kern<0, 4><<<blocks, threads>>>(big, nbig, tab, tmask, iters, out); break;
          case 1: kern<1, 4><<<blocks, threads>>>(big, nbig, tab, tmask, iters, out); break;
          case 2: kern<2, 4><<<blocks, threads>>>(big, nbig, tab, tmask, iters, out); break;
          case 3: kern<3, 4><<<blocks, threads>>>(big, nbig, tab, tmask, iters, out); break;
          default: kern<4, 4><<<blocks, threads>>>(big, nbig, tab, tmask, iters, out); break;
        }
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (rep == 2)
          printf("%-22s table %2u bits: %8.3f ms  %8.2f Gop/s  per-iter latency %.2f us\n", names[mode],
                 tbits, ms, ops / ms / 1e6, ms * 1e3 / iters);
      }
    }
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
