// microbench_l2fetch.cu -- random 4-byte gathers over an 8 GB array: useful
// 32 B sectors/s versus the L2 fetch-granularity limit
// (cudaLimitMaxL2FetchGranularity 0/32/64/128) and the load flavour
// (ld.global.nc default, ld.global.cg, ld.global.L2::64B prefetch hint off).
// Prints one line per configuration; DRAM bytes are read with ncu separately.
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}

template <int MODE>
__device__ __forceinline__ int ld(const int* p) {
  int v;
  if (MODE == 0) v = __ldg(p);
  else if (MODE == 1) asm volatile("ld.global.cg.s32 %0, [%1];" : "=r"(v) : "l"(p));
  else if (MODE == 2) asm volatile("ld.global.cs.s32 %0, [%1];" : "=r"(v) : "l"(p));
  else if (MODE == 3) asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(v) : "l"(p));
  else if (MODE == 4) asm volatile("ld.global.L2::64B.s32 %0, [%1];" : "=r"(v) : "l"(p));
  else if (MODE == 5) asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p));
  else if (MODE == 6) asm volatile("ld.volatile.global.s32 %0, [%1];" : "=r"(v) : "l"(p));
  else if (MODE == 7) asm volatile("atom.global.or.b32 %0, [%1], 0;" : "=r"(v) : "l"(p));
  return v;
}

template <int ILP, int MODE>
__global__ void gath(const int* big, size_t nbig, int iters, int* out) {
  uint32_t s = hsh(blockIdx.x * blockDim.x + threadIdx.x + 777);
  int acc = 0;
  for (int it = 0; it < iters; ++it) {
    size_t idx[ILP];
#pragma unroll
    for (int i = 0; i < ILP; ++i) { s = hsh(s + i); idx[i] = ((size_t)s * 8 + (s >> 29)) % nbig; }
    int v[ILP];
#pragma unroll
    for (int i = 0; i < ILP; ++i) v[i] = ld<MODE>(big + idx[i]);
#pragma unroll
    for (int i = 0; i < ILP; ++i) acc += v[i];
  }
  if (acc == 0x1234567) out[0] = acc;
}

// dependent chains (walk-like): idx_{t+1} = f(value read at idx_t)
__global__ void chase(const int* big, size_t nbig, int iters, int* out) {
  uint32_t s = hsh(blockIdx.x * blockDim.x + threadIdx.x + 99);
  int acc = 0;
  for (int it = 0; it < iters; ++it) {
    const size_t idx = ((size_t)hsh(s) * 8 + (s & 7)) % nbig;
    const int v = __ldg(big + idx);
    s = s * 747796405u + (uint32_t)v + 1u;
    acc += v;
  }
  if (acc == 0x1234567) out[0] = acc;
}

// scattered 4-byte stores into rows of 81 ints (the walk trace pattern)
__global__ void trace_store(int* tr, size_t rows, int len) {
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < rows; i += (size_t)gridDim.x * blockDim.x)
    for (int t = 0; t < len; ++t) tr[i * len + t] = t;
}

int main() {
  const size_t maxn = (size_t)2 << 30;  // 8 GB of int
  int* big;
  cudaMalloc(&big, maxn * 4);
  cudaMemset(big, 1, maxn * 4);
  int* out;
  cudaMalloc(&out, 8);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const char* names[8] = {"ldg", "cg", "cs", "nc.L1::no_allocate", "L2::64B", "relaxed.gpu", "volatile", "atom.or"};
  for (size_t n : {maxn, maxn / 16, maxn / 128}) {
    for (int mode = 0; mode < 8; ++mode) {
      const int blocks = 148 * 4, threads = 512, iters = 32;
      float ms = 0;
      for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(e0);
        switch (mode) {
          case 0: gath<8, 0><<<blocks, threads>>>(big, n, iters, out); break;
          case 1: gath<8, 1><<<blocks, threads>>>(big, n, iters, out); break;
          case 2: gath<8, 2><<<blocks, threads>>>(big, n, iters, out); break;
          case 3: gath<8, 3><<<blocks, threads>>>(big, n, iters, out); break;
          case 4: gath<8, 4><<<blocks, threads>>>(big, n, iters, out); break;
          case 5: gath<8, 5><<<blocks, threads>>>(big, n, iters, out); break;
          case 6: gath<8, 6><<<blocks, threads>>>(big, n, iters, out); break;
          default: gath<8, 7><<<blocks, threads>>>(big, n, iters, out); break;
        }
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
      }
      const double ops = (double)blocks * threads * iters * 8;
      printf("array %6zu MB mode %-20s : %7.2f G random loads/s\n", n * 4 >> 20, names[mode], ops / ms / 1e6);
    }
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
}
