// microbench3.cu -- calibration of the node-wise kernel's memory operations on
// B200: random 4 B loads over a graph-sized array (DRAM), random 8 B loads /
// atomicMin over a small (L2-resident) table, with N in flight per thread.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mb3 tools/microbench3.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}
template <int ILP, int MODE>  // 0 load u32, 1 load u64 (cg), 2 atomicMin u64, 3 red.min u64
__global__ void kern(void* buf, uint64_t n, int iters, unsigned long long* out) {
  uint32_t s = hsh(blockIdx.x * blockDim.x + threadIdx.x + 12345);
  unsigned long long acc = 0;
  for (int it = 0; it < iters; ++it) {
    uint64_t idx[ILP];
#pragma unroll
    for (int i = 0; i < ILP; ++i) { s = hsh(s + i); idx[i] = ((uint64_t)s * 2654435761ull) % n; }
    unsigned long long v[ILP];
#pragma unroll
    for (int i = 0; i < ILP; ++i) {
      if (MODE == 0) v[i] = __ldg((const uint32_t*)buf + idx[i]);
      else if (MODE == 1) v[i] = __ldcg((const unsigned long long*)buf + idx[i]);
      else if (MODE == 2) v[i] = atomicMin((unsigned long long*)buf + idx[i], (unsigned long long)s);
      else { asm volatile("red.global.min.u64 [%0], %1;" ::"l"((unsigned long long*)buf + idx[i]), "l"((unsigned long long)s) : "memory"); v[i] = 0; }
    }
#pragma unroll
    for (int i = 0; i < ILP; ++i) acc += v[i];
  }
  if (acc == 0x1234567) out[0] = acc;
}
template <int ILP, int MODE>
void run(const char* name, void* buf, uint64_t n, int blocks, int threads, int iters) {
  unsigned long long* out; cudaMalloc(&out, 8);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float ms = 0;
  for (int rep = 0; rep < 3; ++rep) {
    cudaEventRecord(e0);
    kern<ILP, MODE><<<blocks, threads>>>(buf, n, iters, out);
    cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
  }
  const double ops = (double)blocks * threads * iters * ILP;
  const double inflight = (double)blocks * threads * ILP;
  printf("%-28s n=%10llu blocks %5d thr %4d ILP %2d: %8.2f G ops/s  latency(Little) %7.2f us\n", name,
         (unsigned long long)n, blocks, threads, ILP, ops / ms / 1e6, inflight / (ops / ms / 1e3) );
  cudaFree(out);
}
int main() {
  const uint64_t big = 125ull << 20;   // 500 MB of u32 (PD indices)
  const uint64_t tab = 256ull << 10;   // 2 MB of u64 (one hop-2 table)
  const uint64_t tab16 = 16 * tab;     // 32 MB (16 tables)
  void* b; cudaMalloc(&b, big * 4); cudaMemset(b, 0xFF, big * 4);
  for (int blocks : {296, 1184}) {
    run<4, 0>("gather u32 500MB", b, big, blocks, 512, 64);
    run<8, 0>("gather u32 500MB", b, big, blocks, 512, 32);
    run<16, 0>("gather u32 500MB", b, big, blocks, 256, 16);
    run<8, 1>("load u64 2MB", b, tab, blocks, 512, 32);
    run<8, 1>("load u64 32MB", b, tab16, blocks, 512, 32);
    run<8, 2>("atomicMin u64 2MB", b, tab, blocks, 512, 32);
    run<8, 2>("atomicMin u64 32MB", b, tab16, blocks, 512, 32);
    run<8, 3>("red.min u64 32MB", b, tab16, blocks, 512, 32);
    run<8, 2>("atomicMin u64 500MB", b, big / 2, blocks, 512, 32);
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
}
