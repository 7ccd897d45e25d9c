// walk.cu -- DeepWalk / Node2Vec random walks (R13, R14).
//
// One thread per walker.  Each step: one Philox
// call, the indptr pair of the current node, one index gather.  Node2Vec uses
// rejection sampling against bmax = max(1/p, 1, 1/q) (KnightKing-style);
// the membership test x in column(prev) is a binary search in prev's sorted
// column and is skipped whenever the accept decision does not depend on it
// (y < min(1, 1/q) always accepts, y >= max(1, 1/q) always rejects): the
// decisions are identical, only the bytes read change.  The previous node's
// column range stays in registers.
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "gs_internal.h"

namespace gsb {

struct WalkParams {
  const int64_t* indptr;
  const int32_t* indices;
  int64_t N;
  const int32_t* starts;
  int64_t num_walkers, walker_base;
  int length;
  int node2vec;
  float bp, bq, bmax;
  uint64_t key;
  int32_t* traces;
  int* err;
};

__device__ __forceinline__ bool in_sorted(const int32_t* __restrict__ a, int64_t n, int32_t x) {
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    const int64_t mid = (lo + hi) >> 1;
    const int32_t y = __ldg(a + mid);
    if (y < x) lo = mid + 1;
    else hi = mid;
  }
  return lo < n && __ldg(a + lo) == x;
}

__global__ void __launch_bounds__(256) walk_kernel(WalkParams P) {
  const int64_t L1 = (int64_t)P.length + 1;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < P.num_walkers;
       i += (int64_t)gridDim.x * blockDim.x) {
    int32_t* tr = P.traces + i * L1;
    const uint32_t walker = (uint32_t)(P.walker_base + i);
    int32_t v = __ldg(P.starts + i);
    tr[0] = v;
    if (v < 0 || (int64_t)v >= P.N) {
      atomicOr(P.err, ERR_SEED_RANGE);
      v = -1;
    }
    int32_t prev = -1;
    int64_t prev_off = 0, prev_d = 0;
    for (int t = 1; t <= P.length; ++t) {
      if (v < 0) {
        tr[t] = -1;
        continue;
      }
      const int64_t off = __ldg(P.indptr + v);
      const int64_t d = __ldg(P.indptr + v + 1) - off;
      if (d == 0) {  // dead end (R13)
        v = -1;
        tr[t] = -1;
        continue;
      }
      int32_t x;
      if (!P.node2vec) {
        const U4 r = philox(walker, 0u, ctr2(t, TAG_DEEPWALK), 0u, P.key);
        x = __ldg(P.indices + off + (int64_t)draw_below((uint64_t)d, r.x, r.y));
      } else if (t == 1) {
        const U4 r = philox(walker, 0u, ctr2(t, TAG_NODE2VEC), 0u, P.key);
        x = __ldg(P.indices + off + (int64_t)draw_below((uint64_t)d, r.x, r.y));
      } else {
        const float lo_b = fminf(1.0f, P.bq), hi_b = fmaxf(1.0f, P.bq);
        for (uint32_t trial = 0;; ++trial) {
          const U4 r = philox(walker, trial, ctr2(t, TAG_NODE2VEC), 0u, P.key);
          x = __ldg(P.indices + off + (int64_t)draw_below((uint64_t)d, r.x, r.y));
          float y = (float)(r.z >> 8) * 0x1p-24f;
          y = __fmul_rn(y, P.bmax);
          bool accept;
          if (trial == 4095u) accept = true;
          else if (x == prev) accept = y < P.bp;
          else if (y < lo_b) accept = true;          // below both 1 and 1/q
          else if (y >= hi_b) accept = false;        // above both
          else accept = y < (in_sorted(P.indices + prev_off, prev_d, x) ? 1.0f : P.bq);
          if (accept) break;
        }
      }
      prev = v;
      prev_off = off;
      prev_d = d;
      v = x;
      tr[t] = x;
    }
  }
}

gs_status launch_walk(const gs_graph* g, const int32_t* starts, int64_t num_walkers,
                      int64_t walker_base, int length, float p, float q, uint64_t key,
                      bool node2vec, cudaStream_t stream, int32_t* traces) {
  WalkParams P;
  P.indptr = g->indptr;
  P.indices = g->indices;
  P.N = g->num_nodes;
  P.starts = starts;
  P.num_walkers = num_walkers;
  P.walker_base = walker_base;
  P.length = length;
  P.node2vec = node2vec ? 1 : 0;
  P.bp = 1.0f / p;
  P.bq = 1.0f / q;
  P.bmax = fmaxf(P.bp, fmaxf(1.0f, P.bq));
  P.key = key;
  P.traces = traces;
  P.err = g->d_err;
  if (num_walkers == 0) return GS_OK;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int threads = 256;
  int64_t blocks = (num_walkers + threads - 1) / threads;
  const int64_t max_blocks = (int64_t)sms * 8 * 64;
  if (blocks > max_blocks) blocks = max_blocks;
  walk_kernel<<<(unsigned)blocks, threads, 0, stream>>>(P);
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

}  // namespace gsb
