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
//
// Walk index (a0 pre-processing, built once per graph on the first walk when
// it fits in memory): rec[e] = (x, indptr[x] lo, hi, in-degree of x) for every
// CSC position e with x = indices[e].  A step then reads ONE random 16-byte
// record -- the chosen neighbour together with its own column range -- instead
// of the index and then the neighbour's indptr pair: one dependent random HBM
// line per step instead of two (each random access moves a 128-byte line on
// this B200, profiles/r01_random_access_probe.md).  Same draws, same walks.
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>

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
  const int4* rec;            // walk index or NULL (plain CSC)
};

// Membership of x in the ascending column a[0..n).  R-MAT ids are a keyed
// permutation, so a column's ids are spread ~uniformly over [0, N):
// interpolation probes (each one dependent random line) find x or its gap in
// ~log log n steps instead of log n; after WALK_INTERP probes the remaining
// interval is bisected.  The probe order changes only the bytes read, never
// the answer.
constexpr int WALK_INTERP = 8;
__device__ __forceinline__ bool in_sorted(const int32_t* __restrict__ a, int64_t n, int32_t x) {
  if (n <= 0) return false;
  int64_t lo = 0, hi = n - 1;
  int32_t alo = __ldg(a), ahi = __ldg(a + hi);  // two independent loads
  if (x < alo || x > ahi) return false;
  if (x == alo || x == ahi) return true;
  // invariant: a[lo] < x < a[hi]; x can only sit strictly between lo and hi
#pragma unroll 1
  for (int it = 0; it < WALK_INTERP && hi - lo > 1; ++it) {
    const double f = (double)((int64_t)x - alo) / (double)((int64_t)ahi - alo);
    int64_t pos = lo + 1 + (int64_t)(f * (double)(hi - lo - 1));
    pos = pos < lo + 1 ? lo + 1 : (pos > hi - 1 ? hi - 1 : pos);
    const int32_t ap = __ldg(a + pos);
    if (ap == x) return true;
    if (ap < x) {
      lo = pos;
      alo = ap;
    } else {
      hi = pos;
      ahi = ap;
    }
  }
  lo += 1;  // bisect [lo, hi)
  while (lo < hi) {
    const int64_t mid = (lo + hi) >> 1;
    const int32_t y = __ldg(a + mid);
    if (y == x) return true;
    if (y < x) lo = mid + 1;
    else hi = mid;
  }
  return false;
}

// The neighbour at CSC position pos (with the walk index also its column range).
__device__ __forceinline__ int32_t walk_pick(const WalkParams& P, int64_t pos, int64_t& off_x, int64_t& d_x) {
  if (P.rec) {
    const int4 R = __ldg(P.rec + pos);
    off_x = (int64_t)(((uint64_t)(uint32_t)R.z << 32) | (uint32_t)R.y);
    d_x = R.w;
    return R.x;
  }
  return __ldg(P.indices + pos);
}

#ifndef WALK_MINB
#define WALK_MINB 4
#endif
__global__ void __launch_bounds__(256, WALK_MINB) walk_kernel(WalkParams P) {
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
    int64_t cur_off = 0, cur_d = 0;  // walk index: the column range of the next node
    for (int t = 1; t <= P.length; ++t) {
      if (v < 0) {
        tr[t] = -1;
        continue;
      }
      int64_t off, d;
      if (P.rec && t > 1) {  // the record of v, read at the previous step
        off = cur_off;
        d = cur_d;
      } else {
        off = __ldg(P.indptr + v);
        d = __ldg(P.indptr + v + 1) - off;
      }
      if (d == 0) {  // dead end (R13)
        v = -1;
        tr[t] = -1;
        continue;
      }
      int32_t x;
      if (!P.node2vec || t == 1) {
        const U4 r = philox(walker, 0u, ctr2(t, P.node2vec ? TAG_NODE2VEC : TAG_DEEPWALK), 0u, P.key);
        x = walk_pick(P, off + (int64_t)draw_below((uint64_t)d, r.x, r.y), cur_off, cur_d);
      } else {
        const float lo_b = fminf(1.0f, P.bq), hi_b = fmaxf(1.0f, P.bq);
        for (uint32_t trial = 0;; ++trial) {
          const U4 r = philox(walker, trial, ctr2(t, TAG_NODE2VEC), 0u, P.key);
          x = walk_pick(P, off + (int64_t)draw_below((uint64_t)d, r.x, r.y), cur_off, cur_d);
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

// a0: the walk index (see the file comment), one thread per CSC position.
__global__ void walk_index_kernel(const int64_t* __restrict__ indptr, const int32_t* __restrict__ indices,
                                  int64_t nnz, int4* __restrict__ rec) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x) {
    const int32_t x = __ldg(indices + e);
    const int64_t o = __ldg(indptr + x), d = __ldg(indptr + x + 1) - o;
    rec[e] = make_int4(x, (int)(uint32_t)(uint64_t)o, (int)(uint32_t)((uint64_t)o >> 32), (int)d);
  }
}

// Builds the walk index once per graph (16 bytes per CSC entry) unless
// disabled (GS_WALK_PLAIN_CSC / GS_WALK_INDEX=0), the graph has in-degrees
// >= 2^31, the graph lives in host memory (GS_GRAPH_HOST_MAPPED: the index
// would put 4x the index array back into HBM), or the allocation fails --
// then the walk reads the plain CSC.
static const int4* walk_index(const gs_graph* g, cudaStream_t stream, bool plain) {
  gs_graph* gm = const_cast<gs_graph*>(g);
  const char* e = getenv("GS_WALK_INDEX");
  if (plain || (e && e[0] == '0') || g->host_mapped) return nullptr;
  if (gm->walk_rec) return gm->walk_rec;
  if (gm->walk_index_failed || g->num_edges == 0 || g->max_in_degree >= (int64_t(1) << 31)) return nullptr;
  if (!gm->b_walk.ensure(gm->al, (size_t)g->num_edges * 16, stream)) {
    gm->walk_index_failed = true;
    cudaGetLastError();
    return nullptr;
  }
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  walk_index_kernel<<<sms * 16, 256, 0, stream>>>(g->indptr, g->indices, g->num_edges, (int4*)gm->b_walk.ptr); count_launch();
  if (cudaGetLastError() != cudaSuccess) {
    gm->walk_index_failed = true;
    return nullptr;
  }
  gm->walk_rec = (const int4*)gm->b_walk.ptr;
  return gm->walk_rec;
}

gs_status launch_walk(const gs_graph* g, const int32_t* starts, int64_t num_walkers,
                      int64_t walker_base, int length, float p, float q, uint64_t key,
                      bool node2vec, bool plain, cudaStream_t stream, int32_t* traces,
                      int* err) {
  WalkParams P;
  P.rec = num_walkers > 0 && length > 0 ? walk_index(g, stream, plain) : nullptr;
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
  P.err = err ? err : g->d_err;
  if (num_walkers == 0) return GS_OK;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int threads = 256;
  int64_t blocks = (num_walkers + threads - 1) / threads;
  const int64_t max_blocks = (int64_t)sms * 8 * 64;
  if (blocks > max_blocks) blocks = max_blocks;
  walk_kernel<<<(unsigned)blocks, threads, 0, stream>>>(P); count_launch();
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

}  // namespace gsb
