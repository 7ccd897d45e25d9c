// layerwise_sm.cu -- layer-wise ECSF sampling with shared-memory state:
// LADIES (Fig. 3(b)) and COUNT, the modes
// whose bias b(u) is accumulated over the extracted edges.
//
// collective_sample for one mini-batch at a time per CTA (two CTAs
// per SM, persistent, batches claimed from a counter; super-batch P:322-336).
// Every per-batch-layer table lives in shared memory; global memory sees only
// the graph reads (A[:, F], L2-resident across the passes) and the outputs.
// Per (batch, layer) with frontier F (T <= 512 columns) and K <= 512:
//   0  frontier: (indptr, degree) per column; B' = sum over the extracted
//      edges of fp32(w*w) (= B up to per-row rounding) sets the A-Res
//      threshold tau = 1.5K / B' (R6: key = -ln(u) / b; ~1.5K candidates
//      expected below it);
//   1  Extract + Compute (edge-map w*w fused with the row reduction), in
//      P hash partitions of the row ids: each pass inserts the rows of its
//      partition into a 4096-slot shared hash (key + fp64 accumulator); then
//      b(u) = fp32(acc), B = fp32(sum_fp64 b), eligibility b > 0, and the
//      candidates whose A-Res key is below tau (cheap fp32 test, exact fp64
//      key for the survivors) are kept in a shared buffer;
//   2  Select: fewer than K survivors (tau too small) or too many (buffer
//      full) -> tau adjusted and step 1 repeated (rare); otherwise the K
//      smallest (key, u) by rank counting over the survivors, then S ranked
//      by u (R24: every eligible row when at most K are);
//   3  Finalize: p(u) = fp32(b/B); a warp per frontier column re-streams it:
//      rows in S (shared hash) -> a_e = fp32(w/p(u)), c_j = sum_fp64 a,
//      counts; then, in column order with ballot-ordered positions, val_e =
//      fp32(a_e / c_j) into the block (CSC, bump-allocated edge range).
// DESIGN.md section 6 records the global-table kernel this replaces for these
// modes (layerwise.cu; FastGCN's ~280 k candidates per batch-layer keep the
// bitmap kernel of layerwise_bm.cu).
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include <algorithm>
#include <cstdlib>

#include "common.cuh"
#include "gs_internal.h"
#include "nodewise_common.cuh"

namespace gsb {

constexpr int LS_THREADS = 512;
constexpr int LS_WARPS = LS_THREADS / 32;
constexpr int LS_MAXT = 512;     // frontier columns (batch size and K)
constexpr int LS_MAXK = 512;
constexpr int LS_HT = 4096;      // hash slots per partition pass
constexpr int LS_PART = 3072;    // extracted edges per partition (load <= 0.75)
constexpr int LS_CB = 2048;      // candidates kept below tau
constexpr uint32_t LS_EMPTY = 0xFFFFFFFFu;

struct LSParams {
  const int64_t* indptr;
  const int32_t* indices;
  const float* weights;
  int64_t N;
  const int32_t* seeds;
  int64_t num_seeds, batch_size, num_batches, batch_base;
  int L;
  int K[MAX_LAYERS];
  int mode;
  uint64_t key;
  int32_t* col0;
  int32_t* row_map[MAX_LAYERS];
  float* row_prob[MAX_LAYERS];
  int64_t* indptr_out[MAX_LAYERS];
  int32_t* row_local[MAX_LAYERS];
  int64_t* eid[MAX_LAYERS];
  float* val[MAX_LAYERS];
  int64_t edge_cap[MAX_LAYERS];
  unsigned long long* edge_ctr;  // [MAX_LAYERS] bump allocators
  unsigned int* claim;           // batch counter
  uint2* flat;                   // [CTA][flat_cap] (row id, weight) of A[:, F] (L2-resident cache)
  int64_t flat_cap;
  int64_t* meta;
  int* err;
};

struct LSSmem {
  // frontier columns
  int64_t off[LS_MAXT];
  int32_t cnt[LS_MAXT];
  double cs[LS_MAXT];
  int32_t cstart[LS_MAXT + 1];
  // partition hash: row id + fp64 accumulator (step 1); S's local ids (step 3)
  uint32_t hkey[LS_HT];
  double hacc[LS_HT];
  // candidates below tau: (key, u, b)
  double ckey[LS_CB];
  uint32_t cu[LS_CB];
  float cb[LS_CB];
  // S
  uint32_t su[LS_MAXK];
  float sp[LS_MAXK];
  double scr[40];
  long long misc[8];
  int imisc[8];
};

__device__ __forceinline__ uint32_t ls_part(uint32_t u, int P) {
  return (uint32_t)(((uint64_t)(u * 0x85EBCA6Bu ^ (u >> 13)) * (uint32_t)P) >> 32);
}
__device__ __forceinline__ uint32_t ls_slot(uint32_t u) { return (u * 0x9E3779B1u) >> (32 - 12); }

// insert u (first time: claims a slot, counted in imisc[1]); returns the
// slot, or -1 once the table is past its load limit (the caller re-partitions)
__device__ __forceinline__ int ls_insert(LSSmem& sm, uint32_t u) {
  uint32_t h = ls_slot(u);
  while (true) {
    const uint32_t k = sm.hkey[h];
    if (k == u) return (int)h;
    if (k == LS_EMPTY) {
      if (sm.imisc[1] > LS_HT - LS_HT / 8) return -1;
      const uint32_t prev = atomicCAS(&sm.hkey[h], LS_EMPTY, u);
      if (prev == LS_EMPTY) {
        atomicAdd(&sm.imisc[1], 1);
        return (int)h;
      }
      if (prev == u) return (int)h;
    }
    h = (h + 1) & (LS_HT - 1);
  }
}
__device__ __forceinline__ int ls_find(const LSSmem& sm, uint32_t u) {
  uint32_t h = ls_slot(u);
  while (true) {
    const uint32_t k = sm.hkey[h];
    if (k == u) return (int)h;
    if (k == LS_EMPTY) return -1;
    h = (h + 1) & (LS_HT - 1);
  }
}

// Flat edge e of the frontier's columns -> column (binary search of the
// column starts in shared memory).
__device__ __forceinline__ int ls_col(const LSSmem& sm, int T, int e) {
  int lo = 0, hi = T - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (sm.cstart[mid] <= e) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

__global__ void __launch_bounds__(LS_THREADS, 2) layerwise_sm_kernel(LSParams P) {
  extern __shared__ __align__(16) unsigned char ls_raw[];
  LSSmem& sm = *reinterpret_cast<LSSmem*>(ls_raw);
  const int lane = threadIdx.x & 31;
  const bool ladies = P.mode == GS_PROB_LADIES;
  uint2* flat = P.flat + (int64_t)blockIdx.x * P.flat_cap;  // this CTA's (u, w) cache of A[:, F]
  while (true) {
    if (threadIdx.x == 0) sm.misc[7] = (long long)atomicAdd(P.claim, 1u);
    __syncthreads();
    const long long b = sm.misc[7];
    __syncthreads();
    if (b >= P.num_batches) break;
    const int64_t bstart = b * P.batch_size;
    const uint32_t gb = (uint32_t)(P.batch_base + b);
    const int32_t* F = P.seeds + bstart;
    int T = (int)min(P.batch_size, P.num_seeds - bstart);
    int64_t colbase = bstart;
    for (int l = 0; l < P.L; ++l) {
      const int K = P.K[l];
      const int64_t rbase = b * (int64_t)K;
      const int64_t ibase = colbase + b;
      // ---- 0: frontier: (indptr, degree), column starts of the flat edges ----
      {
        const int j = threadIdx.x;  // T <= LS_THREADS
        int64_t off = 0, d = 0;
        if (j < T) {
          const int32_t v = __ldcg(F + j);
          if (v < 0 || (int64_t)v >= P.N) {
            atomicOr(P.err, ERR_SEED_RANGE);
          } else {
            off = __ldg(P.indptr + v);
            d = __ldg(P.indptr + v + 1) - off;
          }
          sm.off[j] = off;
          if (l == 0) P.col0[bstart + j] = v;
        }
        long long tot;
        const long long ex = block_exclusive_scan<long long>(d, (long long*)sm.scr, &tot);
        if (j < T) sm.cstart[j] = (int32_t)ex;
        if (j == 0) sm.misc[1] = tot;
        __syncthreads();
      }
      const int nflat = (int)sm.misc[1];
      const bool cached = nflat <= P.flat_cap;
      // edge e of the flat order: (row id, weight)
      auto edge = [&](int e) -> uint2 {
        if (cached) return __ldcg(flat + e);
        const int c = ls_col(sm, T, e);
        const int64_t pos = sm.off[c] + (e - sm.cstart[c]);
        const float w = P.weights ? __ldg(P.weights + pos) : 1.0f;
        return make_uint2((uint32_t)__ldg(P.indices + pos), __float_as_uint(w));
      };
      // ---- B' = sum fp32(w*w) (COUNT: the edge count); fill the flat cache ----
      double bp = 0.0;
      for (int e0 = threadIdx.x; e0 < nflat; e0 += LS_THREADS * 4) {
        uint2 x[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const int e = e0 + q * LS_THREADS;
          x[q] = make_uint2(LS_EMPTY, 0u);
          if (e < nflat) {
            const int c = ls_col(sm, T, e);
            const int64_t pos = sm.off[c] + (e - sm.cstart[c]);
            const float w = P.weights ? __ldg(P.weights + pos) : 1.0f;
            x[q] = make_uint2((uint32_t)__ldg(P.indices + pos), __float_as_uint(w));
          }
        }
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const int e = e0 + q * LS_THREADS;
          if (e >= nflat) continue;
          if (cached) __stcg(flat + e, x[q]);
          const float w = __uint_as_float(x[q].y);
          bp += ladies ? (double)__fmul_rn(w, w) : 1.0;
        }
      }
      const double Bp = block_reduce_sum<double>(bp, sm.scr);  // syncs: the cache is written
      int NP = (int)max(1, (nflat + LS_PART - 1) / LS_PART);
      // ---- 1 + 2: partition passes, threshold, select ----
      float tau = Bp > 0.0 ? (float)(1.5 * K / Bp) : -1.0f;  // ~1.5K candidates expected
      int nsel = 0;
      double Btot = 0.0;
      bool done = false;
      for (int attempt = 0; attempt < 16 && !done; ++attempt) {
        if (threadIdx.x == 0) { sm.imisc[0] = 0; sm.imisc[2] = 0; }
        double bsum = 0.0;
        int elig = 0;
        for (int p = 0; p < NP; ++p) {
          for (int i = threadIdx.x; i < LS_HT; i += LS_THREADS) {
            sm.hkey[i] = LS_EMPTY;
            sm.hacc[i] = 0.0;
          }
          if (threadIdx.x == 0) sm.imisc[1] = 0;
          __syncthreads();
          for (int e0 = threadIdx.x; e0 < nflat; e0 += LS_THREADS * 4) {
            uint2 x[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const int e = e0 + q * LS_THREADS;
              x[q] = e < nflat ? edge(e) : make_uint2(LS_EMPTY, 0u);
            }
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const uint32_t u = x[q].x;
              if (u == LS_EMPTY || (NP > 1 && ls_part(u, NP) != (uint32_t)p)) continue;
              const int h = ls_insert(sm, u);
              if (h < 0) continue;
              const float w = __uint_as_float(x[q].y);
              atomicAdd(&sm.hacc[h], ladies ? (double)__fmul_rn(w, w) : 1.0);
            }
          }
          __syncthreads();
          if (sm.imisc[1] > LS_HT - LS_HT / 8) break;  // table too full: more partitions
          for (int h = threadIdx.x; h < LS_HT; h += LS_THREADS) {
            const uint32_t u = sm.hkey[h];
            if (u == LS_EMPTY) continue;
            const float bias = (float)sm.hacc[h];
            bsum += (double)bias;
            if (!(bias > 0.0f)) continue;
            ++elig;
            const U4 r = philox(u, 0u, ctr2(l, TAG_ARES_LAYER), gb, P.key);
            if (tau >= 0.0f && !ares_maybe_below(r.x, __fmul_rn(__fmul_rn(tau, bias), 1.01f))) continue;
            const double kk = ares_key(r.x, (double)bias);
            if (tau >= 0.0f && !(kk < (double)tau)) continue;
            const int slot = atomicAdd(&sm.imisc[0], 1);
            if (slot < LS_CB) {
              sm.ckey[slot] = kk;
              sm.cu[slot] = u;
              sm.cb[slot] = bias;
            }
          }
          __syncthreads();
        }
        const bool refill = sm.imisc[1] > LS_HT - LS_HT / 8;
        Btot = block_reduce_sum<double>(bsum, sm.scr);
        const int nelig = (int)block_reduce_sum<long long>(elig, (long long*)sm.scr);
        const int ncand = sm.imisc[0];
        __syncthreads();
        if (refill) {  // a partition overflowed the table: twice the partitions
          NP *= 2;
          continue;
        }
        if (nelig <= K) {
          if (tau >= 0.0f && ncand < nelig) {  // every eligible row is needed (R24)
            tau = -1.0f;
            continue;
          }
          nsel = nelig;
          done = true;
          break;
        }
        if (ncand < K) {  // tau too small
          tau = tau < 0.0f ? -1.0f : tau * 4.0f;
          continue;
        }
        if (ncand > LS_CB) {  // buffer overflow: tau too large
          tau = tau < 0.0f ? (float)(1.5 * K / (Btot > 0.0 ? Btot : 1.0)) : tau * 0.5f;
          continue;
        }
        nsel = K;
        done = true;
        break;
      }
      if (done) {
        // selection by rank counting (no sort network, one barrier): rank of
        // (key, u) among the candidates; the K smallest are then ranked by u
        const int ncand = min(sm.imisc[0], LS_CB);
        int* sel = reinterpret_cast<int*>(sm.hacc);  // free until the S hash below
        for (int i = threadIdx.x; i < ncand; i += LS_THREADS) {
          int r = 0;
          if (nsel < ncand) {
            const double ki = sm.ckey[i];
            const uint32_t ui = sm.cu[i];
            for (int j = 0; j < ncand; ++j) {
              const double kj = sm.ckey[j];
              r += (kj < ki || (kj == ki && sm.cu[j] < ui)) ? 1 : 0;
            }
          }
          sel[i] = r < nsel ? 1 : 0;
        }
        __syncthreads();
        for (int i = threadIdx.x; i < ncand; i += LS_THREADS) {
          if (!sel[i]) continue;
          const uint32_t ui = sm.cu[i];
          int r = 0;
          for (int j = 0; j < ncand; ++j) r += (sel[j] && sm.cu[j] < ui) ? 1 : 0;
          sm.su[r] = ui;
          sm.sp[r] = sm.cb[i];
        }
      }
      if (!done && threadIdx.x == 0 && T > 0 && nflat > 0) atomicOr(P.err, ERR_INTERNAL);
      __syncthreads();
      if (T == 0 || nflat == 0) nsel = 0;
      // ---- S (ascending, ranked above), p(u) = b(u) / B ----
      const float B32 = (float)Btot;
      for (int i = threadIdx.x; i < LS_HT; i += LS_THREADS) sm.hkey[i] = LS_EMPTY;
      if (threadIdx.x < T) {
        sm.cnt[threadIdx.x] = 0;
        sm.cs[threadIdx.x] = 0.0;
      }
      __syncthreads();
      for (int i = threadIdx.x; i < nsel; i += LS_THREADS) {
        const uint32_t u = sm.su[i];
        const float p = __fdiv_rn(sm.sp[i], B32);
        sm.sp[i] = p;
        P.row_map[l][rbase + i] = (int32_t)u;
        P.row_prob[l][rbase + i] = p;
        const int h = ls_insert(sm, u);
        sm.hacc[h] = (double)i;  // local id of u
      }
      __syncthreads();
      // ---- 3a: kept edges per thread (contiguous flat ranges = CSC order),
      // per column count and c_j = sum_fp64 a ----
      const int chunk = (nflat + LS_THREADS - 1) / LS_THREADS;
      const int e_lo = min(nflat, threadIdx.x * chunk), e_hi = min(nflat, e_lo + chunk);
      int kept = 0;
      if (nsel > 0)
        for (int e = e_lo; e < e_hi; ++e) {
          const uint2 x = edge(e);
          const int h = ls_find(sm, x.x);
          if (h < 0) continue;
          const int c = ls_col(sm, T, e);
          atomicAdd(&sm.cnt[c], 1);
          atomicAdd(&sm.cs[c], (double)__fdiv_rn(__uint_as_float(x.y), sm.sp[(int)sm.hacc[h]]));
          ++kept;
        }
      long long ktot;
      const long long kex = block_exclusive_scan<long long>(kept, (long long*)sm.scr, &ktot);
      // column starts (CSC), edge range
      long long E = 0;
      {
        const int j = threadIdx.x;
        const long long c = j < T ? sm.cnt[j] : 0;
        long long tot;
        const long long ex = block_exclusive_scan<long long>(c, (long long*)sm.scr, &tot);
        if (j < T) P.indptr_out[l][ibase + j] = ex;
        E = tot;
      }
      if (threadIdx.x == 0) sm.misc[0] = (long long)atomicAdd(P.edge_ctr + l, (unsigned long long)E);
      __syncthreads();
      const long long ebase = sm.misc[0];
      const bool fits = ebase + E <= P.edge_cap[l];
      if (!fits && threadIdx.x == 0) atomicOr(P.err, ERR_CAPACITY);
      // ---- 3b: emit (the flat order is column-major with ascending positions) ----
      if (fits && kept > 0) {
        long long o = ebase + kex;
        for (int e = e_lo; e < e_hi; ++e) {
          const uint2 x = edge(e);
          const int h = ls_find(sm, x.x);
          if (h < 0) continue;
          const int c = ls_col(sm, T, e);
          const int lid = (int)sm.hacc[h];
          const float a = __fdiv_rn(__uint_as_float(x.y), sm.sp[lid]);
          P.row_local[l][o] = lid;
          P.eid[l][o] = sm.off[c] + (e - sm.cstart[c]);
          P.val[l][o] = __fdiv_rn(a, (float)sm.cs[c]);
          ++o;
        }
      }
      if (threadIdx.x == 0) {
        P.indptr_out[l][ibase + T] = E;
        long long* m = (long long*)(P.meta + (b * P.L + l) * 8);
        m[0] = T; m[1] = nsel; m[2] = fits ? E : 0; m[3] = colbase; m[4] = rbase; m[5] = ibase;
        m[6] = fits ? ebase : 0; m[7] = 0;
      }
      __syncthreads();
      F = P.row_map[l] + rbase;
      colbase = rbase;
      T = nsel;
      (void)lane;
    }
  }
}

static int64_t ls_align(int64_t x) { return (x + 255) & ~int64_t(255); }

size_t layerwise_sm_smem() { return sizeof(LSSmem); }

gs_status run_layerwise_sm(const gs_graph* g, const int32_t* seeds, int64_t num_seeds, int64_t batch_size,
                           int64_t batch_base, const int32_t* n_per_layer, int L, int prob_mode, uint64_t key,
                           cudaStream_t stream, gs_blocks* blk) {
  const Allocator& al = blk->al;
  LSParams P = {};
  P.indptr = g->indptr;
  P.indices = g->indices;
  P.weights = g->weights;
  P.N = g->num_nodes;
  P.seeds = seeds;
  P.num_seeds = num_seeds;
  P.batch_size = batch_size;
  P.num_batches = (num_seeds + batch_size - 1) / batch_size;
  P.batch_base = batch_base;
  P.L = L;
  P.mode = prob_mode;
  P.key = key;
  const int64_t nbatch = P.num_batches;
  for (int l = 0; l < L; ++l) P.K[l] = n_per_layer[l];
  blk->kind = gs_blocks::LAYERWISE;
  blk->num_batches = nbatch;
  blk->num_layers = L;
  blk->stream = stream;
  blk->synced = false;
  auto need = [&](DevBuf& b, int64_t bytes) -> bool {
    return b.ensure(al, (size_t)std::max<int64_t>(bytes, 256), stream);
  };
  bool ok = need(blk->b_col[0], num_seeds * 4);
  int64_t edge_cap[MAX_LAYERS];
  for (int l = 0; l < L && ok; ++l) {
    const int64_t rows = nbatch * (int64_t)P.K[l];
    const int64_t cols = l == 0 ? num_seeds : nbatch * (int64_t)P.K[l - 1];
    int64_t ecap = std::max<int64_t>(int64_t(1) << 16, rows * 4);
    ecap = std::max<int64_t>(ecap, blk->lw_edge_hint[l]);
    ok = ok && need(blk->b_row[l], rows * 4) && need(blk->b_rprob[l], rows * 4) &&
         need(blk->b_indptr[l], (cols + nbatch) * 8) && need(blk->b_rowl[l], ecap * 4) &&
         need(blk->b_eid[l], ecap * 8) && need(blk->b_val[l], ecap * 4);
    if (!ok) break;
    edge_cap[l] = std::min<int64_t>({(int64_t)blk->b_rowl[l].bytes / 4, (int64_t)blk->b_eid[l].bytes / 8,
                                     (int64_t)blk->b_val[l].bytes / 4});
  }
  ok = ok && need(blk->b_meta, nbatch * L * 8 * 8) && need(blk->b_err, 16) &&
       need(blk->b_ctr, ls_align(8 * (MAX_LAYERS + 2)) + 256);
  if (!ok) return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (layer-wise blocks)");
  P.col0 = (int32_t*)blk->b_col[0].ptr;
  for (int l = 0; l < L; ++l) {
    P.row_map[l] = (int32_t*)blk->b_row[l].ptr;
    P.row_prob[l] = (float*)blk->b_rprob[l].ptr;
    P.indptr_out[l] = (int64_t*)blk->b_indptr[l].ptr;
    P.row_local[l] = (int32_t*)blk->b_rowl[l].ptr;
    P.eid[l] = (int64_t*)blk->b_eid[l].ptr;
    P.val[l] = (float*)blk->b_val[l].ptr;
    P.edge_cap[l] = edge_cap[l];
    gs_layer_buffers& lb = blk->layers[l];
    lb = gs_layer_buffers{};
    lb.col_map = l == 0 ? P.col0 : P.row_map[l - 1];
    lb.col_capacity = l == 0 ? num_seeds : nbatch * (int64_t)P.K[l - 1];
    lb.row_map = P.row_map[l];
    lb.row_capacity = nbatch * (int64_t)P.K[l];
    lb.indptr = P.indptr_out[l];
    lb.indptr_capacity = lb.col_capacity + nbatch;
    lb.row_local = P.row_local[l];
    lb.eid = P.eid[l];
    lb.val = P.val[l];
    lb.edge_capacity = edge_cap[l];
    lb.row_prob = P.row_prob[l];
  }
  P.edge_ctr = (unsigned long long*)blk->b_ctr.ptr;
  P.claim = (unsigned int*)((char*)blk->b_ctr.ptr + ls_align(8 * (MAX_LAYERS + 2)));
  const size_t smem = sizeof(LSSmem);
  static int grid = 0;
  if (grid == 0) {
    GS_CUDA_TRY(cudaFuncSetAttribute(layerwise_sm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0, dev = 0, sms = 148;
    GS_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, layerwise_sm_kernel, LS_THREADS, smem));
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    grid = std::max(1, per_sm) * sms;
    if (getenv("GS_VERBOSE")) fprintf(stderr, "layerwise_sm: smem %zu B, %d CTAs/SM\n", smem, per_sm);
  }
  const int nctas = (int)std::max<int64_t>(1, std::min<int64_t>(grid, nbatch));
  // flat edge cache: 64 Ki entries per CTA (a larger A[:, F] is read from the graph)
  P.flat_cap = int64_t(1) << 16;
  if (!blk->b_ws.ensure(al, (size_t)nctas * P.flat_cap * 8, stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (layer-wise edge cache)");
  blk->ws_kind_prev = 0;  // b_ws holds no cleared layout for other samplers now
  blk->ws_stride_prev = -1;
  P.flat = (uint2*)blk->b_ws.ptr;
  P.meta = (int64_t*)blk->b_meta.ptr;
  P.err = (int*)blk->b_err.ptr;
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_err.ptr, 0, 16, stream));
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_ctr.ptr, 0, ls_align(8 * (MAX_LAYERS + 2)) + 256, stream));
  if (nbatch == 0) return GS_OK;
  layerwise_sm_kernel<<<nctas, LS_THREADS, smem, stream>>>(P); count_launch();
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

}  // namespace gsb
