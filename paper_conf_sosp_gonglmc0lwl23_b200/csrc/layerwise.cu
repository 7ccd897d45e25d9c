// layerwise.cu -- layer-wise ECSF sampling: FastGCN (DEGREE), LADIES, COUNT.
//
// collective_sample with the LADIES compute/finalize of
// Fig. 3(b) and Table 2.  One persistent CTA owns one
// mini-batch at a time (super-batch) and runs every layer of it:
//   L1 Extract + Compute (edge-map w*w fused with the row reduction):
//      warp per frontier column, hash-insert every row u of A[:, F] into the
//      CTA's generation-tagged table and accumulate b(u) in fp64 (atomicAdd);
//   L2 candidate compaction: b(u) (LADIES sum w^2 / FastGCN in-degree /
//      COUNT), B = sum b over C, A-Res keys for the eligible (b > 0);
//   L3 Select: all eligible if <= K, else the K smallest (key, u) by an
//      11-bit-digit radix select in shared memory (ties -> smaller u); S
//      sorted ascending (bitonic sort in shared memory);
//   L4 p(u) = b(u)/B for u in S, local ids into the table;
//   L5 Finalize (edge-map divide + column reduction fused): warp per
//      column re-streams A[:, F], keeps rows in S, a_e = w_e / p(u),
//      c_j = sum a (fp64), then emits val_e = a_e / c_j in CSC order.
// The table and candidate arrays live in a per-CTA global workspace (L2
// resident at LADIES sizes); shared memory holds histograms and S.
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "common.cuh"
#include "gs_internal.h"

namespace gsb {

constexpr int LW_THREADS = 1024;  // one CTA per SM: 148 batches in flight keep their tables L2-resident
constexpr int LW_MAX_K = 4096;
constexpr int RADIX_BITS = 11;
constexpr int RADIX_BINS = 1 << RADIX_BITS;

struct LWParams {
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
  unsigned long long* edge_ctr;      // [MAX_LAYERS]
  unsigned long long* need_tab;      // largest table a batch-layer needed
  int64_t* meta;
  int* err;
  char* ws;
  int64_t ws_stride;
  int64_t o_tab, o_acc, o_b, o_cu, o_ckey, o_ch, o_ccnt, o_cc, o_ceoff;
  int64_t tab_cap;  // entries
  uint32_t* gen;
  int maxT;         // largest frontier (batch_size, max K)
  int64_t o_flat;   // per flat edge: table slot of its row (-1: column invalid)
};

struct LWs {
  unsigned long long* tab;
  double* acc;
  float* b;
  int32_t* cu;
  double* ckey;
  int32_t* ch;
  int32_t* ccnt;
  float* cc;
  int32_t* ceoff;
  int32_t* flat;   // [flat edge] table slot of the edge's row
};

__device__ __forceinline__ int lw_log2ceil(int64_t x) {
  int l = 0;
  while ((1ll << l) < x) ++l;
  return l;
}

__device__ __forceinline__ unsigned long long dbits(double d) {
  return (unsigned long long)__double_as_longlong(d);
}

// Flat edge e of the frontier's columns -> column (binary search of the
// column starts in shared memory).
__device__ __forceinline__ int lw_col(const int32_t* fstart, int T, int64_t e) {
  int lo = 0, hi = T - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (fstart[mid] <= e) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

constexpr int LW_ILP = 4;  // flat edges per thread in flight

__global__ void __launch_bounds__(LW_THREADS) layerwise_kernel(LWParams P) {
  extern __shared__ __align__(16) unsigned char lw_dyn[];
  // per frontier column (T <= P.maxT): flat start, indptr, kept count, sum of a
  int32_t* s_fstart = (int32_t*)lw_dyn;
  int64_t* s_off = (int64_t*)(lw_dyn + (((size_t)(P.maxT + 1) * 4 + 7) & ~(size_t)7));
  int32_t* s_cnt = (int32_t*)(s_off + P.maxT);
  double* s_cs = (double*)(s_cnt + P.maxT + (P.maxT & 1));
  __shared__ unsigned long long s_scan[33];
  __shared__ double s_dred[33];
  __shared__ int s_hist[RADIX_BINS];
  __shared__ unsigned long long s_sel[LW_MAX_K];
  __shared__ int s_misc[8];
  __shared__ unsigned long long s_u64[4];

  LWs W;
  char* base = P.ws + (int64_t)blockIdx.x * P.ws_stride;
  W.tab = (unsigned long long*)(base + P.o_tab);
  W.acc = (double*)(base + P.o_acc);
  W.b = (float*)(base + P.o_b);
  W.cu = (int32_t*)(base + P.o_cu);
  W.ckey = (double*)(base + P.o_ckey);
  W.ch = (int32_t*)(base + P.o_ch);
  W.ccnt = (int32_t*)(base + P.o_ccnt);
  W.cc = (float*)(base + P.o_cc);
  W.ceoff = (int32_t*)(base + P.o_ceoff);
  W.flat = (int32_t*)(base + P.o_flat);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
  uint32_t gen = P.gen[blockIdx.x];

  for (int64_t b = blockIdx.x; b < P.num_batches; b += gridDim.x) {
    const int64_t bstart = b * P.batch_size;
    const int64_t nb = min(P.batch_size, P.num_seeds - bstart);
    const uint32_t gb = (uint32_t)(P.batch_base + b);
    const int32_t* F = P.seeds + bstart;
    int64_t T = nb;
    int64_t colbase = bstart;
    for (int l = 0; l < P.L; ++l) {
      const int K = P.K[l];
      const int64_t rbase = b * (int64_t)K;
      const int64_t ibase = colbase + b;
      // ---- frontier: column starts in the flat edge order, table size ----
      {
        int64_t run = 0;
        for (int64_t j0 = 0; j0 < T; j0 += blockDim.x) {
          const int64_t j = j0 + threadIdx.x;
          int64_t d = 0, off = 0;
          if (j < T) {
            const int32_t v = __ldcg(F + j);
            if (v < 0 || (int64_t)v >= P.N) {
              atomicOr(P.err, ERR_SEED_RANGE);
            } else {
              off = __ldg(P.indptr + v);
              d = __ldg(P.indptr + v + 1) - off;
            }
          }
          unsigned long long tot;
          const unsigned long long ex = block_exclusive_scan((unsigned long long)d, s_scan, &tot);
          if (j < T) {
            s_fstart[j] = (int32_t)(run + (int64_t)ex);
            s_off[j] = off;
          }
          run += (int64_t)tot;
        }
        if (threadIdx.x == 0) s_fstart[T] = (int32_t)run;
        s_u64[1] = (unsigned long long)run;
      }
      __syncthreads();
      const int64_t dsum = (int64_t)s_u64[1];
      const int log_cap = lw_log2ceil((dsum * 4) / 3 + 64);
      const int64_t cap = 1ll << log_cap;
      if (cap > P.tab_cap || dsum > P.tab_cap) {
        // does not fit this CTA's workspace: report the size, emit an empty layer
        if (threadIdx.x == 0) {
          atomicOr(P.err, ERR_CAPACITY);
          atomicMax(P.need_tab, (unsigned long long)(cap > dsum ? cap : dsum));
        }
        T = 0;
      }
      const int Ti = (int)T;
      if (gen == 255u) {
        for (int64_t i = threadIdx.x; i < P.tab_cap; i += blockDim.x) W.tab[i] = 0ull;
      }
      gen = (gen % 255u) + 1u;
      if (P.mode != GS_PROB_DEGREE)
        for (int64_t i = threadIdx.x; i < cap && T > 0; i += blockDim.x) W.acc[i] = 0.0;
      __syncthreads();

      // ---- L1: Extract + bias accumulation over the flat edges of A[:, F]
      // (LW_ILP rows in flight per thread); a row's first insert appends it
      // to the candidate list C ----
      if (threadIdx.x == 0) s_misc[4] = 0;
      __syncthreads();
      const int64_t nflat = T > 0 ? dsum : 0;
      for (int64_t e0 = (int64_t)threadIdx.x - lane; e0 < nflat; e0 += (int64_t)blockDim.x * LW_ILP) {
        uint32_t u[LW_ILP];
        float w[LW_ILP];
        bool ok[LW_ILP];
#pragma unroll
        for (int q = 0; q < LW_ILP; ++q) {
          const int64_t e = e0 + (int64_t)q * blockDim.x + lane;
          ok[q] = e < nflat;
          u[q] = 0;
          w[q] = 1.0f;
          if (ok[q]) {
            const int c = lw_col(s_fstart, Ti, e);
            const int64_t pos = s_off[c] + (e - s_fstart[c]);
            u[q] = (uint32_t)__ldg(P.indices + pos);
            if (P.mode == GS_PROB_LADIES && P.weights) w[q] = __ldg(P.weights + pos);
          }
        }
#pragma unroll
        for (int q = 0; q < LW_ILP; ++q) {
          const int64_t e = e0 + (int64_t)q * blockDim.x + lane;
          bool ins = false;
          uint32_t h = 0;
          if (ok[q]) {
            h = tab_insert_once(W.tab, log_cap, gen, u[q], 0u, &ins);
            W.flat[e] = (int32_t)h;
            if (P.mode == GS_PROB_LADIES) atomicAdd(W.acc + h, (double)__fmul_rn(w[q], w[q]));
            else if (P.mode == GS_PROB_COUNT) atomicAdd(W.acc + h, 1.0);
          }
          const uint32_t m = __ballot_sync(0xffffffffu, ins);
          if (m) {
            int slot0 = 0;
            if (lane == 0) slot0 = atomicAdd(&s_misc[4], __popc(m));
            slot0 = __shfl_sync(0xffffffffu, slot0, 0);
            if (ins) {
              const int slot = slot0 + __popc(m & ((1u << lane) - 1u));
              W.cu[slot] = (int32_t)u[q];
              W.ch[slot] = (int32_t)h;
            }
          }
        }
      }
      __syncthreads();
      const int64_t ncand = T > 0 ? s_misc[4] : 0;

      // ---- L2: bias, B, A-Res keys of the candidates (b <= 0: ineligible,
      // key +inf, never selected) ----
      double bsum_local = 0.0;
      int elig_local = 0;
      for (int64_t i = threadIdx.x; i < ncand; i += blockDim.x) {
        const uint32_t u = (uint32_t)__ldcg(W.cu + i);
        const int32_t h = __ldcg(W.ch + i);
        float bias;
        if (P.mode == GS_PROB_DEGREE) bias = (float)(__ldg(P.indptr + u + 1) - __ldg(P.indptr + u));
        else bias = (float)__ldcg(W.acc + h);
        W.b[h] = bias;
        bsum_local += (double)bias;
        double kk = INFINITY;
        if (bias > 0.0f) {
          const U4 r = philox(u, 0u, ctr2(l, TAG_ARES_LAYER), gb, P.key);
          kk = ares_key(r.x, (double)bias);
          ++elig_local;
        }
        W.ckey[i] = kk;
      }
      const double Btot = block_reduce_sum(bsum_local, s_dred);
      const float B32 = (float)Btot;
      const int64_t nelig = (int64_t)block_reduce_sum((double)elig_local, s_dred);
      const int64_t nc = ncand;
      __syncthreads();

      // ---- L3: select the K smallest (key, u) ----
      if (threadIdx.x == 0) s_misc[0] = 0;
      __syncthreads();
      int nsel;
      if (nelig <= K) {  // every eligible candidate (R24)
        for (int64_t i = threadIdx.x; i < nc; i += blockDim.x) {
          if (!(__ldcg(W.ckey + i) < INFINITY)) continue;
          const int slot = atomicAdd(&s_misc[0], 1);
          s_sel[slot] = ((unsigned long long)(uint32_t)__ldcg(W.cu + i) << 32) | (uint32_t)__ldcg(W.ch + i);
        }
        nsel = (int)nelig;
      } else {
        unsigned long long prefix = 0, pmask = 0;
        int remaining = K;
        bool all_bucket = false;
        for (int shift = 64 - RADIX_BITS; shift > -RADIX_BITS; shift -= RADIX_BITS) {
          const int sh = shift < 0 ? 0 : shift;
          const int bits = shift < 0 ? RADIX_BITS + shift : RADIX_BITS;
          const unsigned long long dmask = ((1ull << bits) - 1ull);
          for (int i = threadIdx.x; i < RADIX_BINS; i += blockDim.x) s_hist[i] = 0;
          __syncthreads();
          for (int64_t i = threadIdx.x; i < nc; i += blockDim.x) {
            const unsigned long long kb = dbits(__ldcg(W.ckey + i));
            if ((kb & pmask) == prefix) atomicAdd(&s_hist[(kb >> sh) & dmask], 1);
          }
          __syncthreads();
          // find the digit whose cumulative count reaches `remaining`
          if (warp == 0) {
            int run = 0, found = -1, before = 0;
            for (int c0 = 0; c0 < RADIX_BINS && found < 0; c0 += 32) {
              const int hv = s_hist[c0 + lane];
              const int inc = warp_inclusive_scan(hv);
              const unsigned m = __ballot_sync(0xffffffffu, run + inc >= remaining);
              if (m) {
                const int ln = __ffs(m) - 1;
                found = c0 + ln;
                before = run + __shfl_sync(0xffffffffu, inc - hv, ln);
              }
              run += __shfl_sync(0xffffffffu, inc, 31);
            }
            if (lane == 0) {
              s_misc[1] = found;
              s_misc[2] = before;
              s_misc[3] = s_hist[found];
            }
          }
          __syncthreads();
          const int dig = s_misc[1];
          remaining -= s_misc[2];
          prefix |= (unsigned long long)dig << sh;
          pmask |= dmask << sh;
          if (s_misc[3] == remaining) {
            all_bucket = true;
            break;
          }
          if (sh == 0) break;
        }
        // gather: strictly below the bucket, plus the bucket (all, or the
        // `remaining` smallest u among exact ties)
        for (int64_t i = threadIdx.x; i < nc; i += blockDim.x) {
          const unsigned long long kb = dbits(__ldcg(W.ckey + i));
          const unsigned long long hi = kb & pmask;
          bool take = hi < prefix;
          if (hi == prefix) {
            if (all_bucket) {
              take = true;
            } else {
              // exact tie on the full key: rank by u among the ties
              const uint32_t ui = (uint32_t)__ldcg(W.cu + i);
              int rank = 0;
              for (int64_t t = 0; t < nc; ++t) {
                if (dbits(__ldcg(W.ckey + t)) == kb && (uint32_t)__ldcg(W.cu + t) < ui) ++rank;
              }
              take = rank < remaining;
            }
          }
          if (take) {
            const int slot = atomicAdd(&s_misc[0], 1);
            s_sel[slot] = ((unsigned long long)(uint32_t)__ldcg(W.cu + i) << 32) | (uint32_t)__ldcg(W.ch + i);
          }
        }
        __syncthreads();
        nsel = K;
      }
      __syncthreads();
      // bitonic sort of s_sel[0, nsel) ascending (u in the high word)
      int n2 = 1;
      while (n2 < nsel) n2 <<= 1;
      for (int i = nsel + threadIdx.x; i < n2; i += blockDim.x) s_sel[i] = ~0ull;
      __syncthreads();
      for (int kk = 2; kk <= n2; kk <<= 1) {
        for (int jj = kk >> 1; jj > 0; jj >>= 1) {
          for (int i = threadIdx.x; i < n2; i += blockDim.x) {
            const int ixj = i ^ jj;
            if (ixj > i) {
              const unsigned long long a = s_sel[i], c = s_sel[ixj];
              const bool up = (i & kk) == 0;
              if ((a > c) == up) {
                s_sel[i] = c;
                s_sel[ixj] = a;
              }
            }
          }
          __syncthreads();
        }
      }

      // ---- L4: row_map = S, p(u) = b(u) / B, local ids into the table ----
      for (int i = threadIdx.x; i < nsel; i += blockDim.x) {
        const uint32_t u = (uint32_t)(s_sel[i] >> 32);
        const uint32_t h = (uint32_t)(s_sel[i] & 0xffffffffu);
        const float p = __fdiv_rn(__ldcg(W.b + h), B32);
        W.b[h] = p;
        W.tab[h] = tab_entry(gen, u, (uint32_t)i + 1u);
        P.row_map[l][rbase + i] = (int32_t)u;
        P.row_prob[l][rbase + i] = p;
      }
      __syncthreads();

      // ---- L5a: per column kept count and c_j = sum_fp64 a over its kept
      // edges (flat edges, slots staged by L1: no second hash probe) ----
      for (int j = threadIdx.x; j < Ti; j += blockDim.x) {
        s_cnt[j] = 0;
        s_cs[j] = 0.0;
      }
      __syncthreads();
      for (int64_t e0 = threadIdx.x; e0 < nflat; e0 += (int64_t)blockDim.x * LW_ILP) {
        int32_t h[LW_ILP];
#pragma unroll
        for (int q = 0; q < LW_ILP; ++q) {
          const int64_t e = e0 + (int64_t)q * blockDim.x;
          h[q] = e < nflat ? __ldcg(W.flat + e) : -1;
        }
        uint32_t val[LW_ILP];
        float pb[LW_ILP], w[LW_ILP];
#pragma unroll
        for (int q = 0; q < LW_ILP; ++q) {
          val[q] = h[q] >= 0 ? tab_val(__ldcg(W.tab + h[q])) : 0u;
          pb[q] = val[q] ? __ldcg(W.b + h[q]) : 1.0f;
          w[q] = 1.0f;
          const int64_t e = e0 + (int64_t)q * blockDim.x;
          if (val[q] && P.weights) {
            const int c = lw_col(s_fstart, Ti, e);
            w[q] = __ldg(P.weights + s_off[c] + (e - s_fstart[c]));
          }
        }
#pragma unroll
        for (int q = 0; q < LW_ILP; ++q) {
          if (!val[q]) continue;
          const int64_t e = e0 + (int64_t)q * blockDim.x;
          const int c = lw_col(s_fstart, Ti, e);
          atomicAdd(&s_cnt[c], 1);
          atomicAdd(&s_cs[c], (double)__fdiv_rn(w[q], pb[q]));
        }
      }
      __syncthreads();
      int64_t E = 0;
      for (int j0 = 0; j0 < Ti; j0 += blockDim.x) {
        const int j = j0 + threadIdx.x;
        const unsigned long long cv = j < Ti ? (unsigned long long)s_cnt[j] : 0ull;
        unsigned long long tot;
        const unsigned long long ex = block_exclusive_scan(cv, s_scan, &tot);
        if (j < Ti) W.ceoff[j] = (int32_t)(E + (int64_t)ex);
        E += (int64_t)tot;
      }
      if (threadIdx.x == 0) s_u64[0] = atomicAdd(P.edge_ctr + l, (unsigned long long)E);
      __syncthreads();
      const int64_t ebase = (int64_t)s_u64[0];
      const bool fits = ebase + E <= P.edge_cap[l];
      if (!fits && threadIdx.x == 0) atomicOr(P.err, ERR_CAPACITY);
      for (int64_t j = threadIdx.x; j < T; j += blockDim.x) {
        P.indptr_out[l][ibase + j] = __ldcg(W.ceoff + j);
        if (l == 0) P.col0[bstart + j] = __ldcg(F + j);
      }

      // ---- L5b: emit the block in CSC order: the flat order is column-major
      // with ascending positions, so an exclusive scan of the keep flags over
      // the flat edges is each kept edge's output index ----
      int64_t krun = 0;
      for (int64_t e0 = 0; e0 < nflat && fits; e0 += (int64_t)blockDim.x * LW_ILP) {
        // thread t owns flat edges e0 + t*LW_ILP .. + LW_ILP-1 (contiguous)
        const int64_t eb = e0 + (int64_t)threadIdx.x * LW_ILP;
        int32_t h[LW_ILP];
        uint32_t val[LW_ILP];
        int kc = 0;
#pragma unroll
        for (int q = 0; q < LW_ILP; ++q) h[q] = eb + q < nflat ? __ldcg(W.flat + eb + q) : -1;
#pragma unroll
        for (int q = 0; q < LW_ILP; ++q) {
          val[q] = h[q] >= 0 ? tab_val(__ldcg(W.tab + h[q])) : 0u;
          kc += val[q] ? 1 : 0;
        }
        unsigned long long tot;
        const unsigned long long ex = block_exclusive_scan((unsigned long long)kc, s_scan, &tot);
        int64_t o = ebase + krun + (int64_t)ex;
#pragma unroll
        for (int q = 0; q < LW_ILP; ++q) {
          if (!val[q]) continue;
          const int64_t e = eb + q;
          const int c = lw_col(s_fstart, Ti, e);
          const int64_t pos = s_off[c] + (e - s_fstart[c]);
          const float w = P.weights ? __ldg(P.weights + pos) : 1.0f;
          const float a = __fdiv_rn(w, __ldcg(W.b + h[q]));
          P.row_local[l][o] = (int32_t)(val[q] - 1u);
          P.eid[l][o] = pos;
          P.val[l][o] = __fdiv_rn(a, (float)s_cs[c]);
          ++o;
        }
        krun += (int64_t)tot;
      }
      if (threadIdx.x == 0) {
        P.indptr_out[l][ibase + T] = E;
        long long* m = (long long*)(P.meta + (b * P.L + l) * 8);
        // an overflowed block wrote no edges: record it empty (GS_ERR_CAPACITY is raised)
        m[0] = T; m[1] = nsel; m[2] = fits ? E : 0; m[3] = colbase; m[4] = rbase; m[5] = ibase;
        m[6] = fits ? ebase : 0; m[7] = 0;
      }
      __syncthreads();
      F = P.row_map[l] + rbase;
      colbase = rbase;
      T = nsel;
    }
  }
  if (threadIdx.x == 0) P.gen[blockIdx.x] = gen;
}

static int64_t align256(int64_t x) { return (x + 255) & ~int64_t(255); }

gs_status run_layerwise_old(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                            int64_t batch_size, int64_t batch_base, const int32_t* n_per_layer,
                            int L, int prob_mode, uint64_t key, cudaStream_t stream, gs_blocks* blk);
size_t layerwise_bm_smem(int64_t N, int maxT, int* gw_log_out, int* ng_out, int64_t* n4_out);
gs_status run_layerwise_bm(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                           int64_t batch_size, int64_t batch_base, const int32_t* n_per_layer,
                           int L, int prob_mode, uint64_t key, cudaStream_t stream, gs_blocks* blk,
                           size_t smem, int gw_log, int ng, int64_t n4);

// Chooses the kernel.  FastGCN (DEGREE): the bitmap kernel (layerwise_bm.cu)
// when the candidate bitmaps of one CTA per SM fit (N/8 bytes each, <= 2 GB
// in all) and its rank prefixes fit shared memory -- hub-biased frontiers give
// ~280 k candidates per batch-layer (measured on LJ: 282 ms vs 514 ms).
// LADIES / COUNT (~10 k candidates) with K and batch size <= 1024: the
// shared-memory kernel of layerwise_sm.cu; larger: the global hash-table
// kernel below (31 ms vs 69 ms for the bitmap kernel on LJ).
// GS_LW_PATH=old|bm forces one (experiments / tests).
gs_status run_layerwise_sm(const gs_graph* g, const int32_t* seeds, int64_t num_seeds, int64_t batch_size,
                           int64_t batch_base, const int32_t* n_per_layer, int L, int prob_mode, uint64_t key,
                           cudaStream_t stream, gs_blocks* blk);

gs_status run_layerwise(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                        int64_t batch_size, int64_t batch_base, const int32_t* n_per_layer,
                        int L, int prob_mode, uint64_t key, cudaStream_t stream, gs_blocks* blk) {
  {
    // LADIES / COUNT with frontiers and K <= 1024: every per-batch table in
    // shared memory, the extracted edges in registers (layerwise_sm.cu)
    int maxK0 = 1;
    for (int l = 0; l < L; ++l) maxK0 = std::max(maxK0, n_per_layer[l]);
    const char* path0 = getenv("GS_LW_PATH");
    const bool sm_ok = prob_mode != GS_PROB_DEGREE && maxK0 <= 1024 && batch_size <= 1024 && !blk->lw_big;
    const bool forced_other = path0 && (!strcmp(path0, "old") || !strcmp(path0, "bm"));
    if (sm_ok && !forced_other)
      return run_layerwise_sm(g, seeds, num_seeds, batch_size, batch_base, n_per_layer, L, prob_mode, key,
                              stream, blk);
  }
  {
    int maxK = 1;
    for (int l = 0; l < L; ++l) maxK = std::max(maxK, n_per_layer[l]);
    const int maxT = (int)std::max<int64_t>(batch_size, maxK);
    int gw_log = 0, ng = 0;
    int64_t n4 = 0;
    const size_t smem = layerwise_bm_smem(g->num_nodes, maxT, &gw_log, &ng, &n4);
    const char* path = getenv("GS_LW_PATH");
    bool bm = prob_mode == GS_PROB_DEGREE && smem > 0 && n4 * 16 * 148 <= (int64_t(2) << 30) &&
              maxK <= 4096;
    if (path && !strcmp(path, "old")) bm = false;
    if (path && !strcmp(path, "bm") && smem > 0) bm = true;
    if (bm)
      return run_layerwise_bm(g, seeds, num_seeds, batch_size, batch_base, n_per_layer, L, prob_mode,
                              key, stream, blk, smem, gw_log, ng, n4);
  }
  return run_layerwise_old(g, seeds, num_seeds, batch_size, batch_base, n_per_layer, L, prob_mode,
                           key, stream, blk);
}

gs_status run_layerwise_old(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                            int64_t batch_size, int64_t batch_base, const int32_t* n_per_layer,
                            int L, int prob_mode, uint64_t key, cudaStream_t stream, gs_blocks* blk) {
  const Allocator& al = blk->al;
  LWParams P = {};
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
  int maxK = 1;
  int64_t col_cap = batch_size;
  for (int l = 0; l < L; ++l) {
    P.K[l] = n_per_layer[l];
    maxK = std::max(maxK, n_per_layer[l]);
    col_cap = std::max<int64_t>(col_cap, n_per_layer[l]);
  }
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
       need(blk->b_ctr, 8 * (MAX_LAYERS + 2));
  if (!ok) return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (layer-wise blocks)");

  // ---- per-CTA workspace ----
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  P.maxT = (int)std::max<int64_t>(batch_size, maxK);
  const size_t dyn = (((size_t)(P.maxT + 1) * 4 + 7) & ~(size_t)7) + (size_t)P.maxT * 8 +
                     (size_t)(P.maxT + (P.maxT & 1)) * 4 + (size_t)P.maxT * 8;
  GS_CUDA_TRY(cudaFuncSetAttribute(layerwise_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)dyn));
  int per_sm = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, layerwise_kernel, LW_THREADS, dyn);
  per_sm = std::max(1, per_sm);
  const int nctas = (int)std::max<int64_t>(1, std::min<int64_t>(nbatch, (int64_t)sms * per_sm));
  int64_t tab_cap = std::max<int64_t>(int64_t(1) << 15, blk->lw_tab_hint);
  int64_t tc = 1;
  while (tc < tab_cap) tc <<= 1;
  tab_cap = tc;
  int64_t o = 0;
  P.o_tab = o; o = align256(o + tab_cap * 8);
  P.o_acc = o; o = align256(o + tab_cap * 8);
  P.o_b = o; o = align256(o + tab_cap * 4);
  P.o_cu = o; o = align256(o + tab_cap * 4);
  P.o_ckey = o; o = align256(o + tab_cap * 8);
  P.o_ch = o; o = align256(o + tab_cap * 4);
  P.o_ccnt = o; o = align256(o + col_cap * 4);
  P.o_cc = o; o = align256(o + col_cap * 4);
  P.o_ceoff = o; o = align256(o + col_cap * 4);
  P.o_flat = o; o = align256(o + tab_cap * 4);
  P.ws_stride = o;
  P.tab_cap = tab_cap;
  const size_t ws_bytes = (size_t)o * nctas;
  const bool grow = blk->b_ws.bytes < ws_bytes;
  if (!blk->b_ws.ensure(al, ws_bytes, stream, true) || !blk->b_gen.ensure(al, 4096 * 4, stream, true))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (layer-wise workspace)");
  if (grow || blk->ws_stride_prev != P.ws_stride || blk->ws_kind_prev != 2) {
    GS_CUDA_TRY(cudaMemsetAsync(blk->b_ws.ptr, 0, blk->b_ws.bytes, stream));
    GS_CUDA_TRY(cudaMemsetAsync(blk->b_gen.ptr, 0, 4096 * 4, stream));
  }
  blk->ws_stride_prev = P.ws_stride;
  blk->ws_kind_prev = 2;
  P.ws = (char*)blk->b_ws.ptr;
  P.gen = (uint32_t*)blk->b_gen.ptr;
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
  P.need_tab = P.edge_ctr + MAX_LAYERS;
  P.meta = (int64_t*)blk->b_meta.ptr;
  P.err = (int*)blk->b_err.ptr;
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_err.ptr, 0, 16, stream));
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_ctr.ptr, 0, 8 * (MAX_LAYERS + 2), stream));
  if (nbatch == 0) return GS_OK;
  layerwise_kernel<<<nctas, LW_THREADS, dyn, stream>>>(P); count_launch();
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

}  // namespace gsb
