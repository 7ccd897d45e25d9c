// layerwise_bm.cu -- layer-wise ECSF sampling (FastGCN / LADIES / COUNT) with
// the candidate set C of a batch-layer held as an N-bit row bitmap.
//
// collective_sample with the compute/finalize of Fig. 3(b)
// (P:207-229), Table 2 and the FastGCN degree pre-processing
// (P:300).  Same results as layerwise.cu (R7, R9, R24); what
// differs is where the per-batch state lives.  layerwise.cu keys a hash table
// by row and stages a table slot per streamed edge: for FastGCN's hub-biased
// frontiers (~365 k edges, ~280 k candidates per batch-layer) that is ~11 MB
// of random-access state per CTA, so 148 CTAs thrash L2 and every probe is a
// 128-byte HBM line (profiles/r01_random_access_probe.md).  Here one persistent
// 1024-thread CTA per SM owns one mini-batch at a time and keeps:
//   * C as an N-bit bitmap in global memory (N/8 bytes per CTA: 0.6 MB for
//     the LJ-shaped graph, L2-resident), set by fire-and-forget red.or;
//   * a rank prefix per group of GW bitmap words in shared memory, so the rank
//     of a candidate (its index in ascending-id order) is one smem load plus
//     the popcounts of <= GW-1 words;
//   * b(u) for LADIES / COUNT in a rank-indexed fp64 array (|C| entries);
//   * the A-Res candidates, S and a hash of S in shared memory.
// Per batch-layer:
//   L1 Extract: stream A[:, F] (flat edges, ILP 4), set the rows' bits;
//   L2 ranks: warp-contiguous scan of the bitmap -> group prefixes (+ FastGCN:
//      b(u) = in-degree from the a0 degree array, B = sum b, eligible count);
//   L3 (LADIES / COUNT) Compute: stream A[:, F] again, b(rank(u)) += w*w / 1
//      (fp64 atomics, the edge-map + row reduce of Fig. 3(b) lines 2-3);
//   L4 Select: every eligible candidate if <= K, else the K smallest A-Res
//      keys E_u / b(u): a threshold tau = 2K/B keeps ~2K candidates (cheap
//      float pre-test, exact fp64 key only for survivors) in shared memory,
//      which are sorted by (key, u); S sorted by u; p(u) = b(u)/B;
//   L5 Finalize: stream A[:, F], keep rows in S (smem hash), per column count
//      and c_j = sum_fp64 a_e (a_e = w_e / p(u)), then emit the block in CSC
//      order with val_e = a_e / c_j (flat keep-scan).
// The bitmap and b(u) are cleared by the CTA after the select.
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include <algorithm>
#include <cstdlib>

#include "common.cuh"
#include "gs_internal.h"
#include "nodewise_common.cuh"

namespace gsb {

constexpr int LB_THREADS = 1024;
constexpr int LB_WARPS = LB_THREADS / 32;
constexpr int LB_CAP = 4096;        // A-Res candidate buffer (select), >= max K
constexpr int LB_HS = 8192;         // hash of S (aliases the candidate buffer)
constexpr int LB_ILP = 4;           // flat edges per thread in flight
constexpr int LB_ILP5 = 8;          // ... in the finalize re-stream (L5a)
constexpr int LB_MAX_K = 4096;
constexpr int LB_SCAP = 512;        // kept edges a warp stages in L5a (more: L5b streams again)
constexpr int LB_CCAP = 512;        // FastGCN: candidate-row edges a warp stages in L1 (more: L5a streams again)

struct LBParams {
  const int64_t* indptr;
  const int32_t* indices;
  const float* weights;
  const int32_t* deg;               // a0: in-degree per node (FastGCN)
  const int32_t* degsrc;            // a0: deg[indices[e]] per CSC entry (FastGCN), or null
  int64_t N;
  const int32_t* seeds;
  int64_t num_seeds, batch_size, num_batches, batch_base;
  int L;
  int K[MAX_LAYERS];
  int mode;
  uint64_t key;
  PhiloxKeys pk;
  int32_t* col0;
  int32_t* row_map[MAX_LAYERS];
  float* row_prob[MAX_LAYERS];
  int64_t* indptr_out[MAX_LAYERS];
  int32_t* row_local[MAX_LAYERS];
  int64_t* eid[MAX_LAYERS];
  float* val[MAX_LAYERS];
  int64_t edge_cap[MAX_LAYERS];
  unsigned long long* edge_ctr;     // [MAX_LAYERS] bump allocators of the edge ranges
  unsigned long long* need_tab;     // largest |C| a batch-layer needed (LADIES / COUNT)
  int64_t* meta;
  int* err;
  uint32_t* bm;                     // [CTA][n4 * 4] row bitmaps (zero between batch-layers)
  int64_t n4;                       // uint4 per bitmap (a multiple of GW / 4)
  double* acc;                      // [CTA][acc_cap] b(u) by rank (zero between uses)
  int64_t acc_cap;
  int64_t* stg_pos;                 // [CTA][warp][LB_SCAP] kept edges staged by L5a: position,
  int32_t* stg_lid;                 //   local row, column, a = w / p(u)
  int32_t* stg_col;
  float* stg_a;
  int scap;                         // staged kept edges per warp (<= LB_SCAP)
  int64_t* cnd_pos;                 // [CTA][warp][LB_CCAP] FastGCN: L1's edges whose row's key is below
  int32_t* cnd_u;                   //   the previous batch's threshold: position, row, column
  int32_t* cnd_col;
  int ccap;
  int gw_log;                       // log2 words per rank group (>= 2)
  int ng;                           // rank groups per bitmap
  int maxT;
};

struct LBShared {
  unsigned long long scan[33];
  double dred[33];
  int misc[8];
  unsigned long long u64[4];
  double tau_est[MAX_LAYERS];       // FastGCN: select threshold estimate per layer (previous batch)
  int wtot[LB_WARPS];
  int cfill[LB_WARPS];              // FastGCN: candidate-row edges each warp staged in L1
  int cstage_ovf;
};

__device__ __forceinline__ int lb_col(const int32_t* fstart, int T, int64_t e) {
  int lo = 0, hi = T - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (fstart[mid] <= e) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

// Flat-edge stream of one warp: a contiguous range of the batch-layer's flat
// edge space (column-major, positions ascending), 32 * LB_ILP edges per round.
// The column of each lane's edge is tracked incrementally (one binary search
// per warp range, then a forward walk over the column starts).
struct LBStream {
  int64_t beg, end;
  int c;
  __device__ __forceinline__ LBStream(int64_t nflat) {
    const int warp = threadIdx.x >> 5;
    int64_t per = (nflat + LB_WARPS - 1) / LB_WARPS;
    per = (per + 31) & ~int64_t(31);
    beg = min((int64_t)warp * per, nflat);
    end = min(beg + per, nflat);
    c = -1;
  }
  // column of flat edge e (e < end, visited in increasing order per lane)
  __device__ __forceinline__ int col(const int32_t* fstart, int T, int64_t e) {
    if (c < 0) c = lb_col(fstart, T, e);
    while (fstart[c + 1] <= e) ++c;
    return c;
  }
};

__device__ __forceinline__ int popc4(const uint4& x) {
  return __popc(x.x) + __popc(x.y) + __popc(x.z) + __popc(x.w);
}

__device__ __forceinline__ uint32_t word4(const uint4& x, int j) {
  return j == 0 ? x.x : (j == 1 ? x.y : (j == 2 ? x.z : x.w));
}

// Rank of row u in the batch-layer's candidate set (ascending ids).
__device__ __forceinline__ int64_t lb_rank(const LBParams& P, const uint32_t* bm, const int32_t* s_gp,
                                           uint32_t u) {
  const int64_t wi = u >> 5;
  const int64_t g = wi >> P.gw_log;
  int64_t r = s_gp[g];
  for (int64_t k = g << P.gw_log; k < wi; ++k) r += __popc(__ldcg(bm + k));
  return r + __popc(__ldcg(bm + wi) & ((1u << (u & 31)) - 1u));
}

// Walks the set bits of the bitmap in warp-contiguous ranges of rank groups:
// f(u, rank) for every candidate.  Ranks come from s_gp (built by lb_ranks).
template <class Fn>
__device__ __forceinline__ void lb_for_bits(const LBParams& P, const uint4* bm4, const int32_t* s_gp,
                                            Fn f) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int gq = 1 << (P.gw_log - 2);            // uint4 per group
  const int gpw = (P.ng + LB_WARPS - 1) / LB_WARPS;
  const int64_t i_beg = (int64_t)min(warp * gpw, P.ng) * gq;
  const int64_t i_end = (int64_t)min((warp + 1) * gpw, P.ng) * gq;
  for (int64_t i0 = i_beg; i0 < i_end; i0 += 32) {
    const int64_t i = i0 + lane;
    const uint4 x = i < i_end ? __ldcg(bm4 + i) : make_uint4(0, 0, 0, 0);
    const int pc = popc4(x);
    const int inc = warp_inclusive_scan(pc);
    const int first = lane - (lane & (gq - 1));  // first lane of this lane's group
    const int ex_first = __shfl_sync(0xffffffffu, inc, first) - __shfl_sync(0xffffffffu, pc, first);
    if (pc == 0) continue;
    int64_t r = (int64_t)s_gp[i >> (P.gw_log - 2)] + (inc - pc - ex_first);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      uint32_t w = word4(x, j);
      while (w) {
        const int bpos = __ffs(w) - 1;
        w &= w - 1u;
        f((uint32_t)((i * 4 + j) * 32 + bpos), r);
        ++r;
      }
    }
  }
}

// Candidate buffer of the select (shared memory).
struct LBBuf {
  unsigned long long* k;  // exact fp64 key bits
  uint32_t* u;
  float* b;
};

// s_gp[g] = number of candidates before rank group g; returns |C|.  FastGCN:
// also b(u) = deg(u) summed (B, fp64) and the eligible count, and -- with a
// threshold estimate tau_est > 0 (from the CTA's previous batch at this
// layer) -- every candidate with exact key < tau_est appended to the buffer
// (counter sh.misc[6]), so that usually no second pass over C is needed.
__device__ int64_t lb_ranks(const LBParams& P, LBShared& sh, const uint4* bm4, int32_t* s_gp,
                            bool degree, double* B_out, int64_t* nelig_out, double tau_est, int l,
                            uint32_t gb, const LBBuf& buf) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int gq = 1 << (P.gw_log - 2);
  const int gpw = (P.ng + LB_WARPS - 1) / LB_WARPS;
  const int g_beg = min(warp * gpw, P.ng), g_end = min((warp + 1) * gpw, P.ng);
  const int64_t i_beg = (int64_t)g_beg * gq, i_end = (int64_t)g_end * gq;
  int run = 0;
  long long bsum = 0;  // B = sum of integer in-degrees (exact; = the oracle's fp64 sum)
  int elig = 0;
  const float tau_f = (float)tau_est;
  for (int64_t i0 = i_beg; i0 < i_end; i0 += 32) {
    const int64_t i = i0 + lane;
    const uint4 x = i < i_end ? __ldcg(bm4 + i) : make_uint4(0, 0, 0, 0);
    const int pc = popc4(x);
    const int inc = warp_inclusive_scan(pc);
    if (i < i_end && (lane & (gq - 1)) == 0) s_gp[i >> (P.gw_log - 2)] = run + inc - pc;
    const int total = __shfl_sync(0xffffffffu, inc, 31);
    run += total;
    if (!degree) continue;
    // the warp's candidates, 32 at a time across the lanes (balanced: no lane
    // walks its own bits while the others wait): candidate k -> its owner lane
    // (binary search of the inclusive scan) and bit (fns)
    auto locate = [&](int k) -> uint32_t {  // the warp's k-th candidate (all lanes call)
      int o = 0;
#pragma unroll
      for (int step = 16; step > 0; step >>= 1) {
        const int ip = __shfl_sync(0xffffffffu, inc, o + step - 1);
        if (ip <= k) o += step;
      }
      const uint32_t w0 = __shfl_sync(0xffffffffu, x.x, o), w1 = __shfl_sync(0xffffffffu, x.y, o);
      const uint32_t w2 = __shfl_sync(0xffffffffu, x.z, o), w3 = __shfl_sync(0xffffffffu, x.w, o);
      const int ex_o = __shfl_sync(0xffffffffu, inc - pc, o);
      if (k >= total) return 0xFFFFFFFFu;
      int r = k - ex_o;
      int j = 0;
      uint32_t wd = w0;
      const int p0 = __popc(w0), p1 = __popc(w1), p2 = __popc(w2);
      if (r >= p0) { r -= p0; j = 1; wd = w1;
        if (r >= p1) { r -= p1; j = 2; wd = w2;
          if (r >= p2) { r -= p2; j = 3; wd = w3; } } }
      uint32_t bpos;
      asm("fns.b32 %0, %1, 0, %2;" : "=r"(bpos) : "r"(wd), "r"(r + 1));
      return (uint32_t)(((i0 + o) * 4 + j) * 32 + bpos);
    };
    auto take = [&](uint32_t u, int32_t dg) {
      bsum += dg;
      elig += dg > 0 ? 1 : 0;
      if (tau_est > 0.0 && dg > 0) {
        const float bb = (float)dg;
        const uint32_t R = philox_k(u, 0u, ctr2(l, TAG_ARES_LAYER), gb, P.pk).x;
        if (ares_maybe_below(R, __fmul_rn(__fmul_rn(tau_f, bb), 1.01f))) {
          const double kk = ares_key(R, (double)bb);
          if (kk < tau_est) {
            const int slot = atomicAdd(&sh.misc[6], 1);
            if (slot < LB_CAP) {
              buf.k[slot] = (unsigned long long)__double_as_longlong(kk);
              buf.u[slot] = u;
              buf.b[slot] = bb;
            }
          }
        }
      }
    };
    // two candidates per lane in flight (their degree loads overlap)
    for (int k0 = 0; k0 < total; k0 += 64) {
      const uint32_t ua = locate(k0 + lane), ub = locate(k0 + 32 + lane);
      const int32_t da = ua != 0xFFFFFFFFu ? __ldg(P.deg + ua) : 0;
      const int32_t db = ub != 0xFFFFFFFFu ? __ldg(P.deg + ub) : 0;
      if (ua != 0xFFFFFFFFu) take(ua, da);
      if (ub != 0xFFFFFFFFu) take(ub, db);
    }
  }
  if (lane == 0) sh.wtot[warp] = run;
  __syncthreads();
  if (warp == 0) {
    const int v = sh.wtot[lane];
    const int inc = warp_inclusive_scan(v);
    sh.wtot[lane] = inc - v;
    if (lane == 31) sh.misc[5] = inc;
  }
  __syncthreads();
  const int off = sh.wtot[warp];
  for (int g = g_beg + lane; g < g_end; g += 32) s_gp[g] += off;
  if (warp == 0 && lane == 0) s_gp[P.ng] = sh.misc[5];
  const int64_t total = sh.misc[5];
  if (degree) {
    *B_out = (double)block_reduce_sum((unsigned long long)bsum, sh.scan);
    *nelig_out = (int64_t)block_reduce_sum((double)elig, sh.dred);
  } else {
    __syncthreads();
  }
  return total;
}

__device__ __forceinline__ double block_reduce_max(double v, double* scratch) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmax(v, __shfl_xor_sync(0xffffffffu, v, o));
  if (lane == 0) scratch[wid] = v;
  __syncthreads();
  double r = 0.0;
  for (int w = 0; w < nw; ++w) r = fmax(r, scratch[w]);
  __syncthreads();
  return r;
}

// Counting-sort rank of n <= LB_CAP items on LB_THREADS bins (bin(i) monotone
// in the order; less(j, i) the exact order inside a bin): rank[i] for every
// item with take(i).  Every thread of the CTA calls it.
template <class Bin, class Less, class Take>
__device__ __forceinline__ void lb_csrank(int n, int* hist, int* fill, int16_t* ord, int16_t* rank, Bin bin,
                                          Less less, Take take, unsigned long long* scan) {
  const int t = threadIdx.x;
  hist[t] = 0;
  fill[t] = 0;
  __syncthreads();
  for (int i = t; i < n; i += LB_THREADS)
    if (take(i)) atomicAdd(&hist[bin(i)], 1);
  __syncthreads();
  unsigned long long tot;
  const int c = hist[t];
  const int st = (int)block_exclusive_scan<unsigned long long>((unsigned long long)c, scan, &tot);
  hist[t] = st;
  __syncthreads();
  for (int i = t; i < n; i += LB_THREADS)
    if (take(i)) {
      const int bb = bin(i);
      ord[hist[bb] + atomicAdd(&fill[bb], 1)] = (int16_t)i;
    }
  __syncthreads();
  for (int i = t; i < n; i += LB_THREADS)
    if (take(i)) {
      const int bb = bin(i), s0 = hist[bb], s1 = s0 + fill[bb];
      int r = s0;
      for (int k = s0; k < s1; ++k) r += less(ord[k], i) ? 1 : 0;
      rank[i] = (int16_t)r;
    }
  __syncthreads();
}

__device__ __forceinline__ uint32_t lb_hash(uint32_t u) { return (u * 0x9E3779B1u) >> 19; }  // 13 bits

__device__ __forceinline__ int lb_lookup(const int32_t* hk, const int32_t* hv, uint32_t u) {
  uint32_t h = lb_hash(u);
  while (true) {
    const int32_t k = hk[h];
    if (k == (int32_t)u) return hv[h];
    if (k < 0) return -1;
    h = (h + 1) & (LB_HS - 1);
  }
}

__global__ void __launch_bounds__(LB_THREADS, 1) layerwise_bm_kernel(LBParams P) {
  extern __shared__ __align__(16) unsigned char lb_dyn[];
  __shared__ LBShared sh;
  // dynamic smem: candidate buffer (keys, ids, biases; later the hash of S),
  // S, per-column arrays, rank-group prefixes
  unsigned long long* s_bk = (unsigned long long*)lb_dyn;            // [LB_CAP]
  uint32_t* s_bu = (uint32_t*)(s_bk + LB_CAP);                       // [LB_CAP]
  float* s_bb = (float*)(s_bu + LB_CAP);                             // [LB_CAP]
  int32_t* s_hk = (int32_t*)lb_dyn;                                  // [LB_HS] (aliases)
  int32_t* s_hv = s_hk + LB_HS;                                      // [LB_HS]
  unsigned long long* s_sel = (unsigned long long*)(s_bb + LB_CAP);  // [LB_MAX_K] u<<32 | p
  int64_t* s_off = (int64_t*)(s_sel + LB_MAX_K);                     // [maxT]
  double* s_cs = (double*)(s_off + P.maxT);                          // [maxT]
  int32_t* s_fstart = (int32_t*)(s_cs + P.maxT);                     // [maxT + 1]
  int32_t* s_cnt = s_fstart + P.maxT + 1;                            // [maxT]
  int32_t* s_gp = s_cnt + P.maxT;                                    // [ng + 1]

  const int lane = threadIdx.x & 31;
  uint32_t* bm = P.bm + (int64_t)blockIdx.x * P.n4 * 4;
  const uint4* bm4 = (const uint4*)bm;
  double* acc = P.acc ? P.acc + (int64_t)blockIdx.x * P.acc_cap : nullptr;
  const bool degree = P.mode == GS_PROB_DEGREE;
  if (threadIdx.x < MAX_LAYERS) sh.tau_est[threadIdx.x] = 0.0;

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
      // ---- frontier: column starts in the flat edge order ----
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
          const unsigned long long ex = block_exclusive_scan((unsigned long long)d, sh.scan, &tot);
          if (j < T) {
            s_fstart[j] = (int32_t)(run + (int64_t)ex);
            s_off[j] = off;
          }
          run += (int64_t)tot;
        }
        if (threadIdx.x == 0) {
          s_fstart[T] = (int32_t)run;
          sh.u64[1] = (unsigned long long)run;
        }
      }
      __syncthreads();
      const int Ti = (int)T;
      const int64_t nflat = T > 0 ? (int64_t)sh.u64[1] : 0;

      // ---- L1: Extract, the rows' bits (one red.or per distinct row per warp
      // round).  FastGCN with the a0 per-entry degrees: b(u) travels with u, so
      // the edge that sets a row's bit also adds b(u) to B, counts it eligible
      // and runs the fused A-Res filter against the previous batch's threshold
      // (no per-candidate degree lookups, no pass over the bitmap) ----
      const double tau_est = degree ? sh.tau_est[l] : 0.0;
      const float tau_f = (float)tau_est;
      const bool l1_deg = degree && P.degsrc != nullptr;
      // FastGCN with a threshold: every edge whose row's key is below it is
      // staged (position, row, column) in its warp's region, in flat order, so
      // the finalize filters those (~0.5% of the edges) instead of streaming
      // A[:, F] again (the selected rows all have keys below the threshold)
      const bool cstage = l1_deg && tau_est > 0.0 && P.ccap > 0;
      unsigned long long l1_b = 0, l1_e = 0;
      int cfill = 0;
      const int64_t creg = ((int64_t)blockIdx.x * LB_WARPS + (threadIdx.x >> 5)) * LB_CCAP;
      if (threadIdx.x == 0) {
        sh.misc[6] = 0;
        sh.cstage_ovf = 0;
      }
      __syncthreads();
      {
        // the streamed columns are hinted evict-first: the 148 CTAs' candidate
        // bitmaps (the atomics' lines) should keep their place in L2
        const uint64_t pf1 = pol_first(), pl1 = pol_last();
        LBStream st(nflat);
        for (int64_t e0 = st.beg; e0 < st.end; e0 += 32 * LB_ILP) {
          uint32_t u[LB_ILP];
          int32_t dg[LB_ILP];
          int cc[LB_ILP];
#pragma unroll
          for (int q = 0; q < LB_ILP; ++q) {
            const int64_t e = e0 + 32 * q + lane;
            u[q] = 0xFFFFFFFFu;
            dg[q] = 0;
            cc[q] = 0;
            if (e < st.end) {
              const int c = st.col(s_fstart, Ti, e);
              const int64_t pos = s_off[c] + (e - s_fstart[c]);
              cc[q] = c;
              u[q] = (uint32_t)ldg_h(P.indices + pos, pf1);
              if (l1_deg) dg[q] = ldg_h(P.degsrc + pos, pf1);
            }
          }
#pragma unroll
          for (int q = 0; q < LB_ILP; ++q) {
            const uint32_t peers = __match_any_sync(0xffffffffu, u[q]);
            const int leader = __ffs(peers) - 1;
            const bool valid = u[q] != 0xFFFFFFFFu;
            const uint32_t bit = 1u << (u[q] & 31);
            bool cand = false;
            if (valid && leader == lane) {
              if (!l1_deg) {
                atomicOr(bm + (u[q] >> 5), bit);
              } else {
                uint32_t old;
                asm volatile("atom.global.or.L2::cache_hint.b32 %0, [%1], %2, %3;"
                             : "=r"(old) : "l"(bm + (u[q] >> 5)), "r"(bit), "l"(pl1) : "memory");
                const bool is_new = !(old & bit);
                if (is_new) {
                  l1_b += (unsigned long long)dg[q];
                  l1_e += dg[q] > 0 ? 1 : 0;
                }
                // the row's key against the threshold: new rows join the fused
                // pool; every row's edges are staged when it is below
                if (dg[q] > 0 && tau_est > 0.0 && (is_new || cstage)) {
                  const float bb = (float)dg[q];
                  const uint32_t R = philox_k(u[q], 0u, ctr2(l, TAG_ARES_LAYER), gb, P.pk).x;
                  if (ares_maybe_below(R, __fmul_rn(__fmul_rn(tau_f, bb), 1.01f))) {
                    const double kk = ares_key(R, (double)bb);
                    if (kk < tau_est) {
                      cand = true;
                      if (is_new) {
                        const int slot = atomicAdd(&sh.misc[6], 1);
                        if (slot < LB_CAP) {
                          s_bk[slot] = (unsigned long long)__double_as_longlong(kk);
                          s_bu[slot] = u[q];
                          s_bb[slot] = bb;
                        }
                      }
                    }
                  }
                }
              }
            }
            if (cstage) {
              cand = __shfl_sync(0xffffffffu, cand, leader) && valid;  // the row's verdict, for every edge of it
              const unsigned bal = __ballot_sync(0xffffffffu, cand);
              if (bal) {
                const int idx = cfill + __popc(bal & ((1u << lane) - 1u));
                if (cand && idx < P.ccap) {
                  const int64_t e = e0 + 32 * q + lane;
                  P.cnd_pos[creg + idx] = s_off[cc[q]] + (e - s_fstart[cc[q]]);
                  P.cnd_u[creg + idx] = (int32_t)u[q];
                  P.cnd_col[creg + idx] = cc[q];
                }
                cfill += __popc(bal);
              }
            }
          }
        }
      }
      if (cstage && lane == 0) {
        sh.cfill[threadIdx.x >> 5] = cfill;
        if (cfill > P.ccap) sh.cstage_ovf = 1;
      }
      __syncthreads();

      // ---- L2: rank groups (FastGCN: b(u) = in-degree, B, eligible; skipped
      // when L1 already holds B and a usable fused selection) ----
      double Btot = 0.0;
      int64_t nelig = 0;
      int m_fused = 0;
      bool skip_ranks = false;
      if (l1_deg) {
        Btot = (double)block_reduce_sum(l1_b, sh.scan);
        nelig = (int64_t)block_reduce_sum(l1_e, sh.scan);
        m_fused = sh.misc[6];
        skip_ranks = tau_est > 0.0 && m_fused >= K && m_fused <= LB_CAP && nelig > K;
      }
      int64_t nc = 0;
      if (!skip_ranks) {
        if (threadIdx.x == 0) sh.misc[6] = 0;
        __syncthreads();
        double Bx = 0.0;
        int64_t nx = 0;
        nc = lb_ranks(P, sh, bm4, s_gp, degree, &Bx, &nx, l1_deg ? 0.0 : tau_est, l, gb,
                      LBBuf{s_bk, s_bu, s_bb});
        if (!l1_deg) {
          Btot = Bx;
          nelig = nx;
          m_fused = sh.misc[6];
        } else {
          m_fused = 0;  // L1's fused selection was not usable: the select filters the bitmap
        }
      }
      bool acc_ok = true;
      if (!degree && nc > P.acc_cap) {
        if (threadIdx.x == 0) {
          atomicOr(P.err, ERR_CAPACITY);
          atomicMax(P.need_tab, (unsigned long long)nc);
        }
        acc_ok = false;
      }

      // ---- L3 (LADIES / COUNT): b(rank(u)) += fp32(w*w) / 1 in fp64 ----
      if (!degree) {
        if (acc_ok) {
          for (int64_t e0 = threadIdx.x; e0 < nflat; e0 += (int64_t)blockDim.x * LB_ILP) {
            uint32_t u[LB_ILP];
            float w[LB_ILP];
#pragma unroll
            for (int q = 0; q < LB_ILP; ++q) {
              const int64_t e = e0 + (int64_t)q * blockDim.x;
              u[q] = 0xFFFFFFFFu;
              w[q] = 1.0f;
              if (e < nflat) {
                const int c = lb_col(s_fstart, Ti, e);
                const int64_t pos = s_off[c] + (e - s_fstart[c]);
                u[q] = (uint32_t)__ldg(P.indices + pos);
                if (P.mode == GS_PROB_LADIES && P.weights) w[q] = __ldg(P.weights + pos);
              }
            }
#pragma unroll
            for (int q = 0; q < LB_ILP; ++q) {
              if (u[q] == 0xFFFFFFFFu) continue;
              const int64_t r = lb_rank(P, bm, s_gp, u[q]);
              atomicAdd(acc + r, P.mode == GS_PROB_LADIES ? (double)__fmul_rn(w[q], w[q]) : 1.0);
            }
          }
        }
        __syncthreads();
        double bs = 0.0;
        int el = 0;
        for (int64_t r = threadIdx.x; r < nc && acc_ok; r += blockDim.x) {
          const float bb = (float)__ldcg(acc + r);
          bs += (double)bb;
          el += bb > 0.0f ? 1 : 0;
        }
        Btot = block_reduce_sum(bs, sh.dred);
        nelig = acc_ok ? (int64_t)block_reduce_sum((double)el, sh.dred) : 0;
      }
      const float B32 = (float)Btot;

      // ---- L4: Select ----
      auto bias_of = [&](uint32_t u, int64_t r) -> float {
        return degree ? (float)__ldg(P.deg + u) : (float)__ldcg(acc + r);
      };
      if (threadIdx.x == 0) sh.misc[0] = 0;
      __syncthreads();
      int nsel = 0, ncand = 0;
      if (nelig <= K) {  // every eligible candidate (R24)
        if (nelig > 0) {
          lb_for_bits(P, bm4, s_gp, [&](uint32_t u, int64_t r) {
            const float bb = bias_of(u, r);
            if (bb > 0.0f) {
              const int slot = atomicAdd(&sh.misc[0], 1);
              s_bu[slot] = u;
              s_bb[slot] = bb;
            }
          });
        }
        nsel = (int)nelig;
        ncand = nsel;
        __syncthreads();
      } else {
        // threshold filter: keys below tau, ~2K of them (R6: exact fp64 key)
        double tau = 2.0 * K / Btot, lo = 0.0, hi = 0.0;
        int m = 0;
        const bool fused = tau_est > 0.0 && m_fused >= K && m_fused <= LB_CAP;
        if (fused) m = m_fused;
        for (int it = 0; it < 64 && !fused; ++it) {
          if (threadIdx.x == 0) sh.misc[0] = 0;
          __syncthreads();
          lb_for_bits(P, bm4, s_gp, [&](uint32_t u, int64_t r) {
            const float bb = bias_of(u, r);
            if (!(bb > 0.0f)) return;
            const uint32_t R = philox_k(u, 0u, ctr2(l, TAG_ARES_LAYER), gb, P.pk).x;
            const float t = (float)(tau * (double)bb) * 1.01f;
            if (!ares_maybe_below(R, t)) return;
            const double kk = ares_key(R, (double)bb);
            if (!(kk < tau)) return;
            const int slot = atomicAdd(&sh.misc[0], 1);
            if (slot < LB_CAP) {
              s_bk[slot] = (unsigned long long)__double_as_longlong(kk);
              s_bu[slot] = u;
              s_bb[slot] = bb;
            }
          });
          __syncthreads();
          m = sh.misc[0];
          __syncthreads();
          if (m >= K && m <= LB_CAP) break;
          if (m < K) lo = tau;
          else hi = tau;
          tau = (lo > 0.0 && hi > 0.0) ? sqrt(lo * hi) : (lo > 0.0 ? lo * 4.0 : hi * 0.25);
          if (it == 63) {
            if (threadIdx.x == 0) atomicOr(P.err, ERR_INTERNAL);
            m = min(m, LB_CAP);
          }
        }
        ncand = min(m, LB_CAP);
        nsel = min(K, ncand);
        // next batch at this layer: ~3K expected candidates below the estimate
        if (degree && threadIdx.x == 0) sh.tau_est[l] = 3.0 * K / Btot;
      }
      // the K smallest (key, u) of the candidates, then S sorted by node id
      // (R3) as (u << 32 | bias bits): counting-sort ranks (a handful of
      // barriers instead of bitonic networks); scratch in s_sel's region
      {
        int* c_hist = reinterpret_cast<int*>(s_sel);
        int* c_fill = c_hist + LB_THREADS;
        int16_t* c_ord = reinterpret_cast<int16_t*>(c_fill + LB_THREADS);
        int16_t* c_rank = c_ord + LB_CAP;
        uint8_t* c_sel = reinterpret_cast<uint8_t*>(c_rank + LB_CAP);
        if (nsel < ncand) {
          double km = 0.0;
          for (int i = threadIdx.x; i < ncand; i += blockDim.x) km = fmax(km, __longlong_as_double((long long)s_bk[i]));
          km = block_reduce_max(km, sh.dred);
          const double scale = km > 0.0 ? (double)(LB_THREADS - 1) / km : 0.0;
          lb_csrank(
              ncand, c_hist, c_fill, c_ord, c_rank,
              [&](int i) { return min(LB_THREADS - 1, (int)(__longlong_as_double((long long)s_bk[i]) * scale)); },
              [&](int j, int i) { return s_bk[j] < s_bk[i] || (s_bk[j] == s_bk[i] && s_bu[j] < s_bu[i]); },
              [&](int) { return true; }, sh.scan);
          for (int i = threadIdx.x; i < ncand; i += blockDim.x) c_sel[i] = c_rank[i] < nsel ? 1 : 0;
        } else {
          for (int i = threadIdx.x; i < ncand; i += blockDim.x) c_sel[i] = 1;
        }
        __syncthreads();
        const uint64_t NN = (uint64_t)P.N;
        lb_csrank(
            ncand, c_hist, c_fill, c_ord, c_rank,
            [&](int i) { return (int)(((uint64_t)s_bu[i] * LB_THREADS) / NN); },
            [&](int j, int i) { return s_bu[j] < s_bu[i]; },
            [&](int i) { return c_sel[i] != 0; }, sh.scan);
        for (int i = threadIdx.x; i < ncand; i += blockDim.x)
          if (c_sel[i]) s_bk[c_rank[i]] = ((unsigned long long)s_bu[i] << 32) | __float_as_uint(s_bb[i]);
        __syncthreads();
        for (int i = threadIdx.x; i < nsel; i += blockDim.x) s_sel[i] = s_bk[i];
        __syncthreads();
      }
      // p(u) = b(u) / B (R7); hash of S for the finalize
      for (int i = threadIdx.x; i < LB_HS; i += blockDim.x) s_hk[i] = -1;
      __syncthreads();
      for (int i = threadIdx.x; i < nsel; i += blockDim.x) {
        const uint32_t u = (uint32_t)(s_sel[i] >> 32);
        const float p = __fdiv_rn(__uint_as_float((uint32_t)s_sel[i]), B32);
        s_sel[i] = ((unsigned long long)u << 32) | __float_as_uint(p);
        P.row_map[l][rbase + i] = (int32_t)u;
        P.row_prob[l][rbase + i] = p;
        uint32_t h = lb_hash(u);
        while (atomicCAS(&s_hk[h], -1, (int32_t)u) != -1) h = (h + 1) & (LB_HS - 1);
        s_hv[h] = i;
      }
      // clear C for the next batch-layer (bitmap, b(u))
      {
        const uint64_t pl2 = pol_last();  // the cleared lines are the next batch-layer's atomics' lines
        for (int64_t i = threadIdx.x; i < P.n4; i += blockDim.x)
          asm volatile("st.global.L2::cache_hint.v4.b32 [%0], {%1, %1, %1, %1}, %2;" ::"l"((uint4*)bm + i), "r"(0u),
                       "l"(pl2) : "memory");
      }
      if (!degree && acc_ok)
        for (int64_t r = threadIdx.x; r < nc; r += blockDim.x) acc[r] = 0.0;
      for (int j = threadIdx.x; j < Ti; j += blockDim.x) {
        s_cnt[j] = 0;
        s_cs[j] = 0.0;
      }
      __syncthreads();

      // ---- L5a: per column kept count and c_j = sum_fp64 a (a = w / p(u)),
      // per warp kept count (the warp's offset in the CSC emit order) ----
      int wkept = 0;
      const int64_t sreg = ((int64_t)blockIdx.x * LB_WARPS + (threadIdx.x >> 5)) * LB_SCAP;
      int64_t* stg_pos = P.stg_pos + sreg;
      int32_t* stg_lid = P.stg_lid + sreg;
      int32_t* stg_col = P.stg_col + sreg;
      float* stg_a = P.stg_a + sreg;
      if (threadIdx.x == 0) sh.misc[7] = 0;
      __syncthreads();
      if (cstage && skip_ranks && !sh.cstage_ovf) {
        // the kept edges are among L1's staged candidate-row edges (flat order)
        const int n = sh.cfill[threadIdx.x >> 5];
        for (int i0 = 0; i0 < n && nsel > 0; i0 += 32) {
          const int i = i0 + lane;
          const uint32_t uu = i < n ? (uint32_t)P.cnd_u[creg + i] : 0xFFFFFFFFu;
          const int lid = uu == 0xFFFFFFFFu ? -1 : lb_lookup(s_hk, s_hv, uu);
          const unsigned bal = __ballot_sync(0xffffffffu, lid >= 0);
          if (lid >= 0) {
            const int64_t pos = P.cnd_pos[creg + i];
            const int c = P.cnd_col[creg + i];
            const float w = P.weights ? __ldg(P.weights + pos) : 1.0f;
            const float a = __fdiv_rn(w, __uint_as_float((uint32_t)s_sel[lid]));
            atomicAdd(&s_cnt[c], 1);
            atomicAdd(&s_cs[c], (double)a);
            const int idx = wkept + __popc(bal & ((1u << lane) - 1u));
            if (idx < P.scap) {
              stg_pos[idx] = pos;
              stg_lid[idx] = lid;
              stg_col[idx] = c;
              stg_a[idx] = a;
            }
          }
          wkept += __popc(bal);
        }
      } else {
        LBStream st(nflat);
        for (int64_t e0 = st.beg; e0 < st.end && nsel > 0; e0 += 32 * LB_ILP5) {
          uint32_t u[LB_ILP5];
          int c[LB_ILP5];
          int64_t pos[LB_ILP5];
#pragma unroll
          for (int q = 0; q < LB_ILP5; ++q) {
            const int64_t e = e0 + 32 * q + lane;
            u[q] = 0xFFFFFFFFu;
            c[q] = 0;
            pos[q] = 0;
            if (e < st.end) {
              c[q] = st.col(s_fstart, Ti, e);
              pos[q] = s_off[c[q]] + (e - s_fstart[c[q]]);
              u[q] = (uint32_t)__ldg(P.indices + pos[q]);
            }
          }
#pragma unroll
          for (int q = 0; q < LB_ILP5; ++q) {
            const int lid = u[q] == 0xFFFFFFFFu ? -1 : lb_lookup(s_hk, s_hv, u[q]);
            const unsigned bal = __ballot_sync(0xffffffffu, lid >= 0);
            if (lid >= 0) {
              const float w = P.weights ? __ldg(P.weights + pos[q]) : 1.0f;
              const float a = __fdiv_rn(w, __uint_as_float((uint32_t)s_sel[lid]));
              atomicAdd(&s_cnt[c[q]], 1);
              atomicAdd(&s_cs[c[q]], (double)a);
              const int idx = wkept + __popc(bal & ((1u << lane) - 1u));
              if (idx < P.scap) {
                stg_pos[idx] = pos[q];
                stg_lid[idx] = lid;
                stg_col[idx] = c[q];
                stg_a[idx] = a;
              }
            }
            wkept += __popc(bal);
          }
        }
      }
      if (lane == 0) sh.wtot[threadIdx.x >> 5] = wkept;
      if (lane == 0 && wkept > P.scap) sh.misc[7] = 1;  // some warp streams again in L5b
      __syncthreads();
      if (threadIdx.x < 32) {  // warps' exclusive offsets in the emit order
        const int v = sh.wtot[lane];
        sh.wtot[lane] = warp_inclusive_scan(v) - v;
      }
      int64_t E = 0;
      for (int j0 = 0; j0 < Ti; j0 += blockDim.x) {
        const int j = j0 + threadIdx.x;
        const unsigned long long cv = j < Ti ? (unsigned long long)s_cnt[j] : 0ull;
        unsigned long long tot;
        const unsigned long long ex = block_exclusive_scan(cv, sh.scan, &tot);
        if (j < Ti) P.indptr_out[l][ibase + j] = E + (int64_t)ex;
        E += (int64_t)tot;
      }
      if (threadIdx.x == 0) sh.u64[0] = atomicAdd(P.edge_ctr + l, (unsigned long long)E);
      for (int64_t j = threadIdx.x; j < T && l == 0; j += blockDim.x) P.col0[bstart + j] = __ldcg(F + j);
      __syncthreads();
      const int64_t ebase = (int64_t)sh.u64[0];
      const bool fits = ebase + E <= P.edge_cap[l];
      if (!fits && threadIdx.x == 0) atomicOr(P.err, ERR_CAPACITY);

      // ---- L5b: emit in CSC order (the flat order is column-major with
      // ascending positions; warps own contiguous flat ranges in order) ----
      if (fits && E > 0 && !sh.misc[7]) {  // every warp's kept edges are staged: copy them
        const int64_t o = ebase + sh.wtot[threadIdx.x >> 5];
        for (int i = lane; i < wkept; i += 32) {
          P.row_local[l][o + i] = stg_lid[i];
          P.eid[l][o + i] = stg_pos[i];
          P.val[l][o + i] = __fdiv_rn(stg_a[i], (float)s_cs[stg_col[i]]);
        }
      } else if (fits && E > 0) {
        LBStream st(nflat);
        int64_t o = ebase + sh.wtot[threadIdx.x >> 5];
        for (int64_t e0 = st.beg; e0 < st.end; e0 += 32 * LB_ILP) {
          int lid[LB_ILP];
          int c[LB_ILP];
          int64_t pos[LB_ILP];
#pragma unroll
          for (int q = 0; q < LB_ILP; ++q) {
            const int64_t e = e0 + 32 * q + lane;
            lid[q] = -1;
            c[q] = 0;
            pos[q] = 0;
            if (e < st.end) {
              c[q] = st.col(s_fstart, Ti, e);
              pos[q] = s_off[c[q]] + (e - s_fstart[c[q]]);
              lid[q] = lb_lookup(s_hk, s_hv, (uint32_t)__ldg(P.indices + pos[q]));
            }
          }
#pragma unroll
          for (int q = 0; q < LB_ILP; ++q) {
            const unsigned bal = __ballot_sync(0xffffffffu, lid[q] >= 0);
            if (lid[q] >= 0) {
              const int64_t oi = o + __popc(bal & ((1u << lane) - 1u));
              const float w = P.weights ? __ldg(P.weights + pos[q]) : 1.0f;
              const float a = __fdiv_rn(w, __uint_as_float((uint32_t)s_sel[lid[q]]));
              P.row_local[l][oi] = lid[q];
              P.eid[l][oi] = pos[q];
              P.val[l][oi] = __fdiv_rn(a, (float)s_cs[c[q]]);
            }
            o += __popc(bal);
          }
        }
      }
      if (threadIdx.x == 0) {
        P.indptr_out[l][ibase + T] = E;
        long long* mt = (long long*)(P.meta + (b * P.L + l) * 8);
        // an overflowed block wrote no edges: record it empty (GS_ERR_CAPACITY is raised)
        mt[0] = T; mt[1] = nsel; mt[2] = fits ? E : 0; mt[3] = colbase; mt[4] = rbase; mt[5] = ibase;
        mt[6] = fits ? ebase : 0; mt[7] = 0;
      }
      __syncthreads();
      F = P.row_map[l] + rbase;
      colbase = rbase;
      T = nsel;
    }
  }
}

// a0 pre-processing ("degree of each node in FastGCN"): the row's degree
// beside every CSC entry, so the extract stream carries b(u) with u.
__global__ void degsrc_kernel(const int32_t* __restrict__ indices, const int32_t* __restrict__ deg, int64_t nnz,
                              int32_t* __restrict__ out) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x)
    out[e] = deg[indices[e]];
}

// a0 pre-processing ("degree of each node in FastGCN"): deg[u] = in-degree.
__global__ void degree_kernel(const int64_t* __restrict__ indptr, int64_t N, int32_t* __restrict__ deg) {
  for (int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; u < N; u += (int64_t)gridDim.x * blockDim.x)
    deg[u] = (int32_t)(indptr[u + 1] - indptr[u]);
}

static int64_t a256(int64_t x) { return (x + 255) & ~int64_t(255); }

// The a0 degree array of a graph (FastGCN), built once on first use.
gs_status layerwise_degree_array(const gs_graph* g, cudaStream_t stream) {
  gs_graph* gm = const_cast<gs_graph*>(g);
  if (gm->deg) return GS_OK;
  if (!gm->b_deg.ensure(gm->al, (size_t)std::max<int64_t>(g->num_nodes, 1) * 4, stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (degree array)");
  gm->deg = (int32_t*)gm->b_deg.ptr;
  const int64_t blocks = std::min<int64_t>((g->num_nodes + 255) / 256, 148 * 16);
  if (g->num_nodes > 0) {
    degree_kernel<<<(unsigned)std::max<int64_t>(blocks, 1), 256, 0, stream>>>(g->indptr, g->num_nodes, gm->deg);
    count_launch();
  }
  // the per-entry copy (4 B per CSC entry) when memory allows (not for
  // host-mapped graphs: it is as large as their index array); without it the
  // kernel looks b(u) up per candidate
  if (g->num_edges > 0 && !gm->degsrc && !g->host_mapped && gm->b_degsrc.ensure(gm->al, (size_t)g->num_edges * 4, stream)) {
    gm->degsrc = (int32_t*)gm->b_degsrc.ptr;
    const int64_t b2 = std::min<int64_t>((g->num_edges + 255) / 256, 148 * 16);
    degsrc_kernel<<<(unsigned)b2, 256, 0, stream>>>(g->indices, gm->deg, g->num_edges, gm->degsrc);
    count_launch();
  }
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

// Shared-memory bytes of layerwise_bm_kernel for a graph of N nodes (0: does not fit).
size_t layerwise_bm_smem(int64_t N, int maxT, int* gw_log_out, int* ng_out, int64_t* n4_out) {
  const int64_t nwords = (N + 31) / 32;
  int gw_log = 2;
  while (((nwords >> gw_log) + 1) * 4 > 48 * 1024 && gw_log < 6) ++gw_log;
  const int64_t gw = int64_t(1) << gw_log;
  const int64_t ng = (nwords + gw - 1) / gw;
  if ((ng + 1) * 4 > 48 * 1024) return 0;
  const size_t s = (size_t)LB_CAP * (8 + 4 + 4) + (size_t)LB_MAX_K * 8 + (size_t)maxT * (8 + 8) +
                   (size_t)(maxT + 1) * 4 + (size_t)maxT * 4 + (size_t)(ng + 1) * 4 + 16;
  if (s + sizeof(LBShared) > 227 * 1024) return 0;
  *gw_log_out = gw_log;
  *ng_out = (int)ng;
  *n4_out = ng * gw / 4;
  return s;
}

gs_status run_layerwise_bm(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                           int64_t batch_size, int64_t batch_base, const int32_t* n_per_layer,
                           int L, int prob_mode, uint64_t key, cudaStream_t stream, gs_blocks* blk,
                           size_t smem, int gw_log, int ng, int64_t n4) {
  const Allocator& al = blk->al;
  LBParams P = {};
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
  P.pk = philox_keys(key);
  P.gw_log = gw_log;
  P.ng = ng;
  P.n4 = n4;
  const int64_t nbatch = P.num_batches;
  int maxK = 1;
  for (int l = 0; l < L; ++l) {
    P.K[l] = n_per_layer[l];
    maxK = std::max(maxK, n_per_layer[l]);
  }
  P.maxT = (int)std::max<int64_t>(batch_size, maxK);
  if (prob_mode == GS_PROB_DEGREE) {
    const gs_status st = layerwise_degree_array(g, stream);
    if (st) return st;
  }
  P.deg = g->deg;
  P.degsrc = g->degsrc;
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

  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  GS_CUDA_TRY(cudaFuncSetAttribute(layerwise_bm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)smem));
  int ctas = sms;
  if (const char* e = getenv("GS_LW_CTAS")) ctas = std::max(1, std::min(atoi(e), sms));
  const int nctas = (int)std::max<int64_t>(1, std::min<int64_t>(nbatch, ctas));
  // per-CTA workspace: bitmap (kept zero), b(u) by rank (kept zero)
  P.acc_cap = prob_mode == GS_PROB_DEGREE ? 0 : std::max<int64_t>(int64_t(1) << 15, blk->lw_tab_hint);
  const int64_t bm_bytes = a256(n4 * 16);
  const int64_t acc_bytes = a256(P.acc_cap * 8);
  const int64_t stg_bytes = a256((int64_t)LB_WARPS * LB_SCAP * (8 + 4 + 4 + 4)) +
                            a256((int64_t)LB_WARPS * LB_CCAP * (8 + 4 + 4));
  const int64_t stride = bm_bytes + acc_bytes + stg_bytes;
  const size_t ws_bytes = (size_t)stride * nctas;
  const bool grow = blk->b_ws.bytes < ws_bytes;
  if (!blk->b_ws.ensure(al, ws_bytes, stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (layer-wise workspace)");
  if (grow || blk->ws_stride_prev != stride || blk->ws_kind_prev != 3)
    GS_CUDA_TRY(cudaMemsetAsync(blk->b_ws.ptr, 0, blk->b_ws.bytes, stream));
  blk->ws_stride_prev = stride;
  blk->ws_kind_prev = 3;
  // bitmaps of every CTA first, then the b(u) arrays
  P.bm = (uint32_t*)blk->b_ws.ptr;
  P.acc = prob_mode == GS_PROB_DEGREE ? nullptr : (double*)((char*)blk->b_ws.ptr + bm_bytes * nctas);
  P.scap = LB_SCAP;
  if (const char* e = getenv("GS_LW_SCAP")) P.scap = std::max(0, std::min(atoi(e), LB_SCAP));  // tests
  {
    char* sb = (char*)blk->b_ws.ptr + (bm_bytes + acc_bytes) * nctas;
    const int64_t ne = (int64_t)nctas * LB_WARPS * LB_SCAP;
    P.stg_pos = (int64_t*)sb;
    P.stg_lid = (int32_t*)(sb + ne * 8);
    P.stg_col = (int32_t*)(sb + ne * 12);
    P.stg_a = (float*)(sb + ne * 16);
    char* cb = sb + a256(ne * 20);
    const int64_t nc = (int64_t)nctas * LB_WARPS * LB_CCAP;
    P.cnd_pos = (int64_t*)cb;
    P.cnd_u = (int32_t*)(cb + nc * 8);
    P.cnd_col = (int32_t*)(cb + nc * 12);
  }
  P.ccap = prob_mode == GS_PROB_DEGREE ? LB_CCAP : 0;
  if (const char* e = getenv("GS_LW_CCAP")) P.ccap = std::max(0, std::min(atoi(e), LB_CCAP));  // tests
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
  layerwise_bm_kernel<<<nctas, LB_THREADS, smem, stream>>>(P); count_launch();
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

}  // namespace gsb
