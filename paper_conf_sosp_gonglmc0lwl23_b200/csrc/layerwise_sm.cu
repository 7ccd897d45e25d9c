// layerwise_sm.cu -- layer-wise ECSF sampling with shared-memory state:
// LADIES (Fig. 3(b)) and COUNT, the modes
// whose bias b(u) is accumulated over the extracted edges.
//
// collective_sample for one mini-batch at a time per CTA (one
// 1024-thread CTA per SM, persistent, batches claimed from a counter;
// super-batch P:322-336).  Every per-batch-layer table lives in shared memory
// and the extracted edges of A[:, F] live in REGISTERS (12 per thread, so a
// batch-layer of <= 12,288 edges is read from the graph exactly once; larger
// ones are streamed in 12,288-edge chunks per pass).  Per (batch, layer) with
// frontier F (T <= 1024 columns) and K <= 1024:
//   A  frontier: (indptr, degree) per column, block scan -> column starts of
//      the flat edge order (column-major, positions ascending);
//   B  Extract + edge-map: (u, fp32(w*w)) of every flat edge into
//      registers; B' = sum_fp64 w^2 (= B up to per-row rounding) centres the
//      key histogram (R6: key = -ln(u) / b);
//   C  Compute (edge-reduce): the rows are inserted into an 11,264-slot
//      shared hash (row id + fp64 accumulator) in as many hash partitions of
//      the row ids as the edge count needs (one for <= 8,448 edges): one
//      shared CAS per edge (the claiming edge stores its w^2, the rare other
//      edges of a row add theirs after a barrier); per partition a dense list
//      of the occupied slots, b(u) = fp32(acc), B += b, eligibility b > 0, one
//      Philox word per candidate and a 16-bins-per-octave histogram of the
//      approximate keys below 16 K / B'; tau = the histogram's bin edge below
//      which K + K/8 keys lie (one attempt: no threshold guessing), and the
//      candidates whose exact fp64 key is below tau are the survivors;
//   D  Select: R24 (every eligible row when at most K are), else the K
//      smallest (key, u) by a counting sort of the survivors on 1,024 key bins
//      (exact ties inside a bin by (key, u)), then S sorted by u by a second
//      counting sort (R3); too few / too many survivors -> tau adjusted, C
//      repeated (from the table when one partition holds every row);
//   E  Finalize (edge-map divide + column reduction fused): p(u) =
//      fp32(b / B); every register-held edge probes a shared hash of S; kept
//      edges get a_e = fp32(w / p(u)) (w re-read only for them), c_j =
//      sum_fp64 a by shared atomics; CSC positions from one warp-ballot prefix
//      over the flat order, val_e = fp32(a_e / c_j).
// About 20 block barriers per batch-layer and no global workspace: the graph
// reads and the block outputs are the only DRAM traffic (ncu: 7.2 GB per LJ
// epoch against 7.9 GB of algorithmic bytes; the global-table kernel moved
// 33).  FastGCN's ~280 k candidates per batch-layer keep the bitmap kernel of
// layerwise_bm.cu.
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include "common.cuh"
#include "gs_internal.h"
#include "nodewise_common.cuh"

namespace gsb {

// (threads, flat edges per thread held in registers): 16,384-edge chunks
constexpr int LS_CHMAX = 16384;
constexpr int LS_HT = 11264;                 // hash slots (row id + fp64 accumulator)
constexpr int LS_HLIM = LS_HT - LS_HT / 8;   // claims per partition pass before it is split
constexpr int LS_PART = (LS_HT * 3) / 4;     // flat edges per hash partition
constexpr int LS_MAXT = 1024;                // frontier columns (batch size, K)
constexpr int LS_MAXK = 1024;
constexpr int LS_SCAP = 2048;                // survivors (key below tau)
constexpr int LS_SHS = 2048;                 // hash of S
constexpr int LS_NH = 512;                   // approximate-key histogram: 16 bins per octave
constexpr int LS_HSH = 19;                   //   from 2 octaves below K / B' (bin 0: everything
constexpr int LS_HOFF = 32;                  //   lower) to LS_HWIN K / B'
constexpr float LS_HWIN = 16.0f;
constexpr int LS_NBLK = 1024;                // flat-edge blocks indexed to their column
constexpr uint32_t LS_EMPTY = 0xFFFFFFFFu;
constexpr int LS_MAXPASS = 48;              // partitions x chunks a batch-layer may cost

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
  PhiloxKeys pk;
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
  int64_t* meta;
  int* err;
};

struct LSSmem {
  // C: fp64 accumulators, then (b, Philox word) per slot; D: counting-sort scratch
  double acc[LS_HT];
  // C: row ids; E: the hash of S (ids, then local ids)
  uint32_t key[LS_HT];
  // C: the occupied slots (dense candidate list)
  uint16_t clist[LS_HT];
  int32_t hist[LS_NH];
  // survivors: exact key, row id, b(u)
  double skey[LS_SCAP];
  uint32_t scu[LS_SCAP];
  float scb[LS_SCAP];
  // frontier columns
  int64_t off[LS_MAXT];
  double cs[LS_MAXT];
  int32_t cstart[LS_MAXT + 1];
  int32_t cnt[LS_MAXT];
  // S
  uint32_t su[LS_MAXK];
  float sp[LS_MAXK];
  int32_t wpre[LS_CHMAX / 32];
  int16_t colblk[LS_NBLK];
  double scr[72];
  long long misc[8];
  int imisc[8];
  float ftau;
};
static_assert(sizeof(LSSmem) <= 232448, "LSSmem exceeds the 227 KB of shared memory per CTA");

__device__ __forceinline__ uint32_t ls_slot(uint32_t u) { return __umulhi(u * 0x9E3779B1u, (uint32_t)LS_HT); }
__device__ __forceinline__ uint32_t ls_part(uint32_t u, uint32_t np) {
  uint32_t x = (u ^ (u >> 16)) * 0x85EBCA6Bu;
  x ^= x >> 13;
  return __umulhi(x * 0xC2B2AE35u, np);
}
__device__ __forceinline__ uint32_t ls_sslot(uint32_t u) { return (u * 0x9E3779B1u) >> (32 - 11); }

// Inserts row u with one shared atomic (the claiming CAS; shared atomics cost
// ~2 cycles per lane on this part, so nothing else per edge is atomic): the
// slot, *claimed = whether this call took it; -1 once the pass has claimed
// about LS_HLIM slots (nclaim is bumped once per warp and edge round, so it
// lags by at most the CTA's thread count: the table never fills).
__device__ __forceinline__ int ls_claim(uint32_t* key, const int* nclaim, uint32_t u, bool* claimed) {
  uint32_t h = ls_slot(u);
  *claimed = false;
  while (true) {
    const uint32_t k = key[h];
    if (k == u) return (int)h;
    if (k == LS_EMPTY) {
      if (*(const volatile int*)nclaim >= LS_HLIM) return -1;
      const uint32_t prev = atomicCAS(&key[h], LS_EMPTY, u);
      if (prev == LS_EMPTY) {
        *claimed = true;
        return (int)h;
      }
      if (prev == u) return (int)h;
    }
    if (++h == (uint32_t)LS_HT) h = 0;
  }
}
__device__ __forceinline__ int ls_find(const uint32_t* key, uint32_t u) {
  uint32_t h = ls_slot(u);
  while (true) {
    const uint32_t k = key[h];
    if (k == u) return (int)h;
    if (k == LS_EMPTY) return -1;
    if (++h == (uint32_t)LS_HT) h = 0;
  }
}

// local id of u in S (hash of S: ids in key[0, SHS), local ids in key[SHS, 2 SHS)), or -1
__device__ __forceinline__ int ls_find_s(const uint32_t* key, uint32_t u) {
  uint32_t h = ls_sslot(u);
  while (true) {
    const uint32_t k = key[h];
    if (k == u) return (int)key[LS_SHS + h];
    if (k == LS_EMPTY) return -1;
    h = (h + 1) & (LS_SHS - 1);
  }
}

// -ln((r + 0.5) 2^-32) in fp32 to ~1e-6 relative (the histogram's approximate key).
__device__ __forceinline__ float ls_e32(uint32_t r) {
  if (r >= 0x80000000u) {
    const float x = __fmul_rn(__uint2float_rn(0xFFFFFFFFu - r) + 0.5f, 2.3283064365386963e-10f);
    return -log1pf(-x);
  }
  return -__logf(__fmul_rn(__uint2float_rn(r) + 0.5f, 2.3283064365386963e-10f));
}

// One warp: the smallest tau such that the histogram's bins below it hold at
// least `target` approximate keys, widened by 1e-4 (>> the approximation's
// error), so at least `target` exact keys are below it; -1 (no filter) when
// the histogram never reaches the target below its top bin.
__device__ __forceinline__ void ls_tau_from_hist(const int32_t* hist, int target, int tbits, float* out) {
  const int lane = threadIdx.x & 31;
  constexpr int PER = LS_NH / 32;
  int v[PER], sum = 0;
#pragma unroll
  for (int k = 0; k < PER; ++k) {
    v[k] = hist[lane * PER + k];
    sum += v[k];
  }
  const int inc = warp_inclusive_scan(sum);
  const uint32_t m = __ballot_sync(0xffffffffu, inc >= target);
  if (lane == 0) *out = -3.0f;  // the keys below the window do not reach the target
  if (!m) return;
  const int ln = __ffs(m) - 1;
  if (lane == ln) {
    int run = inc - sum, j = lane * PER + PER - 1;
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      run += v[k];
      if (run >= target) {
        j = lane * PER + k;
        break;
      }
    }
    float tau = -1.0f;
    if (j < LS_NH - 1) {
      const long long bits = (long long)tbits + ((long long)(j - LS_HOFF + 1) << LS_HSH);
      if (bits > 0 && bits < 0x7F800000ll) tau = __int_as_float((int)bits) * 1.0001f;
    }
    *out = tau;
  }
}

// Flat edge e -> its frontier column: the column of e's 2^gsh-edge block's
// first edge, then a binary search up to the next block's.
__device__ __forceinline__ int ls_col(const int32_t* cstart, const int16_t* colblk, int gsh, int nblk, int T,
                                       int e) {
  const int bk = e >> gsh;
  int lo = colblk[bk], hi = bk + 1 < nblk ? colblk[bk + 1] : T - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (cstart[mid] <= e) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

// Block-wide sums of two doubles in one pass (scratch >= 66 doubles).
__device__ __forceinline__ void ls_reduce2(double& a, double& b, double* scr) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    a += __shfl_xor_sync(0xffffffffu, a, o);
    b += __shfl_xor_sync(0xffffffffu, b, o);
  }
  if (lane == 0) {
    scr[wid] = a;
    scr[32 + wid] = b;
  }
  __syncthreads();
  double sa = 0.0, sb = 0.0;
  for (int w = 0; w < nw; ++w) {  // every thread sums the warps' partials in the same order
    sa += scr[w];
    sb += scr[32 + w];
  }
  __syncthreads();
  a = sa;
  b = sb;
}

// Counting-sort rank of n <= LS_SCAP items (bin(i) monotone in the order,
// less(j, i) the exact order inside a bin): rank[i] for every item with
// take(i); items without take(i) are ignored.  hist / fill / ord / rank are
// shared scratch; every thread of the CTA calls it.
template <int LS_THREADS, class Bin, class Less, class Take>
__device__ __forceinline__ void ls_rank(int n, int* hist, int* fill, int* ord, int* rank, Bin bin,
                                        Less less, Take take, long long* scr) {
  const int t = threadIdx.x;
  hist[t] = 0;
  fill[t] = 0;
  __syncthreads();
  for (int i = t; i < n; i += LS_THREADS)
    if (take(i)) atomicAdd(&hist[bin(i)], 1);
  __syncthreads();
  long long tot;
  const int c = hist[t];
  const int st = (int)block_exclusive_scan<long long>(c, scr, &tot);
  hist[t] = st;  // bin start (the scan synchronised after reading every count)
  __syncthreads();
  for (int i = t; i < n; i += LS_THREADS)
    if (take(i)) {
      const int bb = bin(i);
      ord[hist[bb] + atomicAdd(&fill[bb], 1)] = i;
    }
  __syncthreads();
  for (int i = t; i < n; i += LS_THREADS)
    if (take(i)) {
      const int bb = bin(i), s0 = hist[bb], s1 = s0 + fill[bb];
      int r = s0;
      for (int k = s0; k < s1; ++k) r += less(ord[k], i) ? 1 : 0;
      rank[i] = r;
    }
  __syncthreads();
}

template <int LS_THREADS, int LS_NQ>
__global__ void __launch_bounds__(LS_THREADS, 1) layerwise_sm_kernel(LSParams P) {
  constexpr int LS_WARPS = LS_THREADS / 32;
  constexpr int LS_CH = LS_THREADS * LS_NQ;  // flat edges per chunk
  constexpr int LS_NB = LS_THREADS;          // counting-sort bins
  extern __shared__ __align__(16) unsigned char ls_raw[];
  LSSmem& sm = *reinterpret_cast<LSSmem*>(ls_raw);
  const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
  const bool ladies = P.mode == GS_PROB_LADIES;
  const bool wts = P.weights != nullptr;
  long long* scrl = reinterpret_cast<long long*>(sm.scr);
  // counting-sort scratch in the accumulator region (free once C is done)
  int* d_hist = reinterpret_cast<int*>(sm.acc);
  int* d_fill = d_hist + LS_NB;
  int* d_ord = d_fill + LS_NB;
  int* d_rank = d_ord + LS_SCAP;
  int* d_rank2 = d_rank + LS_SCAP;
  int* d_sel = d_rank2 + LS_SCAP;
  while (true) {
    if (t == 0) sm.misc[7] = (long long)atomicAdd(P.claim, 1u);
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
      // ---- A: frontier ----
      {
        long long run = 0;
        for (int j0 = 0; j0 < T; j0 += LS_THREADS) {  // T <= LS_MAXT columns, LS_THREADS at a time
          const int j = j0 + t;
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
          const long long ex = block_exclusive_scan<long long>(d, scrl, &tot);
          if (j < T) sm.cstart[j] = (int32_t)(run + ex);
          run += tot;
        }
        if (t == 0) {
          sm.cstart[T] = (int32_t)run;
          sm.misc[1] = run;
        }
        __syncthreads();
      }
      int64_t dsum = sm.misc[1];
      // block index of the flat edges: colblk[k] = column of edge k << gsh
      int gsh = 5;
      while (((dsum - 1) >> gsh) >= LS_NBLK) ++gsh;
      const int nblk = dsum > 0 ? (int)((dsum - 1) >> gsh) + 1 : 0;
      for (int j = t; j < T; j += LS_THREADS) {
        const int s0 = sm.cstart[j], s1 = sm.cstart[j + 1];
        if (s1 > s0 && dsum < (int64_t(1) << 30))
          for (int k = (s0 + (1 << gsh) - 1) >> gsh; k <= ((s1 - 1) >> gsh); ++k) sm.colblk[k] = (int16_t)j;
      }
      __syncthreads();
      if (dsum >= (int64_t(1) << 30)) {  // beyond the int32 flat index: not supported here
        if (t == 0) atomicOr(P.err, ERR_INTERNAL);
        dsum = 0;
      }
      // partition passes re-stream every chunk: beyond LS_MAXPASS chunk loads
      // per pass set the batch-layer is left to the global-table kernel (the
      // binding re-runs the call, gs_blocks.lw_big)
      if (dsum > 0 && ((dsum + LS_PART - 1) / LS_PART) * ((dsum + LS_CH - 1) / LS_CH) > LS_MAXPASS) {
        if (t == 0) {
          atomicOr(P.err, ERR_CAPACITY);
          atomicMax(P.edge_ctr + MAX_LAYERS + 1, 1ull);
        }
        dsum = 0;
      }
      const int nflat = T > 0 ? (int)dsum : 0;
      const int nch = (nflat + LS_CH - 1) / LS_CH;
      uint32_t u[LS_NQ];
      float w2[LS_NQ];
      // chunk ci of the flat edges -> registers: (row id, fp32(w*w)) (COUNT: 1)
      auto load = [&](int ci) {
#pragma unroll
        for (int q = 0; q < LS_NQ; ++q) {
          const int e = ci * LS_CH + q * LS_THREADS + t;
          u[q] = LS_EMPTY;
          w2[q] = 0.0f;
          if (e < nflat) {
            const int c = ls_col(sm.cstart, sm.colblk, gsh, nblk, T, e);
            const int64_t pos = sm.off[c] + (e - sm.cstart[c]);
            u[q] = (uint32_t)__ldg(P.indices + pos);
            if (ladies && wts) {
              const float w = __ldg(P.weights + pos);
              w2[q] = __fmul_rn(w, w);
            } else {
              w2[q] = 1.0f;
            }
          }
        }
      };
      // ---- B: Extract + w^2, B' ----
      double bp = 0.0;
      for (int ci = 0; ci < nch; ++ci) {
        load(ci);
#pragma unroll
        for (int q = 0; q < LS_NQ; ++q) bp += (double)w2[q];
      }
      const double Bp = block_reduce_sum<double>(bp, sm.scr);
      // ---- C: hash partitions of the rows -> b(u), B, one Philox word per
      // candidate and an approximate-key histogram; survivors below tau ----
      int NP = max(1, (nflat + LS_PART - 1) / LS_PART);
      const float tauB = Bp > 0.0 ? (float)((double)K / Bp) : 1.0f;  // histogram centre
      const int tbits = __float_as_int(tauB);
      const float hwin = __fmul_rn(tauB, LS_HWIN);
      int nsel = 0, ncand = 0, nelig = 0;
      double Btot = 0.0;
      bool haveB = false, done = false, hist_tau_used = false;
      float tau = -2.0f;  // -2: not chosen yet
      float lo = 0.0f, hi = 0.0f;
      for (int attempt = 0; attempt < 32 && !done && nflat > 0; ++attempt) {
        // several partitions: a generous first tau (the histogram is complete only
        // after the last partition); one partition: tau from the histogram
        if (tau == -2.0f && NP > 1) tau = Bp > 0.0 ? (float)(3.0 * K / Bp) : -1.0f;
        const bool build = !(NP == 1 && haveB);  // one partition: the table is kept for retries
        if (t == 0) {
          sm.imisc[0] = 0;
          sm.imisc[2] = 0;
        }
        if (!haveB)
          for (int i = t; i < LS_NH; i += LS_THREADS) sm.hist[i] = 0;
        __syncthreads();
        double bsum = 0.0;
        int elig = 0;
        for (int p = 0; p < NP; ++p) {
          if (build) {
            for (int i = t; i < LS_HT; i += LS_THREADS) sm.key[i] = LS_EMPTY;
            if (t == 0) sm.imisc[1] = 0;
            __syncthreads();
            // the claiming edge of a row stores its w^2; the other edges of the
            // row (rare: LADIES rows mostly meet the frontier once) add theirs
            // in fp64 after a barrier (chunk by chunk)
            for (int ci = 0; ci < nch; ++ci) {
              if (nch > 1) load(ci);
              uint64_t dupm = 0;
#pragma unroll
              for (int q = 0; q < LS_NQ; ++q) {
                const bool act = u[q] != LS_EMPTY && (NP == 1 || ls_part(u[q], (uint32_t)NP) == (uint32_t)p);
                bool claimed = false;
                if (act) {
                  const int h = ls_claim(sm.key, &sm.imisc[1], u[q], &claimed);
                  if (h < 0) sm.imisc[2] = 1;
                  else if (claimed) sm.acc[h] = (double)w2[q];
                  else dupm |= 1ull << q;
                }
                const uint32_t bal = __ballot_sync(0xffffffffu, claimed);
                if (lane == 0 && bal) atomicAdd(&sm.imisc[1], __popc(bal));
              }
              if (__syncthreads_or(dupm != 0)) {
#pragma unroll
                for (int q = 0; q < LS_NQ; ++q)
                  if ((dupm >> q) & 1ull) atomicAdd(&sm.acc[ls_find(sm.key, u[q])], (double)w2[q]);
                __syncthreads();
              }
            }
            if (sm.imisc[2]) break;  // uniform: the pass overflowed, split it
            // dense candidate list: the occupied slots, compacted by warp ballots
            if (t == 0) sm.imisc[3] = 0;
            __syncthreads();
            for (int h0 = 0; h0 < LS_HT; h0 += LS_THREADS) {
              const int h = h0 + t;
              const bool occ = h < LS_HT && sm.key[h] != LS_EMPTY;
              const uint32_t bal = __ballot_sync(0xffffffffu, occ);
              int base = 0;
              if (lane == 0 && bal) base = atomicAdd(&sm.imisc[3], __popc(bal));
              base = __shfl_sync(0xffffffffu, base, 0);
              if (occ) sm.clist[base + __popc(bal & ((1u << lane) - 1u))] = (uint16_t)h;
            }
            __syncthreads();
            const int ncl = sm.imisc[3];
            // b(u), B, eligibility, one Philox word per candidate ((b, r) packed in
            // place) and the approximate key's histogram bin
            for (int i = t; i < ncl; i += LS_THREADS) {
              const int h = sm.clist[i];
              const uint32_t uk = sm.key[h];
              const float bias = (float)sm.acc[h];
              bsum += (double)bias;
              uint32_t r = 0;
              if (bias > 0.0f) {
                ++elig;
                r = philox_k(uk, 0u, ctr2(l, TAG_ARES_LAYER), gb, P.pk).x;
                // histogram of the approximate keys below LS_HWIN K / B' only
                // (one shared atomic per counted key)
                if (!haveB && ares_maybe_below(r, __fmul_rn(hwin, bias))) {
                  const float k32 = __fdividef(ls_e32(r), bias);
                  const int bn = max(0, ((__float_as_int(k32) - tbits) >> LS_HSH) + LS_HOFF);
                  if (bn < LS_NH) atomicAdd(&sm.hist[bn], 1);
                }
              }
              sm.acc[h] = __hiloint2double(__float_as_int(bias), (int)r);
            }
          }
          if (NP == 1 && tau == -2.0f) {  // one partition: tau from the complete histogram
            __syncthreads();
            if (warp == 0) ls_tau_from_hist(sm.hist, K + K / 8 + 8, tbits, &sm.ftau);
            __syncthreads();
            tau = sm.ftau == -3.0f ? __fmul_rn(hwin, 4.0f) : sm.ftau;
            hist_tau_used = true;
          }
          // survivors of this partition (list entries of this thread: packed above)
          const int ncl = sm.imisc[3];
          for (int i = t; i < ncl; i += LS_THREADS) {
            const int h = sm.clist[i];
            const double pk = sm.acc[h];
            const float bias = __int_as_float(__double2hiint(pk));
            if (!(bias > 0.0f)) continue;
            const uint32_t r = (uint32_t)__double2loint(pk);
            if (tau >= 0.0f && !ares_maybe_below(r, __fmul_rn(__fmul_rn(tau, bias), 1.01f))) continue;
            const double kk = ares_key(r, (double)bias);
            if (tau >= 0.0f && !(kk < (double)tau)) continue;
            const int slot = atomicAdd(&sm.imisc[0], 1);
            if (slot < LS_SCAP) {
              sm.skey[slot] = kk;
              sm.scu[slot] = sm.key[h];
              sm.scb[slot] = bias;
            }
          }
          __syncthreads();
        }
        const bool ovf = sm.imisc[2] != 0;
        if (build && !ovf && !haveB) {
          double e2 = (double)elig;  // B and the eligible count in one reduction
          ls_reduce2(bsum, e2, sm.scr);
          Btot = bsum;
          nelig = (int)e2;
          haveB = true;
        }
        ncand = sm.imisc[0];
        __syncthreads();
        if (ovf) {  // a partition overflowed the table: twice the partitions
          NP *= 2;
          tau = -2.0f;
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
        if (ncand >= K && ncand <= LS_SCAP) {
          nsel = K;
          done = true;
          break;
        }
        if (!hist_tau_used) {  // several partitions: the first tau missed; the histogram's
          if (warp == 0) ls_tau_from_hist(sm.hist, K + K / 8 + 8, tbits, &sm.ftau);
          __syncthreads();
          tau = sm.ftau == -3.0f ? __fmul_rn(hwin, 4.0f) : sm.ftau;
          __syncthreads();
          hist_tau_used = true;
          continue;
        }
        if (ncand < K) lo = tau;  // tau too small (bisection: should not happen)
        else hi = tau < 0.0f ? (float)(5.2 * K / Btot) : tau;
        tau = (lo > 0.0f && hi > 0.0f) ? sqrtf(lo * hi) : (lo > 0.0f ? lo * 4.0f : hi * 0.25f);
      }
      if (!done && nflat > 0 && t == 0) atomicOr(P.err, ERR_INTERNAL);
      if (!done) nsel = 0;
      ncand = min(ncand, LS_SCAP);
      const uint32_t* cu = sm.scu;
      const float* cb = sm.scb;
      // ---- D: the K smallest (key, u) of the survivors, then S ascending ----
      if (done && nsel > 0) {
        if (nsel < ncand) {
          // the survivors' keys lie below tau (the key bins' range); without a
          // threshold, below their maximum
          double kmax = (double)tau;
          if (!(tau > 0.0f)) {
            double km = 0.0;
            for (int i = t; i < ncand; i += LS_THREADS) km = fmax(km, sm.skey[i]);
            for (int o = 16; o > 0; o >>= 1) km = fmax(km, __shfl_xor_sync(0xffffffffu, km, o));
            if (lane == 0) sm.scr[warp] = km;
            __syncthreads();
            kmax = 0.0;
            for (int w = 0; w < LS_WARPS; ++w) kmax = fmax(kmax, sm.scr[w]);
            __syncthreads();
          }
          const double scale = kmax > 0.0 ? (double)(LS_NB - 1) / kmax : 0.0;
          ls_rank<LS_THREADS>(
              ncand, d_hist, d_fill, d_ord, d_rank,
              [&](int i) { return min(LS_NB - 1, (int)(sm.skey[i] * scale)); },
              [&](int j, int i) {
                const double kj = sm.skey[j], ki = sm.skey[i];
                return kj < ki || (kj == ki && cu[j] < cu[i]);
              },
              [&](int) { return true; }, scrl);
          for (int i = t; i < ncand; i += LS_THREADS) d_sel[i] = d_rank[i] < nsel ? 1 : 0;
        } else {
          for (int i = t; i < ncand; i += LS_THREADS) d_sel[i] = 1;
        }
        __syncthreads();
        const uint64_t NN = (uint64_t)P.N;
        ls_rank<LS_THREADS>(
            ncand, d_hist, d_fill, d_ord, d_rank2,
            [&](int i) { return (int)(((uint64_t)cu[i] * LS_NB) / NN); },
            [&](int j, int i) { return cu[j] < cu[i]; },
            [&](int i) { return d_sel[i] != 0; }, scrl);
        for (int i = t; i < ncand; i += LS_THREADS)
          if (d_sel[i]) {
            sm.su[d_rank2[i]] = cu[i];
            sm.sp[d_rank2[i]] = cb[i];
          }
      }
      // ---- E: S (ascending), p(u) = b(u) / B, hash of S ----
      for (int i = t; i < LS_SHS; i += LS_THREADS) sm.key[i] = LS_EMPTY;
      for (int j = t; j < T; j += LS_THREADS) {
        sm.cnt[j] = 0;
        sm.cs[j] = 0.0;
      }
      __syncthreads();
      const float B32 = (float)Btot;
      for (int i = t; i < nsel; i += LS_THREADS) {
        const uint32_t uu = sm.su[i];
        const float pu = __fdiv_rn(sm.sp[i], B32);
        sm.sp[i] = pu;
        P.row_map[l][rbase + i] = (int32_t)uu;
        P.row_prob[l][rbase + i] = pu;
        uint32_t h = ls_sslot(uu);
        while (atomicCAS(&sm.key[h], LS_EMPTY, uu) != LS_EMPTY) h = (h + 1) & (LS_SHS - 1);
        sm.key[LS_SHS + h] = (uint32_t)i;
      }
      __syncthreads();
      // kept edges of chunk ci: u[q] <- local id, w2[q] <- a_e (kept bit q of the mask)
      auto probe = [&](int ci, bool reload, bool reduce) -> uint64_t {
        if (reload) load(ci);
        uint64_t m = 0;
#pragma unroll
        for (int q = 0; q < LS_NQ; ++q) {
          if (u[q] == LS_EMPTY) continue;
          const int lid = ls_find_s(sm.key, u[q]);
          if (lid < 0) continue;
          const int e = ci * LS_CH + q * LS_THREADS + t;
          const int c = ls_col(sm.cstart, sm.colblk, gsh, nblk, T, e);
          const int64_t pos = sm.off[c] + (e - sm.cstart[c]);
          const float w = wts ? __ldg(P.weights + pos) : 1.0f;
          const float a = __fdiv_rn(w, sm.sp[lid]);
          if (reduce) {
            atomicAdd(&sm.cnt[c], 1);
            atomicAdd(&sm.cs[c], (double)a);
          }
          u[q] = (uint32_t)lid;
          w2[q] = a;
          m |= 1ull << q;
        }
        return m;
      };
      uint64_t kmask = 0;
      if (nsel > 0)
        for (int ci = 0; ci < nch; ++ci) kmask = probe(ci, nch > 1, true);
      __syncthreads();
      long long E = 0;
      for (int j0 = 0; j0 < T; j0 += LS_THREADS) {
        const int j = j0 + t;
        const long long c = j < T ? sm.cnt[j] : 0;
        long long tot;
        const long long ex = block_exclusive_scan<long long>(c, scrl, &tot);
        if (j < T) P.indptr_out[l][ibase + j] = E + ex;
        E += tot;
      }
      if (t == 0) sm.misc[0] = (long long)atomicAdd(P.edge_ctr + l, (unsigned long long)E);
      __syncthreads();
      const long long ebase = sm.misc[0];
      const bool fits = ebase + E <= P.edge_cap[l];
      if (!fits && t == 0) atomicOr(P.err, ERR_CAPACITY);
      // ---- E: emit in CSC order = the flat order (chunk, q, warp, lane) ----
      long long run = 0;
      for (int ci = 0; ci < nch && fits && E > 0; ++ci) {
        if (nch > 1) kmask = probe(ci, true, false);
#pragma unroll
        for (int q = 0; q < LS_NQ; ++q) {
          const uint32_t bal = __ballot_sync(0xffffffffu, (kmask >> q) & 1ull);
          if (lane == 0) sm.wpre[q * LS_WARPS + warp] = __popc(bal);
        }
        __syncthreads();
        if (warp == 0) {
          constexpr int PER = LS_NQ * LS_WARPS / 32;
          int v[PER], s = 0;
#pragma unroll
          for (int k = 0; k < PER; ++k) {
            v[k] = sm.wpre[lane * PER + k];
            s += v[k];
          }
          const int inc = warp_inclusive_scan(s);
          int x = inc - s;
#pragma unroll
          for (int k = 0; k < PER; ++k) {
            sm.wpre[lane * PER + k] = x;
            x += v[k];
          }
          if (lane == 31) sm.misc[2] = inc;
        }
        __syncthreads();
#pragma unroll
        for (int q = 0; q < LS_NQ; ++q) {
          const bool kq = (kmask >> q) & 1ull;
          const uint32_t bal = __ballot_sync(0xffffffffu, kq);
          if (!kq) continue;
          const long long o = ebase + run + sm.wpre[q * LS_WARPS + warp] + __popc(bal & ((1u << lane) - 1u));
          const int e = ci * LS_CH + q * LS_THREADS + t;
          const int c = ls_col(sm.cstart, sm.colblk, gsh, nblk, T, e);
          P.row_local[l][o] = (int32_t)u[q];
          P.eid[l][o] = sm.off[c] + (e - sm.cstart[c]);
          P.val[l][o] = __fdiv_rn(w2[q], (float)sm.cs[c]);
        }
        run += sm.misc[2];
        __syncthreads();
      }
      if (t == 0) {
        P.indptr_out[l][ibase + T] = E;
        long long* m = (long long*)(P.meta + (b * P.L + l) * 8);
        m[0] = T; m[1] = nsel; m[2] = fits ? E : 0; m[3] = colbase; m[4] = rbase; m[5] = ibase;
        m[6] = fits ? ebase : 0; m[7] = 0;
      }
      __syncthreads();
      F = P.row_map[l] + rbase;
      colbase = rbase;
      T = nsel;
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
  P.pk = philox_keys(key);
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
  // 1024 threads x 12 register-held edges: measured on LJ LADIES 512x3,
  // 1024 x 16 / 12 -> 22.8 ms, 512 x 24 / 32 -> 31-33 ms, 384 x 40 -> 38.7 ms,
  // 256 x 64 -> 52.8 ms (the batch-layer phases are latency-bound: threads win)
  void (*kern)(LSParams) = layerwise_sm_kernel<1024, 12>;
  const int nt = 1024;
  GS_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int per_sm = 0, dev = 0, sms = 148;
  GS_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, nt, smem));
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int grid = std::max(1, per_sm) * sms;
  if (getenv("GS_VERBOSE")) fprintf(stderr, "layerwise_sm: %d threads, smem %zu B, %d CTAs/SM\n", nt, smem, per_sm);
  const int nctas = (int)std::max<int64_t>(1, std::min<int64_t>(grid, nbatch));
  P.meta = (int64_t*)blk->b_meta.ptr;
  P.err = (int*)blk->b_err.ptr;
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_err.ptr, 0, 16, stream));
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_ctr.ptr, 0, ls_align(8 * (MAX_LAYERS + 2)) + 256, stream));
  if (nbatch == 0) return GS_OK;
  kern<<<nctas, nt, smem, stream>>>(P); count_launch();
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

}  // namespace gsb
