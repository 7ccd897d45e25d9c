// nodewise_hop.cu -- node-wise ECSF sampling (GraphSAGE, KGCN, weighted
// A-Res, PASS-style A3), hop-synchronous: every hop of a group of mini-batches
// is five plain data-parallel kernels, no grid barrier, no cooperative launch,
// so an epoch is one CUDA-graph-capturable sequence of launches.
//
//   nprep    Extract, column side: per frontier column v,
//            (indptr[v], d(v)) and its sample count (min(k, d); k·[d > 0] with
//            replacement; min(k, #{w > 0}) weighted, from the a0 positive-
//            weight count); a single-pass scan of the counts (decoupled
//            look-back over 2048-column segments, per batch) is the block's CSC
//            indptr (column()), known before anything is sampled.
//   select   Extract + Select fused: a warp per
//            32 frontier columns (claimed dynamically), Floyd / replacement /
//            A-Res positions, every sampled row gathered at once (cp.async),
//            eid and the row id written straight to their final CSC position,
//            the row's bit set in the batch's N-bit row bitmap (red.or).
//   rows     row() (R3): single-pass scan of the bitmap's
//            popcounts (look-back over 2048-word tiles, per batch): each
//            64-bit bitmap word gets the rank of its first row in its high
//            half (bits stay in the low half); row_map = the set bits
//            ascending = the next frontier (R2), written coalesced.
//   relabel  per edge: row id -> rank = word.hi + popc(word.lo below u): one
//            L2 load per edge, in place.
//   clear    the hop's bitmap words back to zero (dense or via its rows).
// Sparse hops (rows << N) keep a summary bit per bitmap word so that rows /
// clear visit only non-empty words.  Groups of batches are sized so that a
// group's bitmaps stay resident in the 126 MB L2 when N allows.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <string>
#include <vector>
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "gs_internal.h"
#include "nodewise_common.cuh"

namespace gsb {

constexpr int HB_THREADS = 256;             // nprep / rows / relabel / clear
constexpr int HS_THREADS = 256;             // select
constexpr int HS_WARPS = HS_THREADS / 32;
constexpr int WPT = 8;                      // bitmap (dense) or summary (sparse) words per thread
#ifndef RW_THREADS
#define RW_THREADS 512                      // row(): threads per tile (512: hop-0 row() 0.078 vs 0.083 ms at 256)
#endif
constexpr int ROWS_TILE = RW_THREADS * WPT;        // bitmap words per dense rows tile
constexpr int SPARSE_TILE = RW_THREADS * WPT * 32; // bitmap words per summary-mode tile
constexpr int CLEAR_TILE = 8192;            // words per dense clear CTA
constexpr int NP_CPT = 8;                   // nprep: columns per thread
#ifndef NP_THREADS
#define NP_THREADS 256                      // nprep: threads per segment
#endif
constexpr int NP_SEG = NP_THREADS * NP_CPT; // columns per nprep segment
#ifndef RL_ILP
#define RL_ILP 4                            // relabel: edges per thread in flight (4 at 8 CTAs/SM: relabel1 0.130 vs 0.137 ms at 8 x 4 CTAs)
#endif
#ifndef RL_MINB
#define RL_MINB 8
#endif
// row() at 8 CTAs/SM (32 registers, 32 B of spills): rows0 / rows1 0.085 /
// 0.104 vs 0.099 / 0.119 ms at 40 registers (6 CTAs/SM); nprep at 4 CTAs/SM
// (64 registers): nprep1 0.083 vs 0.087 ms
#ifndef ROWS_MINB
#define ROWS_MINB (2048 / RW_THREADS)
#endif
#ifndef SP_B
#define SP_B 4                              // summary-mode row(): non-empty words loaded together
#endif
#ifndef NP_MINB
#define NP_MINB (1024 / NP_THREADS)
#endif
#if ROWS_MINB > 0
#define ROWS_LB __launch_bounds__(RW_THREADS, ROWS_MINB)
#else
#define ROWS_LB __launch_bounds__(RW_THREADS)
#endif
#if NP_MINB > 0
#define NP_LB __launch_bounds__(NP_THREADS, NP_MINB)
#else
#define NP_LB __launch_bounds__(NP_THREADS)
#endif
constexpr int RL_TILE = HB_THREADS * RL_ILP;
constexpr int MAX_GROUP = 512;              // batches per group (claim directories in smem)
#ifndef SEL_MINB
#define SEL_MINB 3
#endif
#ifndef SEL_MINB32
#define SEL_MINB32 2
#endif
constexpr int HW_CAP = 128;                 // A-Res candidates per warp
constexpr int ROW_STAGE = 16 * RW_THREADS;  // rows of a tile staged in smem for coalesced writes

struct HopParams {
  NWCore core;
  PhiloxKeys pk;             // round keys of core.key
  const int32_t* poscnt;     // weighted graphs: #{w > 0} per column (a0), else NULL
  const int32_t* seeds;
  const int64_t* bptr;       // [nb + 1] seed offsets of the batches (device)
  int64_t nb, batch_base;
  int L;
  int k[MAX_LAYERS];
  int64_t K[MAX_LAYERS];     // prod k[0..l]
  int use_sum[MAX_LAYERS];
  // outputs (DESIGN.md section 5 layout: fixed per-batch regions)
  int32_t* col0;
  int32_t* row_map[MAX_LAYERS];
  int64_t* indptr_out[MAX_LAYERS];
  int32_t* row_local[MAX_LAYERS];
  int64_t* eid[MAX_LAYERS];
  float* val[MAX_LAYERS];
  int64_t* meta;             // [nb][L][8]
  // workspace
  int64_t* coff;             // per frontier column: indptr[v] (column region of the hop)
  int32_t* dcol;             // per frontier column: in-degree (0 if the id is invalid)
  uint32_t* bm;              // [group slot][nwp] row bitmap, 32-bit words in 4-word groups; lay 1: node
                             // groups of 96 (hb_word), word 0 = the rank of the group's first row (row()),
                             // words 1..3 = bits; lay 0: 128 nodes per group, bits only, ranks in rank4
  int32_t* rank4;            // lay 0: [group slot][nwp / 4] rank of every non-empty group's first row
  int lay;                   // bitmap layout (1: rank inside the group -- one load per relabelled edge)
  int bm_keep;               // a group's bitmaps fit L2: their row bits are set with an evict-last hint
  int gather_normal;         // the graph reads of select / ares_big: evict-normal instead of evict-first
  uint32_t* summ;            // [group slot][nsw] bit w set iff bitmap word w is non-empty
  int64_t nw, nwp, nsw;      // words used / allocated per batch, summary words
  int sel_nq, sel_claim;     // select: claim queues, chunks per claim
  int ares_split;            // A-Res columns with d > 64: 1 hop_ares_big_kernel, 0 in select
  int ares_tau;              // hop_ares_big_kernel's first threshold: 0 normal, 1 too tight,
                             // 2 too loose (tests: every widen / narrow step runs)
};

// Row bitmap layout: node u lives in 16-byte group g = u / 96, bit word
// 1 + (u % 96) / 32 of it; word 0 of the group holds the rank of the group's
// first row once row() ran, so relabel reads one 16-byte group per edge.
constexpr uint32_t HB_GNODES = 96;
__device__ __forceinline__ uint32_t hb_word(uint32_t u) {
  const uint32_t g = u / HB_GNODES;
  return g * 4u + 1u + ((u - g * HB_GNODES) >> 5);
}
__device__ __forceinline__ uint32_t hb_bit(uint32_t u) { return 1u << ((u - (u / HB_GNODES) * HB_GNODES) & 31); }
// A row bit set fire-and-forget; bm_keep (the group's bitmaps fit L2): with an
// evict-last hint, so the gathers streaming through L2 do not push the bitmap
// out before row() / relabel / clear read it.
__device__ __forceinline__ void bm_or(uint32_t* w, uint32_t bit, int keep, uint64_t pk) {
  if (keep)
    asm volatile("red.global.or.L2::cache_hint.b32 [%0], %1, %2;" ::"l"(w), "r"(bit), "l"(pk) : "memory");
  else
    asm volatile("red.global.or.b32 [%0], %1;" ::"l"(w), "r"(bit) : "memory");
}
// the word and bit of node u in either layout
__device__ __forceinline__ uint32_t hb_wd(int lay, uint32_t u) { return lay ? hb_word(u) : (u >> 5); }
__device__ __forceinline__ uint32_t hb_bt(int lay, uint32_t u) { return lay ? hb_bit(u) : 1u << (u & 31); }

// Per-launch scan bookkeeping of nprep / rows (zeroed before the launch):
// ticket counter + one look-back status word per (batch, segment).
struct Scan {
  unsigned int* ticket;
  unsigned long long* status;
};

__device__ __forceinline__ int64_t hp_cbase(const HopParams& P, int64_t b, int l) {
  return __ldg(P.bptr + b) * (l == 0 ? 1 : P.K[l - 1]);
}
__device__ __forceinline__ const int32_t* hp_frontier(const HopParams& P, int64_t b, int l) {
  return l == 0 ? P.seeds + __ldg(P.bptr + b) : P.row_map[l - 1] + __ldg(P.bptr + b) * P.K[l - 1];
}
// frontier size of hop l before / after nprep(l)
__device__ __forceinline__ long long hp_T0(const HopParams& P, int64_t b, int l) {
  return l == 0 ? (long long)(__ldg(P.bptr + b + 1) - __ldg(P.bptr + b))
                : __ldcg((const long long*)P.meta + (b * P.L + l - 1) * 8 + 1);
}
__device__ __forceinline__ long long hp_T(const HopParams& P, int64_t b, int l) {
  return __ldcg((const long long*)P.meta + (b * P.L + l) * 8);
}
// sample count of column v (degree d) at hop l (R5, R6, R10)
__device__ __forceinline__ int hp_count(const HopParams& P, int l, int32_t v, int64_t d) {
  const int k = P.k[l];
  if (P.core.replace) return d > 0 ? k : 0;
  if (P.poscnt) return d > 0 ? min(k, __ldg(P.poscnt + v)) : 0;  // A-Res: min(k, #{w > 0})
  return d < k ? (int)d : k;
}

// ---------------------------------------------------------------------------
// Decoupled look-back (single-pass scan): status word = flag (2 bits) | value.
// Segment s of a chain publishes its aggregate, then warp 0 inspects the 32
// preceding status words at once: the values up to the nearest inclusive
// prefix are summed (all must be published), else the whole window is summed
// and the window moves back.  Segments take tickets in chain order, so every
// segment waited on is already running.  Called by warp 0 (all 32 lanes);
// returns the exclusive prefix in every lane.
// ---------------------------------------------------------------------------
constexpr unsigned long long LB_AGG = 1ull << 62, LB_INC = 2ull << 62, LB_VAL = (1ull << 62) - 1;
__device__ long long lookback(unsigned long long* st, int s, long long agg) {
  volatile unsigned long long* vs = st;
  const int lane = threadIdx.x & 31;
  if (s == 0) {
    if (lane == 0) vs[0] = LB_INC | (unsigned long long)agg;
    return 0;
  }
  if (lane == 0) vs[s] = LB_AGG | (unsigned long long)agg;
  long long ex = 0;
  int base = s - 1;
  while (true) {
    const int i = base - lane;
    const unsigned long long w = i >= 0 ? vs[i] : (2ull << 62);  // before the chain: inclusive 0
    const unsigned flag = (unsigned)(w >> 62);
    const unsigned inc = __ballot_sync(0xffffffffu, flag == 2);
    const unsigned zero = __ballot_sync(0xffffffffu, flag == 0);
    const int k = inc ? __ffs(inc) - 1 : 31;
    const unsigned need = k == 31 ? 0xffffffffu : ((2u << k) - 1u);
    if (zero & need) continue;  // a needed predecessor has not published yet
    long long v = lane <= k ? (long long)(w & LB_VAL) : 0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    ex += v;
    if (inc) break;
    base -= 32;
  }
  if (lane == 0) vs[s] = LB_INC | (unsigned long long)(ex + agg);
  return ex;
}

// Block-wide exclusive scan chained across a segment chain by the look-back
// above, in two barriers (a reduce, the look-back and a scan back to back
// took seven): returns this thread's exclusive prefix over the whole chain,
// *base the CTA's own prefix and *total its aggregate.  scr >= 34 entries.
__device__ __forceinline__ long long block_scan_chain(long long v, long long* scr, unsigned long long* status,
                                                      int seg, long long* base, long long* total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const long long inc = warp_inclusive_scan(v);
  if (lane == 31) scr[wid] = inc;
  __syncthreads();
  if (wid == 0) {
    const long long s = lane < nw ? scr[lane] : 0ll;
    const long long si = warp_inclusive_scan(s);
    const long long agg = __shfl_sync(0xffffffffu, si, nw - 1);
    const long long b = lookback(status, seg, agg);
    if (lane < nw) scr[lane] = b + si - s;
    if (lane == 0) {
      scr[32] = b;
      scr[33] = agg;
    }
  }
  __syncthreads();
  *base = scr[32];
  *total = scr[33];
  return inc - v + scr[wid];
}

// Directory of a group: dir[i] = segments of the group's batches before i;
// ticket -> (batch slot, segment).  All threads; ends synchronised.
template <class NSEG>
__device__ void seg_directory(int nbg, long long* dir, long long* scr, NSEG&& nseg) {
  long long run = 0;
  for (int i0 = 0; i0 < nbg; i0 += blockDim.x) {
    const int i = i0 + threadIdx.x;
    const long long c = i < nbg ? nseg(i) : 0;
    long long tot;
    const long long ex = block_exclusive_scan<long long>(c, scr, &tot);
    if (i < nbg) dir[i] = run + ex;
    run += tot;
  }
  if (threadIdx.x == 0) dir[nbg] = run;
  __syncthreads();
}
__device__ __forceinline__ int dir_find(const long long* dir, int nbg, long long c) {
  int lo = 0, hi = nbg - 1;  // last i with dir[i] <= c
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (dir[mid] <= c) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

// ---------------------------------------------------------------------------
// nprep: hop l's column side, one 2048-column segment per CTA (tickets over
// the group's (batch, segment) pairs in batch order).
// ---------------------------------------------------------------------------
__global__ void NP_LB hop_nprep_kernel(HopParams P, int l, int64_t b0, int nbg, Scan S) {
  __shared__ long long dir[MAX_GROUP + 1];
  __shared__ long long scr[40];
  __shared__ long long sh[2];
  seg_directory(nbg, dir, scr, [&](int i) {
    return max(1ll, (hp_T0(P, b0 + i, l) + NP_SEG - 1) / NP_SEG);  // >= 1: meta is always written
  });
  if (threadIdx.x == 0) sh[0] = (long long)atomicAdd(S.ticket, 1u);
  __syncthreads();
  const long long c = sh[0];
  if (c >= dir[nbg]) return;
  const int i = dir_find(dir, nbg, c);
  const int64_t b = b0 + i;
  const int seg = (int)(c - dir[i]);
  const long long T = hp_T0(P, b, l);
  const int32_t* F = hp_frontier(P, b, l);
  const int64_t s0 = __ldg(P.bptr + b);
  const int64_t cb = hp_cbase(P, b, l), ib = cb + b, rb = s0 * P.K[l];
  const long long j0 = (long long)seg * NP_SEG + (long long)threadIdx.x * NP_CPT;
  int cnt[NP_CPT];
  long long sum = 0;
  int32_t v[NP_CPT];
#pragma unroll
  for (int q = 0; q < NP_CPT; ++q) v[q] = ldcg_if(j0 + q < T, F + j0 + q, -1);
  // predicated loads (no branch between them: all 16 in flight at once), the
  // range check's error flag after them
  int64_t off[NP_CPT], d[NP_CPT];
  bool bad = false;
#pragma unroll
  for (int q = 0; q < NP_CPT; ++q) {
    const bool act = j0 + q < T;
    const bool valid = act && v[q] >= 0 && (int64_t)v[q] < P.core.N;
    bad |= act && !valid;
    off[q] = ldg_if(valid, P.core.indptr + v[q], (int64_t)0);
    d[q] = ldg_if(valid, P.core.indptr + v[q] + 1, (int64_t)0);
  }
#pragma unroll
  for (int q = 0; q < NP_CPT; ++q) d[q] -= off[q];
  if (bad) atomicOr(P.core.err, ERR_SEED_RANGE);
  // weighted (A-Res): the a0 positive-weight counts, all in flight together
  int pc[NP_CPT];
  const bool use_pc = !P.core.replace && P.poscnt != nullptr;
#pragma unroll
  for (int q = 0; q < NP_CPT; ++q) pc[q] = ldg_if(use_pc && d[q] > 0, P.poscnt + v[q], 0);
#pragma unroll
  for (int q = 0; q < NP_CPT; ++q) {
    cnt[q] = use_pc ? (d[q] > 0 ? min(P.k[l], pc[q]) : 0) : hp_count(P, l, v[q], d[q]);  // = hp_count
    sum += cnt[q];
  }
  long long sbase, tot;
  long long ex = block_scan_chain(sum, scr, S.status + (c - seg), seg, &sbase, &tot);
#pragma unroll
  for (int q = 0; q < NP_CPT; ++q) {
    const long long jj = j0 + q;
    if (jj < T) {
      P.coff[cb + jj] = off[q];
      P.dcol[cb + jj] = (int32_t)d[q];
      P.indptr_out[l][ib + jj] = ex;
      if (l == 0) P.col0[s0 + jj] = v[q];
    }
    ex += cnt[q];
  }
  if (threadIdx.x == NP_THREADS - 1 && (long long)(seg + 1) * NP_SEG >= T) {  // the batch's last segment
    P.indptr_out[l][ib + T] = ex;
    long long* m = (long long*)(P.meta + (b * P.L + l) * 8);
    m[0] = T; m[1] = 0; m[2] = ex; m[3] = cb; m[4] = rb; m[5] = ib; m[6] = rb; m[7] = 0;
  }
}

// ---------------------------------------------------------------------------
// select: a warp per 32-column chunk.
// ---------------------------------------------------------------------------
// Ascending bitonic sorting network over a register array (N a power of two).
template <int N>
__device__ __forceinline__ void sort_net(uint32_t (&a)[N]) {
  if constexpr ((N & (N - 1)) != 0) {
    // N not a power of two: odd-even transposition (N rounds)
#pragma unroll
    for (int r = 0; r < N; ++r) {
#pragma unroll
      for (int i = r & 1; i + 1 < N; i += 2) {
        const uint32_t x = a[i], y = a[i + 1];
        a[i] = x < y ? x : y;
        a[i + 1] = x < y ? y : x;
      }
    }
    return;
  }
#pragma unroll
  for (int kk = 2; kk <= N; kk <<= 1) {
#pragma unroll
    for (int jj = kk >> 1; jj > 0; jj >>= 1) {
#pragma unroll
      for (int i = 0; i < N; ++i) {
        const int o = i ^ jj;
        if (o > i) {
          const bool up = (i & kk) == 0;
          const uint32_t x = a[i], y = a[o];
          const bool sw = up ? (x > y) : (x < y);
          a[i] = sw ? y : x;
          a[o] = sw ? x : y;
        }
      }
    }
  }
}

template <int KCAP, bool WEIGHTED>
struct HChunk {
  unsigned long long se[32 * KCAP];  // flat staging (slot-major): edge id
  uint32_t su[32 * KCAP];            // ... gathered row id
};
template <int KCAP>
struct HChunk<KCAP, true> {  // (>= 16 slots per lane: the k < d <= 64 group lists alias se / su / sv)
  unsigned long long se[32 * (KCAP < 16 ? 16 : KCAP)];
  uint32_t su[32 * (KCAP < 16 ? 16 : KCAP)];
  float sv[32 * (KCAP < 16 ? 16 : KCAP)];  // ... PASS value
  uint32_t list[KCAP][32];           // selected positions, [rank][column lane]
};

struct HWarpA {
  uint32_t pos[HW_CAP];
  double key[HW_CAP];
  int rk[HW_CAP];
  AresState st;
};

template <bool WEIGHTED, int KCAP>
struct HSmem {
  HChunk<KCAP, WEIGHTED> ch[HS_WARPS];
  long long cpre[MAX_GROUP + 1];  // chunk prefix over the group's batches
  long long scr[40];
};  // weighted: HWarpA[HS_WARPS] follows in dynamic shared memory

// One warp = 32 frontier columns, a lane per column: positions in registers,
// the lane's sampled rows gathered 16 at a time, bitmap bits set, edge id / row
// id staged slot-major in shared memory, then written out coalesced.
template <bool WEIGHTED, int KCAP>
#ifndef SEL_MINB8
#define SEL_MINB8 3
#endif
#ifndef SEL_U12
#define SEL_U12 12                          // uniform 8 < k <= 12: a 12-slot variant
#endif
#ifndef SEL_W12
#define SEL_W12 12                          // weighted 8 < k <= 12: a 12-slot variant
#endif
#ifndef SEL_MINBW8
#define SEL_MINBW8 2                        // weighted k <= 8 (PP hop 2): select2 20.5 ms vs 22.6 at 3 CTAs/SM, 23.0 with the 16-slot variant
#endif
__global__ void __launch_bounds__(HS_THREADS, (WEIGHTED ? (KCAP <= 8 ? SEL_MINBW8 : 2) : (KCAP <= 8 ? SEL_MINB8 : (KCAP <= 16 ? SEL_MINB : SEL_MINB32)))) hop_select_kernel(HopParams P, int l, int64_t b0, int nbg,
                                                                 unsigned int* claim) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  using SM = HSmem<WEIGHTED, KCAP>;
  SM& sm = *reinterpret_cast<SM*>(smem_raw);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  // chunk directory: cpre[i] = 32-column chunks of the group's batches before i
  {
    long long run = 0;
    for (int i0 = 0; i0 < nbg; i0 += HS_THREADS) {
      const int i = i0 + threadIdx.x;
      const long long c = i < nbg ? (hp_T(P, b0 + i, l) + 31) / 32 : 0;
      long long tot;
      const long long ex = block_exclusive_scan<long long>(c, sm.scr, &tot);
      if (i < nbg) sm.cpre[i] = run + ex;
      run += tot;
    }
    if (threadIdx.x == 0) sm.cpre[nbg] = run;
    __syncthreads();
  }
  const long long nchunks = sm.cpre[nbg];
  HChunk<KCAP, WEIGHTED>& C = sm.ch[warp];
  const int k = P.k[l];
  const uint64_t pf = P.gather_normal ? pol_normal() : pol_first(), pk = pol_last();
#ifndef SEL_EID_FIRST
#define SEL_EID_FIRST 1
#endif
  const uint64_t pe = SEL_EID_FIRST ? pol_first() : pf;
  const int use_sum = P.use_sum[l];
  // chunks are claimed from NQ queues (contiguous chunk ranges, counters
  // 128 B apart): a warp drains its home queue, then steals from the next
  // ones -- one counter hit by every warp serialises the claims otherwise
  const int NQ = P.sel_nq;
  const int CLAIM = (int)min((long long)P.sel_claim, max(1ll, nchunks / ((long long)gridDim.x * HS_WARPS * 4)));
  const long long qlen = (nchunks + NQ - 1) / NQ;
  int q = (int)((blockIdx.x * HS_WARPS + warp) % NQ), visited = 0;
  auto grab = [&]() -> long long {
    while (visited < NQ) {
      unsigned int x = 0;
      if (lane == 0) x = atomicAdd(claim + q * 32, (unsigned)CLAIM);
      x = __shfl_sync(0xffffffffu, x, 0);
      const long long c0 = (long long)q * qlen + x;
      if ((long long)x < qlen && c0 < nchunks) return c0;
      q = (q + 1) % NQ;
      ++visited;
    }
    return -1;
  };
  long long c = grab();
  long long cend = c < 0 ? -1 : min(min(c + CLAIM, (long long)(q + 1) * qlen), nchunks);
  int lo = 0;  // batch slot of the previous chunk (claims mostly stay in one batch)
  while (c >= 0) {
    if (!(sm.cpre[lo] <= c && c < sm.cpre[lo + 1])) {
      int lo2 = 0, hi2 = nbg - 1;  // batch slot: last i with cpre[i] <= c
      while (lo2 < hi2) {
        const int mid = (lo2 + hi2 + 1) >> 1;
        if (sm.cpre[mid] <= c) lo2 = mid;
        else hi2 = mid - 1;
      }
      lo = lo2;
    }
    const int64_t b = b0 + lo;
    const long long T = hp_T(P, b, l);
    const long long jb = (c - sm.cpre[lo]) * 32;
    const int64_t cb = hp_cbase(P, b, l);
    const int64_t rb = __ldg(P.bptr + b) * P.K[l];
    const uint32_t gb = (uint32_t)(P.batch_base + b);
    const long long jcol = jb + lane;
    const bool active = jcol < T;
    const int32_t* F = hp_frontier(P, b, l);
    const int32_t v = active ? __ldcg(F + jcol) : -1;
    const int64_t off = active ? __ldcg(P.coff + cb + jcol) : 0;
    const int64_t d = active ? (int64_t)__ldcg(P.dcol + cb + jcol) : 0;
    const int64_t ebase = __ldcg(P.indptr_out[l] + cb + b + jb);  // first edge of the chunk
    int cnt = 0;
    bool all = false;
    bool defer = false;  // weighted, d > 64: written by hop_ares_big_kernel
    float csum = 1.0f;
    uint32_t a[KCAP];  // positions (compile-time indexed registers)
#pragma unroll
    for (int i = 0; i < KCAP; ++i) a[i] = 0xFFFFFFFFu;
    if constexpr (!WEIGHTED) {
      if (P.core.replace) {  // KGCN (R10): k i.i.d. positions in slot order
        cnt = d > 0 ? k : 0;
        for (int s = 0; s < cnt; ++s) {
          const U4 r = philox_k((uint32_t)v, (uint32_t)s, ctr2(l, TAG_REPLACE), gb, P.pk);
          const uint32_t x = (uint32_t)draw_below((uint64_t)d, r.x, r.y);
#pragma unroll
          for (int i = 0; i < KCAP; ++i) if (i == s) a[i] = x;
        }
      } else if (d <= k) {  // GraphSAGE, d <= k: every neighbour (R5)
        cnt = (int)d;
        all = true;
      } else {  // GraphSAGE (R5): Floyd (membership test against the unsorted set), then sorted
        cnt = k;
        for (int s = 0; s < k; ++s) {
          const U4 r = philox_k((uint32_t)v, (uint32_t)s, ctr2(l, TAG_FLOYD), gb, P.pk);
          const uint32_t m = (uint32_t)(d - k + s);
          const uint32_t t = (uint32_t)draw_below((uint64_t)m + 1, r.x, r.y);
          bool dup = false;
#pragma unroll
          for (int i = 0; i < KCAP; ++i) dup |= a[i] == t;  // free slots hold ~0 > any position
          const uint32_t x = dup ? m : t;
#pragma unroll
          for (int i = 0; i < KCAP; ++i) if (i == s) a[i] = x;
        }
        sort_net(a);
      }
    } else {
      // A-Res (R6): d <= k -> every eligible edge (lane per column); heavier
      // columns one at a time by the whole warp (candidate filtering)
      const float* wts = P.core.weights;
      if (d > 0 && P.core.bias == GS_W_PASS_COLNORM) csum = wts ? __ldg(P.core.colsum + v) : (float)d;
      if (d <= k) {  // the d weights loaded at once (unrolled), then the eligible ones listed
        float wl[KCAP];
#pragma unroll
        for (int i = 0; i < KCAP; ++i) wl[i] = i < d ? (wts ? __ldg(wts + off + i) : 1.0f) : 0.0f;
#pragma unroll
        for (int i = 0; i < KCAP; ++i)
          if (wl[i] > 0.0f) C.list[cnt++][lane] = (uint32_t)i;
      }
      HWarpA& A = reinterpret_cast<HWarpA*>(&sm + 1)[warp];
      // k < d <= 64: four columns at a time, eight lanes each (lane s holds
      // positions 32 t + 4 s + q).  Candidates x <= tau w (1 + 1%), tau =
      // (k + 8) / W, get exact fp64 keys; a group with fewer than want keys
      // below tau retakes every eligible edge.  The candidates are listed in
      // position order in shared memory (the idle staging area), each is
      // ranked by (key, position) against its group's list, and the want
      // winners are written in list order = position order.
      static_assert(sizeof(C.se) >= 4 * 64 * 12 && sizeof(C.su) >= 4 * 64 * 5 && sizeof(C.sv) >= 4 * 64 * 4,
                    "group lists");
      uint32_t sml = __ballot_sync(0xffffffffu, d > k && d <= 64);
      const int g8 = lane >> 3, s8 = lane & 7;
      double* gkey = reinterpret_cast<double*>(C.se) + g8 * 64;
      uint32_t* gpos = reinterpret_cast<uint32_t*>(reinterpret_cast<double*>(C.se) + 4 * 64) + g8 * 64;
      uint32_t* grnd = reinterpret_cast<uint32_t*>(C.su) + g8 * 64;
      uint8_t* gwin = reinterpret_cast<uint8_t*>(reinterpret_cast<uint32_t*>(C.su) + 4 * 64) + g8 * 64;
      float* gw = reinterpret_cast<float*>(C.sv) + g8 * 64;
      while (sml) {
        int cc = -1;
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          const int bt = __ffs(sml) - 1;
          if (sml) {
            sml &= sml - 1u;
            if (t == g8) cc = bt;
          }
        }
        const int src = cc < 0 ? 0 : cc;
        const int32_t vc = __shfl_sync(0xffffffffu, v, src);
        const int64_t oc = __shfl_sync(0xffffffffu, off, src);
        const int dsrc = __shfl_sync(0xffffffffu, (int)d, src);
        const int dc = cc < 0 ? 0 : dsrc;
        const float W = dc > 0 ? (wts ? __ldg(P.core.colsum + vc) : (float)dc) : 0.0f;
        uint32_t rw[8];
        float w8[8];
        int elig = 0;
#pragma unroll
        for (int t = 0; t < 2; ++t) {
          const int i0 = 32 * t + 4 * s8;
          U4 R{0u, 0u, 0u, 0u};
          if (i0 < dc) R = philox_k((uint32_t)vc, (uint32_t)(i0 >> 2), ctr2(l, TAG_ARES_NODE), gb, P.pk);
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            w8[4 * t + q] = i0 + q < dc ? (wts ? __ldg(wts + oc + i0 + q) : 1.0f) : 0.0f;
            rw[4 * t + q] = sel_word(R, q);
            elig += w8[4 * t + q] > 0.0f ? 1 : 0;
          }
        }
        elig += __shfl_xor_sync(0xffffffffu, elig, 4);
        elig += __shfl_xor_sync(0xffffffffu, elig, 2);
        elig += __shfl_xor_sync(0xffffffffu, elig, 1);
        const int want = min(k, elig);
        float tau = W > 0.0f ? (float)(k + 8) / W : -1.0f;
        if (P.ares_tau == 1) tau *= 0.25f;
        int M = 0;
        for (int pass = 0; pass < 2; ++pass) {
          // candidates (no logarithm yet), listed in position order (t, lane, q)
          const float t32 = __fmul_rn(__fmul_rn(tau, 1.01f), 4294967296.0f);
          unsigned cm = 0u;
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const bool cnd = w8[j] > 0.0f && (tau < 0.0f || __uint2float_rn(~rw[j]) <= __fmaf_rn(t32, w8[j], -0.5f));
            cm |= cnd ? (1u << j) : 0u;
          }
          __syncwarp();
          M = 0;
#pragma unroll
          for (int t = 0; t < 2; ++t) {
            const int c = __popc((cm >> (4 * t)) & 0xFu);
            int x = c;
#pragma unroll
            for (int o = 1; o < 8; o <<= 1) {
              const int y = __shfl_up_sync(0xffffffffu, x, o, 8);
              if (s8 >= o) x += y;
            }
            int o = M + x - c;
            M += __shfl_sync(0xffffffffu, x, 7, 8);
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const int j = 4 * t + q;
              if (cm & (1u << j)) {
                gpos[o] = (uint32_t)(32 * t + 4 * s8 + q);
                grnd[o] = rw[j];
                gw[o] = w8[j];
                ++o;
              }
            }
          }
          __syncwarp();
          // exact keys of the listed candidates, eight lanes per group
          int below = 0;
          for (int e = s8; e < M; e += 8) {
            const double ke = ares_key_nl(grnd[e], (double)gw[e]);
            gkey[e] = ke;
            below += (tau < 0.0f || ke < (double)tau) ? 1 : 0;
          }
          below += __shfl_xor_sync(0xffffffffu, below, 4);
          below += __shfl_xor_sync(0xffffffffu, below, 2);
          below += __shfl_xor_sync(0xffffffffu, below, 1);
          const bool redo = below < want;
          if (!__any_sync(0xffffffffu, redo)) break;
          if (redo) tau = -1.0f;  // every eligible edge (the others recompute the same)
        }
        __syncwarp();
        // rank the list entries s, s + 8, ... of the group against all M
        for (int e = s8; e < M; e += 8) {
          const double ke = gkey[e];
          const uint32_t pe = gpos[e];
          int r = 0;
          for (int i = 0; i < M; ++i) r += key_less(gkey[i], gpos[i], ke, pe) ? 1 : 0;
          gwin[e] = r < want ? 1 : 0;
        }
        __syncwarp();
        for (int e = s8; e < M; e += 8) {
          if (gwin[e]) {
            int o = 0;
            for (int i = 0; i < e; ++i) o += gwin[i];
            C.list[o][cc] = gpos[e];
          }
        }
        if (cc >= 0 && s8 == 0) A.rk[cc] = want;
        __syncwarp();
      }
      if (d > k && d <= 64) cnt = A.rk[lane];
      __syncwarp();
      // d > 64: the heavy-column kernel (hop_ares_big_kernel) selects, gathers
      // and writes these columns; here only their output range is reserved
      const bool big = d > 64;
      if (big && P.ares_split) {
        defer = true;
        cnt = min(k, P.poscnt && wts ? __ldg(P.poscnt + v) : (int)d);
      }
      uint32_t med = __ballot_sync(0xffffffffu, big && !defer);
      while (med) {
        const int cc = __ffs(med) - 1;
        med &= med - 1u;
        const int32_t vc = __shfl_sync(0xffffffffu, v, cc);
        const int64_t oc = __shfl_sync(0xffffffffu, off, cc);
        const int64_t dc = __shfl_sync(0xffffffffu, d, cc);
        const float W = wts ? __ldg(P.core.colsum + vc) : (float)dc;
        const float tau0 = dc <= 64 ? -1.0f : (W > 0.0f ? 2.0f * (float)k / W : -1.0f);
        TauSearch ts{tau0, 0.0f, 0.0f};
        int r;
        while (true) {
          if (lane == 0) A.st = AresState{0, 0};
          __syncwarp();
          ares_filter<32>(P.core, vc, oc, dc, l, gb, ts.tau, lane, A.pos, HW_CAP, &A.st);
          __syncwarp();
          r = ares_exact(P.core, vc, oc, l, gb, k, ts.tau, A.pos, A.key, A.rk, HW_CAP, A.st, C.list, cc);
          if (r >= 0) break;
          if (!ts.next(r, tau0 > 0.0f ? tau0 : 2.0f * k / (float)dc)) {
            if (lane == 0) atomicOr(P.core.err, ERR_INTERNAL);
            r = 0;
            break;
          }
        }
        if (lane == cc) cnt = r;
        __syncwarp();
      }
      __syncwarp();
#pragma unroll
      for (int i = 0; i < KCAP; ++i)
        if (i < cnt) a[i] = C.list[i][lane];
    }
    int total;
    const int pre = warp_excl(cnt, &total);
    // gather (16 loads in flight per lane), bitmap bits, slot-major staging
    const int64_t slot = b - b0;
    uint32_t* bits = P.bm + slot * P.nwp;
    uint32_t* summ = P.summ + slot * P.nsw;
#pragma unroll
    for (int h = 0; h < KCAP; h += 16) {
      uint32_t u[16];
#pragma unroll
      for (int q = 0; q < 16 && h + q < KCAP; ++q) {
        const int i = h + q;
        const uint32_t ps = all ? (uint32_t)i : a[i];
        u[q] = ldg_h_if(i < cnt && !defer, P.core.indices + off + ps, pf, 0u);
      }
#pragma unroll
      for (int q = 0; q < 16 && h + q < KCAP; ++q) {
        const int i = h + q;
        if (i < cnt && defer) {
          C.se[pre + i] = ~0ull;  // reserved (hop_ares_big_kernel)
        } else if (i < cnt) {
          const uint32_t ps = all ? (uint32_t)i : a[i];
          C.se[pre + i] = (unsigned long long)(off + ps);
          C.su[pre + i] = u[q];
          if constexpr (WEIGHTED) {
            if (P.val[l]) {
              const float w = P.core.weights ? __ldg(P.core.weights + off + ps) : 1.0f;
              C.sv[pre + i] = w / csum;
            }
          }
          const uint32_t wd = hb_wd(P.lay, u[q]);
          bm_or(bits + wd, hb_bt(P.lay, u[q]), P.bm_keep, pk);
          if (use_sum) bm_or(summ + (wd >> 5), 1u << (wd & 31), P.bm_keep, pk);
        }
      }
    }
    __syncwarp();
    int32_t* rl_out = P.row_local[l] + rb + ebase;
    int64_t* eid_out = P.eid[l] + rb + ebase;
    float* val_out = P.val[l] ? P.val[l] + rb + ebase : nullptr;
    for (int f = lane; f < total; f += 32) {
      if (WEIGHTED && C.se[f] == ~0ull) continue;
      sth(eid_out + f, (int64_t)C.se[f], pe);  // edge ids: never read again on the device
      sth(rl_out + f, (int32_t)C.su[f], pf);
      if constexpr (WEIGHTED) {
        if (val_out) sth(val_out + f, C.sv[f], pf);
      }
    }
    __syncwarp();
    if (++c >= cend) {
      c = grab();
      cend = c < 0 ? -1 : min(min(c + CLAIM, (long long)(q + 1) * qlen), nchunks);
    }
  }
}

// ---------------------------------------------------------------------------
// A-Res (R6) for the heavy columns (d > 64) of a hop: a warp per column, in a
// lean kernel of its own (2 KB of shared memory and <= 64 registers per warp,
// so 32 warps per SM hide the weight stream's latency; inside the select
// kernel the same loop ran at 16 warps per SM and stalled on instruction
// fetch).  Candidate filter (one Philox per 4 edges, the next 128 edges'
// weights loaded while the current ones are tested), exact fp64 keys of the
// <= 128 candidates held in registers, want = min(k, eligible) rounds of a
// warp argmin over (key, position), then the winners in position order are
// gathered and written to the block's reserved CSC range (hop_select left it
// untouched) and their rows' bitmap bits set.
// ---------------------------------------------------------------------------
constexpr int AB_THREADS = 256;
constexpr int AB_WARPS = AB_THREADS / 32;
constexpr int AB_CAP = 128;  // candidates per column pass (4 per lane)
#ifndef AB_MINB
#define AB_MINB 3            // CTAs per SM (80 registers; 4 -> 64 registers spills)
#endif

__global__ void __launch_bounds__(AB_THREADS, AB_MINB) hop_ares_big_kernel(HopParams P, int l, int64_t b0, int nbg,
                                                                     unsigned int* claim) {
  __shared__ long long cpre[MAX_GROUP + 1];
  __shared__ long long scr[40];
  __shared__ uint32_t cpos[AB_WARPS][AB_CAP];  // candidates: position, random word, weight
  __shared__ uint32_t crnd[AB_WARPS][AB_CAP];
  __shared__ float cwt[AB_WARPS][AB_CAP];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  {
    long long run = 0;
    for (int i0 = 0; i0 < nbg; i0 += AB_THREADS) {
      const int i = i0 + threadIdx.x;
      const long long c = i < nbg ? (hp_T(P, b0 + i, l) + 31) / 32 : 0;
      long long tot;
      const long long ex = block_exclusive_scan<long long>(c, scr, &tot);
      if (i < nbg) cpre[i] = run + ex;
      run += tot;
    }
    if (threadIdx.x == 0) cpre[nbg] = run;
    __syncthreads();
  }
  const long long nchunks = cpre[nbg];
  const int k = P.k[l];
  const uint64_t pf = P.gather_normal ? pol_normal() : pol_first(), pk = pol_last();
  const float* wts = P.core.weights;
  uint32_t* pos = cpos[warp];
  uint32_t* rnd = crnd[warp];
  float* cw = cwt[warp];
  int lo = 0;
  for (;;) {
    unsigned int x = 0;
    if (lane == 0) x = atomicAdd(claim, 1u);
    const long long c = (long long)__shfl_sync(0xffffffffu, x, 0);
    if (c >= nchunks) break;
    if (!(cpre[lo] <= c && c < cpre[lo + 1])) {
      int lo2 = 0, hi2 = nbg - 1;
      while (lo2 < hi2) {
        const int mid = (lo2 + hi2 + 1) >> 1;
        if (cpre[mid] <= c) lo2 = mid;
        else hi2 = mid - 1;
      }
      lo = lo2;
    }
    const int64_t b = b0 + lo;
    const long long T = hp_T(P, b, l);
    const long long jb = (c - cpre[lo]) * 32;
    const int64_t cb = hp_cbase(P, b, l);
    const int64_t rb = __ldg(P.bptr + b) * P.K[l];
    const uint32_t gb = (uint32_t)(P.batch_base + b);
    const long long jcol = jb + lane;
    const bool active = jcol < T;
    const int64_t d = active ? (int64_t)__ldcg(P.dcol + cb + jcol) : 0;
    uint32_t bigm = __ballot_sync(0xffffffffu, d > 64);
    if (!bigm) continue;
    const int32_t* F = hp_frontier(P, b, l);
    const int32_t v = active ? __ldcg(F + jcol) : -1;
    const int64_t off = active ? __ldcg(P.coff + cb + jcol) : 0;
    const int64_t slot = b - b0;
    uint32_t* bits = P.bm + slot * P.nwp;
    uint32_t* summ = P.summ + slot * P.nsw;
    const int use_sum = P.use_sum[l];
    // per-column a0 values and output offsets, loaded for all heavy columns
    // of the chunk at once (one latency per chunk, not three per column)
    const bool mybig = d > 64;
    const int my_elig = mybig ? (P.poscnt && wts ? __ldg(P.poscnt + v) : (int)d) : 0;
    const float my_W = mybig ? (wts ? __ldg(P.core.colsum + v) : (float)d) : 0.0f;
    const int64_t my_ce = mybig ? __ldcg(P.indptr_out[l] + cb + b + jcol) : 0;  // the column's first edge
    while (bigm) {
      const int cc = __ffs(bigm) - 1;
      bigm &= bigm - 1u;
      const int32_t vc = __shfl_sync(0xffffffffu, v, cc);
      const int64_t oc = __shfl_sync(0xffffffffu, off, cc);
      const int dc = (int)__shfl_sync(0xffffffffu, d, cc);
      const int elig = __shfl_sync(0xffffffffu, my_elig, cc);
      const float W = __shfl_sync(0xffffffffu, my_W, cc);
      const int64_t ce = __shfl_sync(0xffffffffu, my_ce, cc);
      const int want = min(k, elig);
      if (want == 0) continue;
      // tau ~ (k + 8) / W expects k + 8 keys below it (widened when fewer
      // than want, narrowed when the candidates overflow); tau < 0: every
      // eligible edge is a candidate
      const float tau0 = W > 0.0f ? (float)(k + 8) / W : -1.0f;
      float tau = tau0 < 0.0f ? -1.0f : (P.ares_tau == 1 ? 0.25f * tau0 : (P.ares_tau == 2 ? 16.0f * tau0 : tau0));
      TauSearch ts{tau, 0.0f, 0.0f};
      const float* wc = wts ? wts + oc : nullptr;
      double kk[4];
      uint32_t pp[4];
      int M = 0;
      bool good = false;
      const unsigned lt = (1u << lane) - 1u;
      for (int it = 0; it < 64 && !good; ++it) {
        tau = ts.tau;
        const float t32 = __fmul_rn(__fmul_rn(tau, 1.01f), 4294967296.0f);
        // filter: candidate iff x <= tau w (1 + 1%), x = (2^32 - r - 0.5) 2^-32:
        // E(r) = -ln(1 - x) >= x, so every key below tau is a candidate
        M = 0;
        float wn[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const int i = 4 * lane + q;
          wn[q] = i < dc ? (wc ? ldg_h(wc + i, pf) : 1.0f) : 0.0f;
        }
        for (int base = 0; base < dc; base += 128) {
          float w[4];
#pragma unroll
          for (int q = 0; q < 4; ++q) w[q] = wn[q];
          const int i0 = base + 4 * lane;
          if (base + 128 < dc) {
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const int i = i0 + 128 + q;
              wn[q] = i < dc ? (wc ? ldg_h(wc + i, pf) : 1.0f) : 0.0f;
            }
          }
          unsigned fl = 0u;
          const U4 R = philox_k((uint32_t)vc, (uint32_t)(i0 >> 2), ctr2(l, TAG_ARES_NODE), gb, P.pk);
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            // x <= tau w (1 + 1%) in units of 2^-32 (w = 0: the bound is < 0)
            const bool cnd = tau < 0.0f ? w[q] > 0.0f
                                        : __uint2float_rn(~sel_word(R, q)) <= __fmaf_rn(t32, w[q], -0.5f);
            fl |= cnd ? (1u << q) : 0u;
          }
          // append in (lane, q) order -- position order -- with the prefix of
          // the per-lane counts from bit ballots
          const int n = __popc(fl);
          const unsigned b0 = __ballot_sync(0xffffffffu, n & 1), b1 = __ballot_sync(0xffffffffu, n & 2),
                         b2 = __ballot_sync(0xffffffffu, n & 4);
          if (b0 | b1 | b2) {
            int o = M + __popc(b0 & lt) + 2 * __popc(b1 & lt) + 4 * __popc(b2 & lt);
#pragma unroll
            for (int q = 0; q < 4; ++q)
              if (fl & (1u << q)) {
                if (o < AB_CAP) {
                  pos[o] = (uint32_t)(i0 + q);
                  rnd[o] = sel_word(R, q);
                  cw[o] = w[q];
                }
                ++o;
              }
            M += __popc(b0) + 2 * __popc(b1) + 4 * __popc(b2);
          }
        }
        __syncwarp();
        if (M > AB_CAP) {  // too many candidates: narrow
          if (!ts.next(-2, tau0)) break;
          continue;
        }
        // exact keys (fp64, as the oracle)
        int below = 0;
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          const int j = lane + 32 * t;
          kk[t] = INFINITY;
          pp[t] = 0xFFFFFFFFu;
          if (32 * t < M && j < M) {
            kk[t] = ares_key(rnd[j], (double)cw[j]);
            pp[t] = pos[j];
            below += (tau < 0.0f || kk[t] < (double)tau) ? 1 : 0;
          }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) below += __shfl_xor_sync(0xffffffffu, below, o);
        __syncwarp();
        if (below < want) {  // too few keys below tau: widen
          if (!ts.next(-1, tau0)) break;
          continue;
        }
        good = true;
      }
      if (!good) {
        if (lane == 0) atomicOr(P.core.err, ERR_INTERNAL);
        continue;
      }
      uint32_t mine = 0xFFFFFFFFu;  // a winner's position
      int o = 0;                     // its rank in position order
      bool sel = false;
      if (M <= 20) {
        // rank of each candidate by (key, position) against all M; the pool
        // is in position order, so the winners' order is their lane order
        const double K = kk[0];
        const uint32_t Q = pp[0];
        int r = 0;
        for (int i = 0; i < M; ++i) {
          const double ok = __shfl_sync(0xffffffffu, K, i);
          const uint32_t oq = __shfl_sync(0xffffffffu, Q, i);
          r += key_less(ok, oq, K, Q) ? 1 : 0;
        }
        sel = lane < M && r < want;
        o = __popc(__ballot_sync(0xffffffffu, sel) & lt);
        mine = Q;
      } else {
        if (M <= 32) {
          // one candidate per lane: bitonic sort of (key, position) across
          // the warp; lanes 0 .. want-1 then hold the want smallest
          double K = kk[0];
          uint32_t Q = pp[0];
#pragma unroll
          for (int size = 2; size <= 32; size <<= 1) {
#pragma unroll
            for (int stride = size >> 1; stride > 0; stride >>= 1) {
              const double ok = __shfl_xor_sync(0xffffffffu, K, stride);
              const uint32_t oq = __shfl_xor_sync(0xffffffffu, Q, stride);
              const bool asc = (lane & size) == 0 || size == 32;
              const bool low = (lane & stride) == 0;
              const bool ol = key_less(ok, oq, K, Q);
              if (low == asc ? ol : (!ol && !(ok == K && oq == Q))) { K = ok; Q = oq; }
            }
          }
          if (lane < want) mine = Q;
        } else {
          // want rounds of a warp argmin over (key, position)
          for (int r = 0; r < want; ++r) {
            double bk = INFINITY;
            uint32_t bp = 0xFFFFFFFFu;
#pragma unroll
            for (int t = 0; t < 4; ++t)
              if (key_less(kk[t], pp[t], bk, bp)) { bk = kk[t]; bp = pp[t]; }
#pragma unroll
            for (int o2 = 16; o2 > 0; o2 >>= 1) {
              const double ok = __shfl_xor_sync(0xffffffffu, bk, o2);
              const uint32_t op = __shfl_xor_sync(0xffffffffu, bp, o2);
              if (key_less(ok, op, bk, bp)) { bk = ok; bp = op; }
            }
#pragma unroll
            for (int t = 0; t < 4; ++t)
              if (pp[t] == bp) { kk[t] = INFINITY; pp[t] = 0xFFFFFFFFu; }
            if (lane == r) mine = bp;
          }
        }
        for (int s2 = 0; s2 < want; ++s2) o += __shfl_sync(0xffffffffu, mine, s2) < mine ? 1 : 0;
        sel = lane < want;
      }
      // the winners, gathered and written out in position order
      if (sel) {
        const int64_t e = oc + mine;
        const uint32_t u = (uint32_t)ldg_h(P.core.indices + e, pf);
        sth(P.eid[l] + rb + ce + o, (int64_t)e, pf);
        sth(P.row_local[l] + rb + ce + o, (int32_t)u, pf);
        if (P.val[l]) {
          const float w = wts ? __ldg(wts + e) : 1.0f;
          sth(P.val[l] + rb + ce + o, w / W, pf);
        }
        const uint32_t wd = hb_wd(P.lay, u);
        bm_or(bits + wd, hb_bt(P.lay, u), P.bm_keep, pk);
        if (use_sum) bm_or(summ + (wd >> 5), 1u << (wd & 31), P.bm_keep, pk);
      }
    }
  }
}

// ---------------------------------------------------------------------------
// rows: row() by a single-pass scan over bitmap tiles (tickets in batch order:
// ticket = batch slot * ntile + tile).  Each thread owns WPT consecutive
// bitmap words (dense) or the non-empty words under WPT summary words
// (sparse); the tile's aggregate is published for a decoupled look-back, each
// non-empty word gets the rank of its first row in its high half, and the
// rows (ascending) are staged in shared memory and written out coalesced.
// (Measured and not kept: the next hop's column side fused in here -- its
// degree loads delay every tile's look-back: 0.24 vs 0.09 + 0.085 ms.)
// ---------------------------------------------------------------------------
__global__ void ROWS_LB hop_rows_kernel(HopParams P, int l, int64_t b0, int nbg, int ntile,
                                                              Scan S) {
  __shared__ long long scr[40];
  __shared__ long long sh[2];
  __shared__ uint32_t stage[ROW_STAGE];
  if (threadIdx.x == 0) sh[0] = (long long)atomicAdd(S.ticket, 1u);
  __syncthreads();
  const long long c = sh[0];
  if (c >= (long long)nbg * ntile) return;
  const int64_t j = c / ntile;
  const int t = (int)(c - j * ntile);
  const int64_t b = b0 + j;
  uint32_t* bm = P.bm + j * P.nwp;
  int32_t* rank4 = P.rank4 + j * (P.nwp >> 2);
  const int lay = P.lay;
  const uint32_t* summ = P.summ + j * P.nsw;
  const bool sparse = P.use_sum[l];
  uint32_t wlo[WPT];
  int64_t w0 = 0;
  uint32_t sw[WPT];
  int r = 0;
  if (!sparse) {
    w0 = (int64_t)t * ROWS_TILE + (int64_t)threadIdx.x * WPT;
#pragma unroll
    for (int q = 0; q < WPT / 4; ++q) {
      const uint4 x = __ldcg((const uint4*)(bm + w0) + q);
      wlo[4 * q] = x.x;
      wlo[4 * q + 1] = x.y;
      wlo[4 * q + 2] = x.z;
      wlo[4 * q + 3] = x.w;
    }
#pragma unroll
    for (int q = 0; q < WPT; q += 4)
      if (lay) wlo[q] = 0u;  // the groups' rank words (a thread owns whole groups)
#pragma unroll
    for (int q = 0; q < WPT; ++q) r += __popc(wlo[q]);
  } else {
    w0 = ((int64_t)t * SPARSE_TILE >> 5) + (int64_t)threadIdx.x * WPT;  // first summary word
#pragma unroll
    for (int q = 0; q < WPT / 4; ++q) {
      const uint4 x = __ldcg((const uint4*)(summ + w0) + q);
      sw[4 * q] = x.x; sw[4 * q + 1] = x.y; sw[4 * q + 2] = x.z; sw[4 * q + 3] = x.w;
    }
    // the non-empty words, RL_B at a time: their loads are issued together
    // (one at a time, each popcount waited for its own load)
    for (int q = 0; q < WPT; ++q) {
      uint32_t x = sw[q];
      while (x) {
        uint32_t v[SP_B];
#pragma unroll
        for (int j = 0; j < SP_B; ++j) {
          const int bit = x ? __ffs(x) - 1 : 0;
          v[j] = (uint32_t)ldcg_if(x != 0u, (const int32_t*)bm + ((w0 + q) << 5) + bit, 0);
          x &= x - 1u;
        }
#pragma unroll
        for (int j = 0; j < SP_B; ++j) r += __popc(v[j]);
      }
    }
  }
  const long long agg = block_reduce_sum<long long>(r, scr);
  if (threadIdx.x < 32) {
    const long long ex0 = lookback(S.status + j * ntile, t, agg);
    if (threadIdx.x == 0) sh[1] = ex0;
  }
  long long tot;
  const long long ex = block_exclusive_scan<long long>(r, scr, &tot);  // syncs: sh[1] visible
  const long long tbase = sh[1];
  const int64_t rb = __ldg(P.bptr + b) * P.K[l];
  int32_t* row_map = P.row_map[l] + rb + tbase;
  const bool staged = tot <= ROW_STAGE;
  long long q0 = ex;  // rank of the thread's next row inside the tile
  int64_t last_g = -1;  // a thread's words ascend and its range holds whole groups:
                        // a group's first non-empty word starts the group's rank
  auto emit_word = [&](int64_t wi, uint32_t bits) {
    if ((wi >> 2) != last_g) {
      last_g = wi >> 2;
      if (lay) bm[last_g << 2] = (uint32_t)(tbase + q0);
      else rank4[last_g] = (int32_t)(tbase + q0);
    }
    while (bits) {
      const int bit = __ffs(bits) - 1;
      bits &= bits - 1u;
      const uint32_t u = lay ? (uint32_t)((wi >> 2) * HB_GNODES + (((wi & 3) - 1) << 5) + bit)
                             : (uint32_t)((wi << 5) + bit);
      if (staged) stage[q0] = u;
      else row_map[q0] = (int32_t)u;
      ++q0;
    }
  };
  if (!sparse) {
#pragma unroll
    for (int q = 0; q < WPT; ++q)
      if (wlo[q]) emit_word(w0 + q, wlo[q]);
  } else {
    for (int q = 0; q < WPT; ++q) {
      uint32_t x = sw[q];
      while (x) {
        uint32_t v[SP_B];
        int64_t wi[SP_B];
#pragma unroll
        for (int j = 0; j < SP_B; ++j) {
          const int bit = x ? __ffs(x) - 1 : 0;
          wi[j] = x ? ((w0 + q) << 5) + bit : -1;
          v[j] = (uint32_t)ldcg_if(x != 0u, (const int32_t*)bm + ((w0 + q) << 5) + bit, 0);
          x &= x - 1u;
        }
#pragma unroll
        for (int j = 0; j < SP_B; ++j)
          if (wi[j] >= 0) emit_word(wi[j], v[j]);
      }
    }
  }
  if (staged) {
    __syncthreads();
    for (int i = threadIdx.x; i < (int)tot; i += RW_THREADS) row_map[i] = (int32_t)stage[i];
  }
  if (t == ntile - 1 && threadIdx.x == 0) {  // the batch's row count
    long long* m = (long long*)(P.meta + (b * P.L + l) * 8);
    m[1] = tbase + tot;
  }
}

// ---------------------------------------------------------------------------
// relabel: row id -> rank in place (grid: edge tiles x batches of the group).
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(HB_THREADS, RL_MINB) hop_relabel_kernel(HopParams P, int l, int64_t b0) {
  const int64_t j = blockIdx.y;
  const int64_t b = b0 + j;
  const long long E = __ldcg((const long long*)P.meta + (b * P.L + l) * 8 + 2);
  const long long e0 = (long long)blockIdx.x * RL_TILE;
  if (e0 >= E) return;
  const uint4* bm4 = (const uint4*)(P.bm + j * P.nwp);
  const int32_t* rank4 = P.rank4 + j * (P.nwp >> 2);
  const int lay = P.lay;
  int32_t* rl = P.row_local[l] + __ldg(P.bptr + b) * P.K[l];
  uint32_t u[RL_ILP];
#pragma unroll
  for (int i = 0; i < RL_ILP; ++i) {
    const long long e = e0 + i * HB_THREADS + threadIdx.x;
    u[i] = e < E ? (uint32_t)__ldcs(rl + e) : 0u;
  }
  // rank = the group's rank word + the set bits of the group before u: one
  // 16-byte load per edge (16 bytes per 96 nodes in all)
  // (lay 0: the group's 128 nodes' bits + a separate rank load)
  if (lay) {
    uint4 w[RL_ILP];
#pragma unroll
    for (int i = 0; i < RL_ILP; ++i) {
      const long long e = e0 + i * HB_THREADS + threadIdx.x;
      w[i] = e < E ? __ldcg(bm4 + u[i] / HB_GNODES) : make_uint4(0, 0, 0, 0);
    }
#pragma unroll
    for (int i = 0; i < RL_ILP; ++i) {
      const long long e = e0 + i * HB_THREADS + threadIdx.x;
      const uint32_t o = u[i] - (u[i] / HB_GNODES) * HB_GNODES;  // offset in the group
      const int wq = (int)(o >> 5);
      const uint32_t below = (1u << (o & 31)) - 1u;
      int r = (int)w[i].x;
      r += wq > 0 ? __popc(w[i].y) : __popc(w[i].y & below);
      if (wq >= 1) r += wq > 1 ? __popc(w[i].z) : __popc(w[i].z & below);
      if (wq == 2) r += __popc(w[i].w & below);
      if (e < E) __stcs(rl + e, r);
    }
    return;
  }
  uint4 w[RL_ILP];
  int32_t g[RL_ILP];
#pragma unroll
  for (int i = 0; i < RL_ILP; ++i) {
    const long long e = e0 + i * HB_THREADS + threadIdx.x;
    w[i] = e < E ? __ldcg(bm4 + (u[i] >> 7)) : make_uint4(0, 0, 0, 0);
    g[i] = e < E ? __ldcg(rank4 + (u[i] >> 7)) : 0;
  }
#pragma unroll
  for (int i = 0; i < RL_ILP; ++i) {
    const long long e = e0 + i * HB_THREADS + threadIdx.x;
    const int wq = (int)((u[i] >> 5) & 3);
    const uint32_t below = (1u << (u[i] & 31)) - 1u;
    int r = g[i];
    r += wq > 0 ? __popc(w[i].x) : __popc(w[i].x & below);
    if (wq >= 1) r += wq > 1 ? __popc(w[i].y) : __popc(w[i].y & below);
    if (wq >= 2) r += wq > 2 ? __popc(w[i].z) : __popc(w[i].z & below);
    if (wq == 3) r += __popc(w[i].w & below);
    if (e < E) __stcs(rl + e, r);
  }
}

// clear: hop l's bitmap words back to zero.  Dense hops: grid (tiles x
// batches), every word of the tile; sparse hops: grid (row tiles x batches),
// the words of the batch's rows (row_map) and their summary words.
__global__ void __launch_bounds__(HB_THREADS) hop_clear_kernel(HopParams P, int l, int64_t b0) {
  const int64_t j = blockIdx.y;
  const int64_t b = b0 + j;
  uint32_t* bm = P.bm + j * P.nwp;
  uint32_t* summ = P.summ + j * P.nsw;
  if (!P.use_sum[l]) {
    const int64_t t0 = (int64_t)blockIdx.x * CLEAR_TILE;
    if (t0 >= P.nw) return;
    for (int q = 0; q < CLEAR_TILE / (4 * HB_THREADS); ++q) {
      const int64_t w = t0 + ((int64_t)q * HB_THREADS + threadIdx.x) * 4;
      *(uint4*)(bm + w) = make_uint4(0, 0, 0, 0);
    }
    return;
  }
  const long long R = __ldcg((const long long*)P.meta + (b * P.L + l) * 8 + 1);
  const int32_t* rows = P.row_map[l] + __ldg(P.bptr + b) * P.K[l];
  for (long long i = (long long)blockIdx.x * HB_THREADS + threadIdx.x; i < R; i += (long long)gridDim.x * HB_THREADS) {
    const uint32_t u = (uint32_t)__ldcg(rows + i);
    const uint32_t wd = hb_wd(P.lay, u);
    bm[wd] = 0u;
    summ[wd >> 5] = 0u;
  }
}

__global__ void bptr_fill_kernel(int64_t* bptr, int64_t nb, int64_t bs, int64_t num_seeds) {
  for (int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; b <= nb; b += (int64_t)gridDim.x * blockDim.x)
    bptr[b] = min(b * bs, num_seeds);
}

// ---------------------------------------------------------------------------
// Host side
// ---------------------------------------------------------------------------
static int64_t a256h(int64_t x) { return (x + 255) & ~int64_t(255); }

template <bool W, int KCAP>
static gs_status launch_select(const HopParams& P, int l, int64_t b0, int nbg, unsigned int* claim,
                               int64_t chunks_ub, cudaStream_t stream) {
  const size_t smem = sizeof(HSmem<W, KCAP>) + (W ? sizeof(HWarpA) * HS_WARPS : 0);
  auto kfn = hop_select_kernel<W, KCAP>;
  static int grid = 0;
  if (grid == 0) {
    GS_CUDA_TRY(cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0, dev = 0, sms = 148;
    GS_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kfn, HS_THREADS, smem));
    if (const char* e = getenv("GS_SEL_CTAS")) per_sm = std::min(per_sm, std::max(1, atoi(e)));
    if (const char* e = getenv("GS_SEL_CARVE"))
      GS_CUDA_TRY(cudaFuncSetAttribute(kfn, cudaFuncAttributePreferredSharedMemoryCarveout, atoi(e)));
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    grid = std::max(1, per_sm) * sms;
    if (getenv("GS_VERBOSE"))
      fprintf(stderr, "hop_select<%d,%d>: smem %zu B, %d CTAs/SM\n", (int)W, KCAP, smem, per_sm);
  }
  // small groups (hop 0, per-rank shards of a strong-scaled epoch): no more
  // CTAs than the group has chunks for -- the surplus warps otherwise walk
  // every claim queue with an atomic each and find nothing
  static int64_t cpw = -1;
  if (cpw < 0) { cpw = 1; if (const char* e = getenv("GS_SEL_CPW")) cpw = std::max(0, atoi(e)); }
  int g = grid;
  if (cpw > 0) g = (int)std::max<int64_t>(1, std::min<int64_t>(grid, (chunks_ub + cpw * HS_WARPS - 1) / (cpw * HS_WARPS)));
  kfn<<<g, HS_THREADS, smem, stream>>>(P, l, b0, nbg, claim); count_launch();
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

gs_status run_nodewise_hop(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                           const int64_t* bptr_host, int64_t batch_size, int64_t nbatch,
                           int64_t batch_base, const int32_t* fanouts, int L, int replace, int bias,
                           uint64_t key, cudaStream_t stream, gs_blocks* blk) {
  const Allocator& al = blk->al;
  HopParams P = {};
  P.core.indptr = g->indptr;
  P.core.indices = g->indices;
  P.core.weights = g->weights;
  P.core.colsum = g->colsum;
  P.core.N = g->num_nodes;
  P.core.replace = replace;
  P.core.bias = bias;
  P.core.key = key;
  P.pk = philox_keys(key);
  const bool weighted = !replace && bias != GS_W_UNIFORM;
  P.poscnt = weighted && g->weights ? g->poscnt : nullptr;
  if (weighted && g->weights && !g->poscnt)
    return fail(GS_ERR_CUDA, "weighted graph without its a0 positive-weight counts");
  P.seeds = seeds;
  P.nb = nbatch;
  P.batch_base = batch_base;
  P.L = L;
  int64_t maxbs = batch_size;
  if (bptr_host) {
    maxbs = 0;
    for (int64_t b = 0; b < nbatch; ++b) maxbs = std::max(maxbs, bptr_host[b + 1] - bptr_host[b]);
  }
  int64_t prod = 1;
  for (int l = 0; l < L; ++l) {
    P.k[l] = fanouts[l];
    prod *= fanouts[l];
    P.K[l] = prod;
  }
  // bitmap geometry: nwp words per batch slot (whole summary-mode tiles); a
  // hop is sparse (summary mode) when its slots are few against the words
  // layout 1 (rank inside each 96-node group: one load per relabelled edge)
  // for graphs whose per-batch bitmaps stay small; layout 0 (bits only, a
  // rank per 128 nodes beside them) above 2^24 nodes, where sparse row()
  // measured 5x slower in layout 1 (PP hop 2: 78 vs 14.6 ms)
  P.lay = g->num_nodes <= (int64_t(1) << 24) ? 1 : 0;
  if (const char* e = getenv("GS_HOP_LAYOUT")) P.lay = atoi(e) ? 1 : 0;
  P.nw = P.lay ? (g->num_nodes + HB_GNODES - 1) / HB_GNODES * 4 : (g->num_nodes + 31) / 32;
  P.nwp = (P.nw + SPARSE_TILE - 1) / SPARSE_TILE * SPARSE_TILE;
  P.nsw = P.nwp / 32;
  P.sel_nq = 32;
  P.sel_claim = 2;
  P.ares_split = 1;
  if (const char* e = getenv("GS_ARES_SPLIT")) P.ares_split = atoi(e);
  P.ares_tau = 0;
  if (const char* e = getenv("GS_ARES_TAU")) P.ares_tau = atoi(e);
  if (const char* e = getenv("GS_SEL_NQ")) P.sel_nq = std::max(1, std::min(32, atoi(e)));
  if (const char* e = getenv("GS_SEL_CLAIM")) P.sel_claim = std::max(1, atoi(e));
  int ntile[MAX_LAYERS];
  int64_t foot = 0;  // L2 footprint of one batch slot (bytes)
  for (int l = 0; l < L; ++l) {
    const int64_t slots = maxbs * P.K[l];
    // summary (sparse) row() only when rows are far fewer than bitmap words:
    // in the 96-node-group layout the rows of a batch touch a large share of
    // the groups, and the dense scan of an L2-resident bitmap is cheaper
    // (PD hop 0 with k = 10: 0.086 vs 0.229 ms; PP's 111 M-node layout-0
    // bitmaps keep the summary at 4 slots per word: dense 16.2 vs 1.1 ms)
    P.use_sum[l] = slots * (P.lay ? 32 : 4) < P.nw ? 1 : 0;
    if (getenv("GS_HOP_DENSE")) P.use_sum[l] = 0;
    if (getenv("GS_HOP_SPARSE")) P.use_sum[l] = 1;  // tests: the summary path at any density
    const int64_t tile = P.use_sum[l] ? SPARSE_TILE : ROWS_TILE;
    ntile[l] = (int)((P.nw + tile - 1) / tile);
    foot = std::max(foot, P.use_sum[l] ? std::min(P.nw * 5, slots * 48) + P.nsw * 4 : P.nw * (P.lay ? 4 : 5));
  }
  blk->kind = gs_blocks::NODEWISE;
  blk->num_batches = nbatch;
  blk->num_layers = L;
  blk->stream = stream;
  blk->synced = false;

  // group size: a group's bitmaps within an L2 budget, but enough batches to
  // fill the GPU (huge-N graphs: the bitmaps then live in HBM)
  int64_t budget = int64_t(128) << 20;
  if (const char* e = getenv("GS_HOP_L2MB")) budget = std::max<int64_t>(1, atoll(e)) << 20;
  int64_t WB = std::max<int64_t>(1, budget / std::max<int64_t>(foot, 1));
  int64_t minwb = 64;
  if (const char* e = getenv("GS_HOP_MINWB")) minwb = std::max<int64_t>(1, atoll(e));
  WB = std::max<int64_t>(WB, std::min<int64_t>(minwb, (int64_t(8) << 30) / std::max<int64_t>(P.nwp * 5, 1)));
  WB = std::min<int64_t>(WB, MAX_GROUP);
  WB = std::min<int64_t>(WB, std::max<int64_t>(nbatch, 1));
  const int64_t G = nbatch > 0 ? (nbatch + WB - 1) / WB : 0;
  P.bm_keep = WB * foot <= budget ? 1 : 0;
  // with the bitmaps protected (evict-last), the gathers may keep hub columns
  // in L2 for the other batches: PD 1.129 -> 1.101 ms (evict-first before)
  P.gather_normal = 1;
  if (const char* e = getenv("GS_HOP_GATHER_NORMAL")) P.gather_normal = atoi(e);
  if (const char* e = getenv("GS_HOP_BMKEEP")) P.bm_keep = atoi(e) ? 1 : 0;
  WB = G > 0 ? (nbatch + G - 1) / G : WB;  // balanced groups
  if (getenv("GS_VERBOSE"))
    fprintf(stderr, "nodewise_hop: %lld groups of %lld batches, footprint %lld KB/batch, sparse hops:%s%s%s\n",
            (long long)G, (long long)WB, (long long)(foot >> 10), P.use_sum[0] ? " 0" : "",
            L > 1 && P.use_sum[1] ? " 1" : "", L > 2 && P.use_sum[2] ? " 2" : "");

  auto need = [&](DevBuf& b, int64_t bytes) -> bool {
    return b.ensure(al, (size_t)std::max<int64_t>(bytes, 256), stream);
  };
  bool ok = need(blk->b_col[0], num_seeds * 4);
  int64_t maxcols = 0;
  int64_t nseg_max[MAX_LAYERS];
  for (int l = 0; l < L && ok; ++l) {
    const int64_t rows = num_seeds * P.K[l];
    const int64_t cols = num_seeds * (l == 0 ? 1 : P.K[l - 1]);
    maxcols = std::max(maxcols, cols);
    nseg_max[l] = (maxbs * (l == 0 ? 1 : P.K[l - 1]) + NP_SEG - 1) / NP_SEG + 1;
    ok = ok && need(blk->b_row[l], rows * 4) && need(blk->b_indptr[l], (cols + nbatch + 1) * 8) &&
         need(blk->b_rowl[l], rows * 4) && need(blk->b_eid[l], rows * 8);
    if (bias == GS_W_PASS_COLNORM) ok = ok && need(blk->b_val[l], rows * 4);
  }
  // scheduling area (zeroed per call): per (group, hop) 4 counters + the
  // look-back status words of nprep and rows; then bptr
  int64_t stat_words = 0;
  for (int l = 0; l < L; ++l) stat_words += WB * (nseg_max[l] + ntile[l]);
  const int64_t ctr_q_off = std::max<int64_t>(G * L, 1) * 4 + G * stat_words * 2;  // in uints
  const int64_t ctr_bytes = a256h(ctr_q_off * 4 + std::max<int64_t>(G * L, 1) * 8192);
  const int64_t bptr_bytes = a256h((nbatch + 1) * 8);
  ok = ok && need(blk->b_meta, nbatch * L * 8 * 8) && need(blk->b_err, 16) &&
       need(blk->b_sched, ctr_bytes + bptr_bytes);
  if (!ok) return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (blocks buffers)");
  // concurrent streams: groups alternate between the caller's stream and a
  // second one, so one group's L2-bound row() / relabel overlaps the next
  // group's HBM-bound select (each stream has its own bitmap slots)
  int NS = G > 1 ? 2 : 1;
  if (const char* e = getenv("GS_HOP_STREAMS")) NS = std::max(1, std::min(2, atoi(e)));
  if (g_profiling || getenv("GS_HOP_TIMING")) NS = 1;
  // workspace: bitmaps + summaries (kept clear between calls), column staging
  const int64_t o_bm = 0;
  const int64_t o_summ = a256h(o_bm + NS * WB * P.nwp * 4);
  const int64_t o_coff = a256h(o_summ + NS * WB * P.nsw * 4);
  const int64_t o_dcol = a256h(o_coff + (maxcols + 64) * 8);
  const int64_t o_rank = a256h(o_dcol + (maxcols + 64) * 4);  // not cleared: written before read
  const int64_t ws_bytes = a256h(o_rank + (P.lay ? 256 : NS * WB * (P.nwp / 4) * 4));
  const int64_t layout = o_coff;  // the cleared part
  const bool fresh = blk->b_ws.bytes < (size_t)ws_bytes || blk->ws_kind_prev != 15 + P.lay ||
                     blk->ws_stride_prev != layout;
  if (!blk->b_ws.ensure(al, (size_t)ws_bytes, stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (workspace)");
  if (fresh) GS_CUDA_TRY(cudaMemsetAsync(blk->b_ws.ptr, 0, (size_t)layout, stream));
  blk->ws_kind_prev = 15 + P.lay;
  blk->ws_stride_prev = layout;
  char* ws = (char*)blk->b_ws.ptr;
  P.bm = (uint32_t*)(ws + o_bm);
  P.rank4 = (int32_t*)(ws + o_rank);
  P.summ = (uint32_t*)(ws + o_summ);
  P.coff = (int64_t*)(ws + o_coff);
  P.dcol = (int32_t*)(ws + o_dcol);
  unsigned int* ctr = (unsigned int*)blk->b_sched.ptr;
  unsigned long long* stat = (unsigned long long*)((char*)blk->b_sched.ptr + std::max<int64_t>(G * L, 1) * 16);
  int64_t* bptr_dev = (int64_t*)((char*)blk->b_sched.ptr + ctr_bytes);
  P.bptr = bptr_dev;
  blk->bptr_dev = bptr_dev;
  blk->num_seeds = num_seeds;
  blk->batch_size = bptr_host ? 0 : batch_size;

  P.col0 = (int32_t*)blk->b_col[0].ptr;
  for (int l = 0; l < L; ++l) {
    P.row_map[l] = (int32_t*)blk->b_row[l].ptr;
    P.indptr_out[l] = (int64_t*)blk->b_indptr[l].ptr;
    P.row_local[l] = (int32_t*)blk->b_rowl[l].ptr;
    P.eid[l] = (int64_t*)blk->b_eid[l].ptr;
    P.val[l] = bias == GS_W_PASS_COLNORM ? (float*)blk->b_val[l].ptr : nullptr;
    gs_layer_buffers& lb = blk->layers[l];
    lb = gs_layer_buffers{};
    lb.col_map = l == 0 ? P.col0 : P.row_map[l - 1];
    lb.col_capacity = num_seeds * (l == 0 ? 1 : P.K[l - 1]);
    lb.row_map = P.row_map[l];
    lb.row_capacity = num_seeds * P.K[l];
    lb.indptr = P.indptr_out[l];
    lb.indptr_capacity = lb.col_capacity + nbatch;
    lb.row_local = P.row_local[l];
    lb.eid = P.eid[l];
    lb.val = P.val[l];
    lb.edge_capacity = num_seeds * P.K[l];
  }
  P.meta = (int64_t*)blk->b_meta.ptr;
  P.core.err = (int*)blk->b_err.ptr;
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_err.ptr, 0, 16, stream));
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_sched.ptr, 0, ctr_bytes, stream));
  if (bptr_host) {
    GS_CUDA_TRY(cudaMemcpyAsync(bptr_dev, bptr_host, (nbatch + 1) * 8, cudaMemcpyHostToDevice, stream));
  } else {
    bptr_fill_kernel<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>((nbatch + 256) / 256, 1024)), 256, 0,
                       stream>>>(bptr_dev, nbatch, batch_size, num_seeds); count_launch();
    GS_CUDA_TRY(cudaGetLastError());
  }
  if (nbatch == 0) return GS_OK;

  // profiling (gs_set_profiling / GS_HOP_TIMING): per-kernel event timing,
  // one stream, synchronises at the end of the call; kept in the result
  const bool timing = g_profiling || getenv("GS_HOP_TIMING") != nullptr;
  blk->prof.clear();
  std::vector<cudaEvent_t> ev;
  std::vector<std::string> evname;
  auto mark = [&](const char* name, int l) {
    if (!timing) return;
    cudaEvent_t e;
    cudaEventCreate(&e);
    cudaEventRecord(e, stream);
    ev.push_back(e);
    evname.push_back(std::string(name) + std::to_string(l));
  };
  mark("start", 0);
  cudaStream_t streams[2] = {stream, stream};
  if (NS > 1) {
    if (!blk->side) GS_CUDA_TRY(cudaStreamCreateWithFlags(&blk->side, cudaStreamNonBlocking));
    if (!blk->ev_fork) GS_CUDA_TRY(cudaEventCreateWithFlags(&blk->ev_fork, cudaEventDisableTiming));
    if (!blk->ev_join) GS_CUDA_TRY(cudaEventCreateWithFlags(&blk->ev_join, cudaEventDisableTiming));
    GS_CUDA_TRY(cudaEventRecord(blk->ev_fork, stream));
    GS_CUDA_TRY(cudaStreamWaitEvent(blk->side, blk->ev_fork, 0));
    streams[1] = blk->side;
  }
  const HopParams P0 = P;
  unsigned long long* st = stat;
  for (int64_t gi = 0; gi < G; ++gi) {
    const int64_t b0 = gi * WB;
    const int nbg = (int)std::min<int64_t>(WB, nbatch - b0);
    const int si = (int)(gi % NS);
    cudaStream_t stream = streams[si];
    P.bm = P0.bm + si * WB * P.nwp;
    if (!P.lay) P.rank4 = P0.rank4 + si * WB * (P.nwp / 4);
    P.summ = P0.summ + si * WB * P.nsw;
    for (int l = 0; l < L; ++l) {
      unsigned int* c4 = ctr + (gi * L + l) * 4;
      unsigned int* cq = ctr + ctr_q_off + (gi * L + l) * 2048;  // select queues, then the heavy-column counter
      const Scan snp{c4 + 0, st};
      st += WB * nseg_max[l];
      const Scan srow{c4 + 1, st};
      st += WB * ntile[l];
      {
        hop_nprep_kernel<<<(unsigned)(nbg * nseg_max[l]), NP_THREADS, 0, stream>>>(P, l, b0, nbg, snp); count_launch();
        GS_CUDA_TRY(cudaGetLastError());
        mark("nprep", l);
      }
      const int k = P.k[l];
      const int64_t cub = (int64_t)nbg * ((maxbs * (l == 0 ? 1 : P.K[l - 1]) + 31) / 32);
      gs_status rc;
      if (weighted) {
        rc = k <= 8 ? launch_select<true, 8>(P, l, b0, nbg, cq, cub, stream)
                    : (k <= SEL_W12 ? launch_select<true, 12>(P, l, b0, nbg, cq, cub, stream)
                    : (k <= 16 ? launch_select<true, 16>(P, l, b0, nbg, cq, cub, stream)
                               : launch_select<true, 32>(P, l, b0, nbg, cq, cub, stream)));
      } else {
        rc = k <= 8 ? launch_select<false, 8>(P, l, b0, nbg, cq, cub, stream)
                    : (k <= SEL_U12 ? launch_select<false, 12>(P, l, b0, nbg, cq, cub, stream)
                    : (k <= 16 ? launch_select<false, 16>(P, l, b0, nbg, cq, cub, stream)
                               : launch_select<false, 32>(P, l, b0, nbg, cq, cub, stream)));
      }
      if (rc) return rc;
      mark("select", l);
      if (weighted && P.ares_split) {
        static int grid_big = 0;
        if (grid_big == 0) {
          int per_sm = 0, dev = 0, sms = 148;
          GS_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, hop_ares_big_kernel, AB_THREADS, 0));
          cudaGetDevice(&dev);
          cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
          grid_big = std::max(1, per_sm) * sms;
          if (getenv("GS_VERBOSE")) fprintf(stderr, "hop_ares_big: %d CTAs/SM\n", per_sm);
        }
        hop_ares_big_kernel<<<grid_big, AB_THREADS, 0, stream>>>(P, l, b0, nbg, cq + 1024); count_launch();
        GS_CUDA_TRY(cudaGetLastError());
        mark("ares", l);
      }
      hop_rows_kernel<<<(unsigned)(nbg * ntile[l]), RW_THREADS, 0, stream>>>(P, l, b0, nbg, ntile[l], srow); count_launch();
      GS_CUDA_TRY(cudaGetLastError());
      mark("rows", l);
      const int64_t tiles = (maxbs * P.K[l] + RL_TILE - 1) / RL_TILE;
      hop_relabel_kernel<<<dim3((unsigned)std::max<int64_t>(tiles, 1), (unsigned)nbg), HB_THREADS, 0, stream>>>(
          P, l, b0); count_launch();
      mark("relabel", l);
      const unsigned ct = P.use_sum[l] ? (unsigned)std::max<int64_t>(1, std::min<int64_t>(tiles, 64))
                                       : (unsigned)((P.nw + CLEAR_TILE - 1) / CLEAR_TILE);
      hop_clear_kernel<<<dim3(ct, (unsigned)nbg), HB_THREADS, 0, stream>>>(P, l, b0); count_launch();
      GS_CUDA_TRY(cudaGetLastError());
      mark("clear", l);
    }
  }
  if (NS > 1) {
    GS_CUDA_TRY(cudaEventRecord(blk->ev_join, blk->side));
    GS_CUDA_TRY(cudaStreamWaitEvent(stream, blk->ev_join, 0));
  }
  if (timing) {
    cudaEventSynchronize(ev.back());
    std::vector<std::pair<std::string, float>> acc;
    for (size_t i = 1; i < ev.size(); ++i) {
      float ms = 0.f;
      cudaEventElapsedTime(&ms, ev[i - 1], ev[i]);
      bool found = false;
      for (auto& a : acc)
        if (a.first == evname[i]) { a.second += ms; found = true; }
      if (!found) acc.push_back({evname[i], ms});
    }
    float tot = 0.f;
    cudaEventElapsedTime(&tot, ev.front(), ev.back());
    for (auto& a : acc) blk->prof.push_back({"hop_" + a.first, (double)a.second});
    if (getenv("GS_HOP_TIMING")) {
      fprintf(stderr, "nodewise_hop timing (ms): total %.3f", tot);
      for (auto& a : acc) fprintf(stderr, " %s %.3f", a.first.c_str(), a.second);
      fprintf(stderr, "\n");
    }
    for (auto e : ev) cudaEventDestroy(e);
  }
  return GS_OK;
}

}  // namespace gsb
