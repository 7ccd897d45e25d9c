// nodewise_wave.cu -- node-wise ECSF sampling (GraphSAGE, KGCN, weighted
// A-Res, PASS-style A3) as ONE cooperative persistent kernel per epoch: a
// software pipeline of bulk-synchronous stages over groups of mini-batches.
//
// The super-batch is cut into groups of WB mini-batches.  Every
// hop of a group passes through three stages, one per super-step:
//   A  Extract + Select (fused): warp per 32
//      frontier columns -- indptr, Floyd / replacement / A-Res positions, the
//      gather of every sampled row at once (cp.async) into staging, and the
//      row's bit in the segment's row bitmap (fire-and-forget red.or);
//   B  row() (Finalize; R3): tiles of 8192 bitmap words count
//      their rows and store each word's in-tile prefix in its high half
//      (64-bit words: prefix | bits); the segment's last tile scans the tile
//      counts and the stage-A edge counts and publishes the block shape and
//      the next hop's frontier size;
//   C  relabel + compaction: row rank = tile prefix + word prefix + popc(bits
//      below u) (one L2 load per edge), row_map[rank] = u (the block's rows
//      ascending = the next frontier, R2), CSC indptr, COO row_local / eid.
// A rotating bitmap is cleared (Z) by the step after its last reader.  Hop l
// of group g runs stage A at super-step g + 3l, B at +1, C at +2, so a step
// mixes the HBM-bound gather stream of one group with the L2-bound scan and
// relabel of the previous ones; one grid barrier per step, no spin-waits.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <string>
#include <vector>
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "gs_internal.h"
#include "nodewise_common.cuh"

namespace cg = cooperative_groups;

namespace gsb {

constexpr int NV_THREADS = 512;
constexpr int NV_WARPS = NV_THREADS / 32;
constexpr int NV_TC = 512;        // frontier columns per tile (stages A, C)
constexpr int NV_MAXSEG = 512;    // live (stage, hop, batch) segments per super-step (<= NV_THREADS)
constexpr int NV_MAXSEG_W = 256;  // ... in the weighted (A-Res) kernel
constexpr int NV_BW = 16;         // bitmap words per thread (stage B)
constexpr int NV_BT = NV_THREADS * NV_BW;  // bitmap words per stage-B tile
constexpr int NV_BT_LOG = 13;
static_assert((1 << NV_BT_LOG) == NV_BT, "stage-B tile");
enum { ST_A = 0, ST_C = 1, ST_B = 2, ST_Z = 3 };  // claim order inside a step (longest first)
constexpr int NV_ZR = 4096;       // rows per stage-Z task

struct NVParams {
  NWCore core;
  const int32_t* seeds;
  int64_t num_seeds, batch_size, num_batches, batch_base;
  int L, WB, G, S;
  int64_t b_first;              // first batch of group 0 of this launch
  int k[MAX_LAYERS];
  int64_t K[MAX_LAYERS];
  // outputs (DESIGN.md section 5 layout)
  int32_t* col0;
  int32_t* row_map[MAX_LAYERS];
  int64_t* indptr_out[MAX_LAYERS];
  int32_t* row_local[MAX_LAYERS];
  int64_t* eid[MAX_LAYERS];
  float* val[MAX_LAYERS];
  int64_t* meta;
  long long* T;                 // [num_batches][L] frontier sizes (l > 0 written by stage B)
  unsigned int* ctr;            // [S][4 + NV_MAXSEG] work counters, zeroed per launch
  unsigned long long* bm;       // row bitmaps: (j, l, g & 3) at bm + ((g&3)*L + l)*WB + j) * nw
  uint32_t* sm;                 // summaries (hops with use_sum): bit w set iff bitmap word w is non-empty
  int64_t nsw;                  // 32-bit summary words per bitmap
  int use_sum[MAX_LAYERS];      // hop l's rows are sparse in N (B visits only non-empty words)
  int64_t nw;                   // 64-bit bitmap words per bitmap = ceil(N / 32)
  char* stg;                    // staging, per (j, l, g & 3)
  int64_t stg_off[MAX_LAYERS], stg_stride[MAX_LAYERS];
  int64_t o_u[MAX_LAYERS], o_pos[MAX_LAYERS], o_val[MAX_LAYERS];
  int64_t o_coff[MAX_LAYERS], o_cnt[MAX_LAYERS], o_tcnt[MAX_LAYERS], o_tx[MAX_LAYERS];
  int64_t o_bcnt[MAX_LAYERS], o_bx[MAX_LAYERS];
  int nbt;                      // stage-B tiles per bitmap
  unsigned long long* trace;    // optional [S][4] globaltimer stamps (GS_TRACE)
  unsigned long long* trace2;   // optional [S][4096][3] per-task (start, end, kind)
};

// Staging of one live (batch, hop, group) segment.
struct NVStage {
  int32_t* u;                // [slot] sampled row (padded slot = column * k + rank)
  uint32_t* pos;             // [slot] position inside the column
  float* val;                // [slot] PASS prob or NULL
  int64_t* coff;             // [col] indptr[v]
  int32_t* cnt;              // [col] sampled edges
  long long* tcnt;           // [tile] sampled edges of the tile (stage A)
  long long* tx;             // [tile] exclusive edge prefix (stage B)
  int32_t* bcnt;             // [bitmap tile] rows of the tile (stage B)
  int32_t* bx;               // [bitmap tile] exclusive row prefix (stage B)
  unsigned long long* bm;    // [nw] row bitmap: bits (low) | row prefix (high)
  uint32_t* sm;              // [nsw] summary of the bitmap's non-empty words
};

__device__ __forceinline__ NVStage nv_stage(const NVParams& P, int j, int l, int g) {
  const int r = g & 3;
  char* base = P.stg + P.stg_off[l] + (int64_t)(r * P.WB + j) * P.stg_stride[l];
  NVStage s;
  s.u = (int32_t*)(base + P.o_u[l]);
  s.pos = (uint32_t*)(base + P.o_pos[l]);
  s.val = P.o_val[l] >= 0 ? (float*)(base + P.o_val[l]) : nullptr;
  s.coff = (int64_t*)(base + P.o_coff[l]);
  s.cnt = (int32_t*)(base + P.o_cnt[l]);
  s.tcnt = (long long*)(base + P.o_tcnt[l]);
  s.tx = (long long*)(base + P.o_tx[l]);
  s.bcnt = (int32_t*)(base + P.o_bcnt[l]);
  s.bx = (int32_t*)(base + P.o_bx[l]);
  s.bm = P.bm + ((int64_t)(r * P.L + l) * P.WB + j) * P.nw;
  s.sm = P.sm + ((int64_t)(r * P.L + l) * P.WB + j) * P.nsw;
  return s;
}

__device__ __forceinline__ unsigned long long gtimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

struct NVSeg {
  long long b;
  int T;                    // frontier columns (< 2^25)
  int task0;                // exclusive prefix of tasks over the step's segments
  int g;
  short j;
  unsigned char l, st;
};

struct NVTileC {            // stage C's per-tile arrays
  int32_t sceo[NV_TC];
  int32_t scnt[NV_TC];
  int64_t scoff[NV_TC];
};

// Kept small: two CTAs per SM plus as much L1 as possible (the carveout is
// the smallest that fits both CTAs' shared memory).
// MAXSEG: the weighted kernel keeps 256 segments (its A-Res buffers follow in
// dynamic smem and two CTAs per SM must still fit).
template <int MAXSEG>
struct NVSmemT {
  union {
    WarpChunk wc[NV_WARPS];  // stage A
    NVTileC tc;              // stage C (tasks never overlap inside a CTA)
  };
  NVSeg seg[MAXSEG];
  long long ntasks;
  int nseg;
  long long work;
  int wtot[NV_WARPS];
  int flag;
  long long scr64[40];
  int scr32[40];
};

constexpr int NV_WCAP = 64;       // A-Res candidates per warp (expected ~2k)
constexpr int NV_CCAP = 256;      // A-Res candidates per CTA (heavy columns)
constexpr int64_t NV_DHEAVY = 2048;  // columns above this are filtered by the whole CTA

struct NVWarpA {
  uint32_t pos[NV_WCAP];
  double key[NV_WCAP];
  int rk[NV_WCAP];
  AresState st;
};

struct NVWeighted {  // weighted mode only: placed after NVSmem in dynamic shared memory
  NVWarpA a[NV_WARPS];
  uint32_t hpos[NV_CCAP];
  double hkey[NV_CCAP];
  int hrk[NV_CCAP];
  AresState hst;
  int hres, nheavy;
  int heavy[NV_TC];
};

template <class SM>
__device__ __forceinline__ int nv_find_seg(const SM& sm, long long x) {
  int lo = 0, hi = sm.nseg - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (sm.seg[mid].task0 <= x) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

__device__ __forceinline__ const int32_t* nv_frontier(const NVParams& P, long long b, int l) {
  return l == 0 ? P.seeds + b * P.batch_size : P.row_map[l - 1] + b * P.batch_size * P.K[l - 1];
}

// Stage Z tasks for a block of R rows: sparse (clear the words of NV_ZR rows
// per task, via row_map) while that is fewer tasks than a dense clear of the
// whole bitmap in stage-B tiles, else dense.
__device__ __forceinline__ long long nv_z_tasks(const NVParams& P, long long R) {
  const long long sparse = (R + NV_ZR - 1) / NV_ZR;
  return sparse > P.nbt ? (long long)P.nbt : sparse;
}

// Live segments of super-step s, stage-major in claim order (B, A, C, Z).
// All threads; ends with __syncthreads.
template <class SM>
__device__ void nv_segments(const NVParams& P, SM& sm, int s) {
  const int tid = threadIdx.x;
  long long T = 0, nt = 0, b = -1;
  int j = 0, l = 0, st = 0, g = 0;
  if (tid < 4 * P.L * P.WB) {
    j = tid % P.WB;
    l = (tid / P.WB) % P.L;
    st = tid / (P.WB * P.L);
    // stage offset inside the hop: A 0, B 1, C 2, Z 3 (clears group g's bitmaps)
    const int off = st == ST_A ? 0 : (st == ST_B ? 1 : (st == ST_C ? 2 : 3));
    g = s - 3 * l - off;
    if (g >= 0 && g < P.G) {
      b = P.b_first + (long long)g * P.WB + j;
      if (b < P.num_batches) {
        T = l == 0 ? (long long)min((int64_t)P.batch_size, (int64_t)(P.num_seeds - b * P.batch_size))
                   : __ldcg(&P.T[b * P.L + l]);
        if (st == ST_A || st == ST_C) nt = (T + NV_TC - 1) / NV_TC;
        else if (st == ST_B) nt = P.nbt;
        else nt = nv_z_tasks(P, __ldcg((const long long*)(P.meta + (b * P.L + l) * 8) + 1));
      } else {
        b = -1;
      }
    }
  }
  long long tot;
  const long long x = block_exclusive_scan<long long>(nt, sm.scr64, &tot);
  if (tid == 0) sm.ntasks = tot;
  const int live = (b >= 0) ? 1 : 0;
  int nlive;
  const int pos = block_exclusive_scan<int>(live, sm.scr32, &nlive);
  if (live) sm.seg[pos] = NVSeg{b, (int)T, (int)x, g, (short)j, (unsigned char)l, (unsigned char)st};
  if (tid == 0) sm.nseg = nlive;
  __syncthreads();
}

// ---------------------------------------------------------------------------
// Stage A: select + gather + bitmap insert for one chunk of 32 columns.
// ---------------------------------------------------------------------------
// Per lane: the chunk's column jb + lane (v, indptr[v], in-degree) into C.
__device__ __forceinline__ void nv_cols(const NVParams& P, WarpChunk& C, const NVSeg& sg, long long jb,
                                        int32_t& v_out, int64_t& d_out) {
  const int lane = threadIdx.x & 31;
  const int32_t* F = nv_frontier(P, sg.b, sg.l);
  const long long jcol = jb + lane;
  const bool active = jcol < sg.T;
  const int32_t v = active ? __ldcg(F + jcol) : -1;
  const bool valid = active && v >= 0 && (int64_t)v < P.core.N;
  if (active && !valid) atomicOr(P.core.err, ERR_SEED_RANGE);
  int64_t off = 0, d = 0;
  if (valid) {
    off = __ldg(P.core.indptr + v);
    d = __ldg(P.core.indptr + v + 1) - off;
  }
  C.vcol[lane] = v;
  C.coff[lane] = off;
  C.dcol[lane] = d;
  C.csum[lane] = 1.0f;
  v_out = v;
  d_out = d;
}

__device__ __forceinline__ float nv_tau0(const NVParams& P, int k, int32_t v, int64_t d) {
  const float W = P.core.weights ? __ldg(P.core.colsum + v) : (float)d;
  return W > 0.0f ? 2.0f * (float)k / W : -1.0f;
}

// Weighted select (A-Res, R6), phase 1 (warp): columns with d <= k take every
// eligible edge (lane per column); k < d <= NV_DHEAVY are filtered by the whole
// warp one at a time; heavier columns are queued for the CTA (phase 2).
template <class SM>
__device__ void nv_select_weighted(const NVParams& P, SM& sm, NVWeighted& W, WarpChunk& C,
                                   const NVSeg& sg) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int l = sg.l, k = P.k[l];
  const uint32_t gb = (uint32_t)(P.batch_base + sg.b);
  const int32_t v = C.vcol[lane];
  const int64_t off = C.coff[lane], d = C.dcol[lane];
  if (d > 0) C.csum[lane] = P.core.weights ? __ldg(P.core.colsum + v) : (float)d;  // PASS A3 denominator
  int cnt = 0;
  if (d <= k) {
    for (int i = 0; i < (int)d; ++i) {
      const float w = P.core.weights ? __ldg(nw_w(P.core, off + i)) : 1.0f;
      if (w > 0.0f) C.list[cnt++][lane] = (uint32_t)i;
    }
  }
  C.cnt_all[lane] = cnt;
  if (d > NV_DHEAVY) W.heavy[atomicAdd(&W.nheavy, 1)] = (warp << 5) | lane;
  NVWarpA& A = W.a[warp];
  uint32_t med = __ballot_sync(0xffffffffu, d > k && d <= NV_DHEAVY);
  while (med) {
    const int c = __ffs(med) - 1;
    med &= med - 1u;
    const int32_t vc = C.vcol[c];
    const int64_t oc = C.coff[c], dc = C.dcol[c];
    const float tau0 = dc <= 64 ? -1.0f : nv_tau0(P, k, vc, dc);
    TauSearch ts{tau0, 0.0f, 0.0f};
    int r;
    while (true) {
      if (lane == 0) A.st = AresState{0, 0};
      __syncwarp();
      ares_filter<32>(P.core, vc, oc, dc, l, gb, ts.tau, lane, A.pos, NV_WCAP, &A.st);
      __syncwarp();
      r = ares_exact(P.core, vc, oc, l, gb, k, ts.tau, A.pos, A.key, A.rk, NV_WCAP, A.st, C.list, c);
      if (r >= 0) break;
      if (!ts.next(r, tau0 > 0.0f ? tau0 : 2.0f * k / (float)dc)) {
        if (lane == 0) atomicOr(P.core.err, ERR_INTERNAL);
        r = 0;
        break;
      }
    }
    if (lane == 0) C.cnt_all[c] = r;
    __syncwarp();
  }
}

// Weighted select, phase 2 (whole CTA): the queued heavy columns one by one.
template <class SM>
__device__ void nv_select_heavy(const NVParams& P, SM& sm, NVWeighted& W, const NVSeg& sg) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int l = sg.l, k = P.k[l];
  const uint32_t gb = (uint32_t)(P.batch_base + sg.b);
  const int nh = W.nheavy;
  for (int h = 0; h < nh; ++h) {
    const int e = W.heavy[h];
    WarpChunk& C = sm.wc[e >> 5];
    const int c = e & 31;
    const int32_t v = C.vcol[c];
    const int64_t off = C.coff[c], d = C.dcol[c];
    const float tau0 = nv_tau0(P, k, v, d);
    TauSearch ts{tau0, 0.0f, 0.0f};
    while (true) {
      if (threadIdx.x == 0) W.hst = AresState{0, 0};
      __syncthreads();
      ares_filter<NV_THREADS>(P.core, v, off, d, l, gb, ts.tau, threadIdx.x, W.hpos, NV_CCAP, &W.hst);
      __syncthreads();
      if (warp == 0) {
        const int r = ares_exact(P.core, v, off, l, gb, k, ts.tau, W.hpos, W.hkey, W.hrk, NV_CCAP,
                                 W.hst, C.list, c);
        if (lane == 0) W.hres = r;
      }
      __syncthreads();
      const int r = W.hres;
      __syncthreads();
      if (r >= 0) {
        if (threadIdx.x == 0) C.cnt_all[c] = r;
        break;
      }
      if (!ts.next(r, tau0 > 0.0f ? tau0 : 2.0f * k / (float)d)) {
        if (threadIdx.x == 0) {
          atomicOr(P.core.err, ERR_INTERNAL);
          C.cnt_all[c] = 0;
        }
        break;
      }
    }
  }
  __syncthreads();
}

// Stage A, per warp after the select: stage the positions, gather every
// sampled row of the chunk at once and set the rows' bits.  Returns the
// chunk's edge count.
__device__ int nv_gather(const NVParams& P, WarpChunk& C, const NVSeg& sg, long long jb) {
  const int lane = threadIdx.x & 31;
  const int l = sg.l;
  const int k = P.k[l];
  const NVStage S = nv_stage(P, sg.j, l, sg.g);
  const uint64_t pf = pol_first(), pl = pol_last();
  const long long jcol = jb + lane;
  const int cnt = C.cnt_all[lane] & ~(1 << 30);
  int total;
  const int pre = warp_excl(cnt, &total);
  C.pre[lane] = pre;
  if (jcol < sg.T) {
    sth(S.coff + jcol, C.coff[lane], pl);
    sth(S.cnt + jcol, cnt, pl);
  }
  __syncwarp();
  chunk_map_build(C, C.cnt_all[lane] & ~(1 << 30), C.pre[lane]);
  // (a) every sampled row of the chunk is requested at once: cp.async of the
  // gathered id straight into the position's own list cell (the position is
  // read, and staged, before its cell is overwritten)
  int starts = 0;
  for (int f0 = 0; f0 < total; f0 += 32) {
    const int f = f0 + lane;
    const int c = chunk_map_col(C, f0, starts);
    if (f >= total) continue;
    const int q = f - C.pre[c];
    const uint32_t ps = (C.cnt_all[c] & (1 << 30)) ? (uint32_t)q : C.list[q][c];
    const uint32_t p = (uint32_t)((jb + c) * k + q);
    sth(S.pos + p, ps, pl);
    if (S.val) {
      const float w = P.core.weights ? __ldg(nw_w(P.core, C.coff[c] + ps)) : 1.0f;
      sth(S.val + p, w / C.csum[c], pl);
    }
    const unsigned dst = (unsigned)__cvta_generic_to_shared(&C.list[q][c]);
    asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 4, %2;" ::"r"(dst),
                 "l"(nw_idx(P.core, C.coff[c] + ps)), "l"(pf)
                 : "memory");
  }
  asm volatile("cp.async.commit_group;" ::: "memory");
  asm volatile("cp.async.wait_all;" ::: "memory");
  __syncwarp();
  // (b) stage the rows and set their bits in the segment's row bitmap
  // (fire-and-forget red.or; a row's bit is set once per warp round)
  starts = 0;
  for (int f0 = 0; f0 < total; f0 += 32) {
    const int f = f0 + lane;
    uint32_t u = 0xFFFFFFFFu;
    const int c = chunk_map_col(C, f0, starts);
    if (f < total) {
      const int q = f - C.pre[c];
      u = C.list[q][c];
      sth(S.u + (jb + c) * k + q, (int32_t)u, pl);
    }
    const uint32_t peers = __match_any_sync(0xffffffffu, u);
    if (f < total && (__ffs(peers) - 1) == lane)
      asm volatile("red.global.or.b32 [%0], %1;" ::"l"((uint32_t*)(S.bm + (u >> 5))),
                   "r"(1u << (u & 31))
                   : "memory");
    if (P.use_sum[sg.l] && f < total && (__ffs(peers) - 1) == lane)
      asm volatile("red.global.or.b32 [%0], %1;" ::"l"(S.sm + (u >> 10)), "r"(1u << ((u >> 5) & 31))
                   : "memory");
  }
  __syncwarp();
  return total;
}

// Stage A for the uniform modes: select + gather of one chunk in one pass
// (column data stay in registers).
__device__ int nv_chunk_uniform(const NVParams& P, WarpChunk& C, const NVSeg& sg, long long jb) {
  const int lane = threadIdx.x & 31;
  const int l = sg.l;
  const int k = P.k[l];
  const NVStage S = nv_stage(P, sg.j, l, sg.g);
  const uint64_t pf = pol_first(), pl = pol_last();
  const int32_t* F = nv_frontier(P, sg.b, l);
  const uint32_t gb = (uint32_t)(P.batch_base + sg.b);
  const long long jcol = jb + lane;
  const bool active = jcol < sg.T;
  const int32_t v = active ? __ldcg(F + jcol) : -1;
  const bool valid = active && v >= 0 && (int64_t)v < P.core.N;
  if (active && !valid) atomicOr(P.core.err, ERR_SEED_RANGE);
  int64_t off = 0, d = 0;
  if (valid) {
    off = __ldg(P.core.indptr + v);
    d = __ldg(P.core.indptr + v + 1) - off;
  }
  const bool weighted = false;
  int cnt = 0;
  bool all = false;
  if (P.core.replace) {  // KGCN (R10): k i.i.d. positions in slot order
    cnt = d > 0 ? k : 0;
    for (int s = 0; s < cnt; ++s) {
      const U4 r = philox((uint32_t)v, (uint32_t)s, ctr2(l, TAG_REPLACE), gb, P.core.key);
      C.list[s][lane] = (uint32_t)draw_below((uint64_t)d, r.x, r.y);
    }
  } else if (d <= k) {  // GraphSAGE, d <= k: every neighbour (R5)
    cnt = (int)d;
    all = true;
  } else {  // GraphSAGE (R5): Floyd; the list stays sorted (m is always appended)
    cnt = k;
    int n = 0;
    for (int s = 0; s < k; ++s) {
      const U4 r = philox((uint32_t)v, (uint32_t)s, ctr2(l, TAG_FLOYD), gb, P.core.key);
      const uint32_t m = (uint32_t)(d - k + s);
      const uint32_t t = (uint32_t)draw_below((uint64_t)m + 1, r.x, r.y);
      int lo = 0, hi = n;
      while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (C.list[mid][lane] < t) lo = mid + 1;
        else hi = mid;
      }
      if (lo < n && C.list[lo][lane] == t) {
        C.list[n][lane] = m;
      } else {
        for (int q = n; q > lo; --q) C.list[q][lane] = C.list[q - 1][lane];
        C.list[lo][lane] = t;
      }
      ++n;
    }
  }
  int total;
  const int pre = warp_excl(cnt, &total);
  C.coff[lane] = off;
  C.pre[lane] = pre;
  if (!weighted) C.cnt_all[lane] = cnt | (all ? (1 << 30) : 0);
  if (active) {
    sth(S.coff + jcol, off, pl);
    sth(S.cnt + jcol, cnt, pl);
  }
  __syncwarp();
  chunk_map_build(C, C.cnt_all[lane] & ~(1 << 30), C.pre[lane]);
  // (a) every sampled row of the chunk is requested at once: cp.async of the
  // gathered id straight into the position's own list cell (the position is
  // read, and staged, before its cell is overwritten)
  int starts = 0;
  for (int f0 = 0; f0 < total; f0 += 32) {
    const int f = f0 + lane;
    const int c = chunk_map_col(C, f0, starts);
    if (f >= total) continue;
    const int q = f - C.pre[c];
    const uint32_t ps = (C.cnt_all[c] & (1 << 30)) ? (uint32_t)q : C.list[q][c];
    const uint32_t p = (uint32_t)((jb + c) * k + q);
    sth(S.pos + p, ps, pl);
    if (S.val) {
      const float w = P.core.weights ? __ldg(nw_w(P.core, C.coff[c] + ps)) : 1.0f;
      sth(S.val + p, w / C.csum[c], pl);
    }
    const unsigned dst = (unsigned)__cvta_generic_to_shared(&C.list[q][c]);
    asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 4, %2;" ::"r"(dst),
                 "l"(nw_idx(P.core, C.coff[c] + ps)), "l"(pf)
                 : "memory");
  }
  asm volatile("cp.async.commit_group;" ::: "memory");
  asm volatile("cp.async.wait_all;" ::: "memory");
  __syncwarp();
  // (b) stage the rows and set their bits in the segment's row bitmap
  // (fire-and-forget red.or; a row's bit is set once per warp round)
  starts = 0;
  for (int f0 = 0; f0 < total; f0 += 32) {
    const int f = f0 + lane;
    uint32_t u = 0xFFFFFFFFu;
    const int c = chunk_map_col(C, f0, starts);
    if (f < total) {
      const int q = f - C.pre[c];
      u = C.list[q][c];
      sth(S.u + (jb + c) * k + q, (int32_t)u, pl);
    }
    const uint32_t peers = __match_any_sync(0xffffffffu, u);
    if (f < total && (__ffs(peers) - 1) == lane)
      asm volatile("red.global.or.b32 [%0], %1;" ::"l"((uint32_t*)(S.bm + (u >> 5))),
                   "r"(1u << (u & 31))
                   : "memory");
    if (P.use_sum[sg.l] && f < total && (__ffs(peers) - 1) == lane)
      asm volatile("red.global.or.b32 [%0], %1;" ::"l"(S.sm + (u >> 10)), "r"(1u << ((u >> 5) & 31))
                   : "memory");
  }
  __syncwarp();
  return total;
}

// Stage A tile: 512 columns, one 32-column chunk per warp; the tile's edge count.
template <bool WEIGHTED, class SM>
__device__ void nv_stage_a(const NVParams& P, SM& sm, const NVSeg& sg, int t) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long jb = (long long)t * NV_TC + warp * 32;
  const bool has = jb < sg.T;
  WarpChunk& C = sm.wc[warp];
  int e = 0;
  if (WEIGHTED) {
    NVWeighted& W = *reinterpret_cast<NVWeighted*>(&sm + 1);
    if (threadIdx.x == 0) W.nheavy = 0;
    __syncthreads();
    if (has) {
      int32_t v;
      int64_t d;
      nv_cols(P, C, sg, jb, v, d);
      nv_select_weighted(P, sm, W, C, sg);
    }
    __syncthreads();
    nv_select_heavy(P, sm, W, sg);
    if (has) e = nv_gather(P, C, sg, jb);
  } else if (has) {
    e = nv_chunk_uniform(P, C, sg, jb);
  }
  if (lane == 0) sm.wtot[warp] = e;
  __syncthreads();
  if (threadIdx.x == 0) {
    long long sum = 0;
    for (int w = 0; w < NV_WARPS; ++w) sum += sm.wtot[w];
    const NVStage S = nv_stage(P, sg.j, sg.l, sg.g);
    S.tcnt[t] = sum;
  }
}

// Stage B tile: NV_BW consecutive bitmap words per thread; each non-empty
// word gets its in-tile row prefix in its high half.  The segment's last tile
// scans the tile row counts (-> bx, R) and stage A's tile edge counts (-> tx,
// E) and publishes the block's shape and the next hop's frontier size.
template <class SM>
__device__ void nv_stage_b(const NVParams& P, SM& sm, const NVSeg& sg, int t,
                           unsigned int* segdone) {
  const int l = sg.l;
  const NVStage S = nv_stage(P, sg.j, l, sg.g);
  const uint64_t pl = pol_last();
  const int64_t wb = ((int64_t)t << NV_BT_LOG) + (int64_t)threadIdx.x * NV_BW;
  uint32_t bits[NV_BW];
  int c = 0;
  // summary hops: only the non-empty words are read (NV_BW = 16 bits of one summary word)
  const uint32_t smask = P.use_sum[l] ? (wb < P.nw ? (__ldcg(S.sm + (wb >> 5)) >> (wb & 31)) : 0u) : 0xFFFFu;
#pragma unroll
  for (int i = 0; i < NV_BW; ++i) {
    bits[i] = wb + i < P.nw && ((smask >> i) & 1u) ? (uint32_t)__ldcg(S.bm + wb + i) : 0u;
    c += __popc(bits[i]);
  }
  int tot;
  int run = block_exclusive_scan<int>(c, sm.scr32, &tot);
#pragma unroll
  for (int i = 0; i < NV_BW; ++i) {
    if (bits[i] == 0u) continue;  // an empty word's prefix is never read
    sth(S.bm + wb + i, ((unsigned long long)run << 32) | bits[i], pl);
    run += __popc(bits[i]);
  }
  if (threadIdx.x == 0) {
    S.bcnt[t] = tot;
    __threadfence();
    sm.flag = atomicAdd(segdone, 1u) + 1u == (unsigned int)P.nbt;
    __threadfence();
  }
  __syncthreads();
  if (!sm.flag) return;
  const long long b = sg.b;
  const int64_t bstart = b * P.batch_size;
  const int64_t colbase = l == 0 ? bstart : bstart * P.K[l - 1];
  const int64_t rbase = bstart * P.K[l];
  const int64_t ibase = colbase + b;
  long long R = 0;
  for (int i0 = 0; i0 < P.nbt; i0 += NV_THREADS) {
    const int i = i0 + threadIdx.x;
    const int cc = i < P.nbt ? __ldcg(S.bcnt + i) : 0;
    int tt;
    const int ex = block_exclusive_scan<int>(cc, sm.scr32, &tt);
    if (i < P.nbt) S.bx[i] = (int32_t)(R + ex);
    R += tt;
  }
  const int nt = (int)((sg.T + NV_TC - 1) / NV_TC);
  long long E = 0;
  for (int i0 = 0; i0 < nt; i0 += NV_THREADS) {
    const int i = i0 + threadIdx.x;
    const long long cc = i < nt ? __ldcg(S.tcnt + i) : 0;
    long long tt;
    const long long ex = block_exclusive_scan<long long>(cc, sm.scr64, &tt);
    if (i < nt) S.tx[i] = E + ex;
    E += tt;
  }
  if (threadIdx.x == 0) {
    P.indptr_out[l][ibase + sg.T] = E;
    long long* m = (long long*)(P.meta + (b * P.L + l) * 8);
    m[0] = sg.T; m[1] = R; m[2] = E; m[3] = colbase; m[4] = rbase; m[5] = ibase; m[6] = rbase;
    m[7] = 0;
    if (l + 1 < P.L) P.T[b * P.L + l + 1] = R;
  }
}

// Stage C: relabel + compaction of one tile of 512 columns.
template <class SM>
__device__ void nv_stage_c(const NVParams& P, SM& sm, const NVSeg& sg, int t) {
  const int l = sg.l, k = P.k[l];
  const NVStage S = nv_stage(P, sg.j, l, sg.g);
  const uint64_t pf = pol_first(), pl = pol_last();
  const long long b = sg.b;
  const long long c0 = (long long)t * NV_TC;
  const int ncols = (int)min((long long)NV_TC, sg.T - c0);
  const long long s0 = c0 * k;
  const int nslots = ncols * k;
  const long long xe = __ldcg(S.tx + t);
  const int64_t bstart = b * P.batch_size;
  const int64_t colbase = l == 0 ? bstart : bstart * P.K[l - 1];
  const int64_t rbase = bstart * P.K[l];
  const int64_t ibase = colbase + b;
  {  // column offsets inside the tile (ncols <= NV_THREADS)
    const int jl = threadIdx.x;
    const int c = jl < ncols ? ldh(S.cnt + c0 + jl, pl) : 0;
    int tot;
    const int ex = block_exclusive_scan<int>(c, sm.scr32, &tot);
    if (jl < ncols) {
      sm.tc.sceo[jl] = ex;
      sm.tc.scnt[jl] = c;
      sm.tc.scoff[jl] = __ldcg(S.coff + c0 + jl);
      sth(P.indptr_out[l] + ibase + c0 + jl, (int64_t)(xe + ex), pf);
      if (l == 0) sth(P.col0 + bstart + c0 + jl, __ldcg(P.seeds + bstart + c0 + jl), pf);
    }
  }
  __syncthreads();
  int32_t* row_local = P.row_local[l] + rbase;
  int32_t* row_map = P.row_map[l] + rbase;
  int64_t* eid_out = P.eid[l] + rbase;
  float* val_out = P.val[l] ? P.val[l] + rbase : nullptr;
  constexpr int NV_EM = 4;  // slots per thread in flight
  for (int r0 = threadIdx.x; r0 < nslots; r0 += NV_THREADS * NV_EM) {
    bool vv[NV_EM];
    uint32_t uu[NV_EM], ps[NV_EM];
#pragma unroll
    for (int i = 0; i < NV_EM; ++i) {
      const int r = r0 + i * NV_THREADS;
      vv[i] = false;
      if (r < nslots) {
        const int jl = r / k, q = r - jl * k;
        vv[i] = q < sm.tc.scnt[jl];
      }
      uu[i] = vv[i] ? (uint32_t)ldh(S.u + s0 + r, pl) : 0u;
      ps[i] = vv[i] ? ldh(S.pos + s0 + r, pl) : 0u;
    }
    unsigned long long wd[NV_EM];
    int32_t bx[NV_EM];
#pragma unroll
    for (int i = 0; i < NV_EM; ++i) {
      wd[i] = vv[i] ? __ldcg(S.bm + (uu[i] >> 5)) : 0ull;
      bx[i] = vv[i] ? __ldcg(S.bx + (uu[i] >> (5 + NV_BT_LOG))) : 0;
    }
#pragma unroll
    for (int i = 0; i < NV_EM; ++i) {
      if (!vv[i]) continue;
      const int r = r0 + i * NV_THREADS;
      const int jl = r / k, q = r - jl * k;
      const long long e = xe + sm.tc.sceo[jl] + q;
      const long long lid = (long long)bx[i] + (long long)(wd[i] >> 32) +
                            __popc((uint32_t)wd[i] & ((1u << (uu[i] & 31)) - 1u));
      sth(row_local + e, (int32_t)lid, pf);
      sth(row_map + lid, (int32_t)uu[i], pf);  // every slot of the row writes the same id
      sth(eid_out + e, (int64_t)(sm.tc.scoff[jl] + ps[i]), pf);
      if (val_out) sth(val_out + e, ldh(S.val + s0 + r, pl), pf);
    }
  }
}

// Stage Z: clear the bitmap of a finished group (the words of NV_ZR of its rows).
__device__ void nv_stage_z(const NVParams& P, const NVSeg& sg, int t) {
  const int l = sg.l;
  const NVStage S = nv_stage(P, sg.j, l, sg.g);
  const long long b = sg.b;
  const long long R = __ldcg((const long long*)(P.meta + (b * P.L + l) * 8) + 1);
  if ((R + NV_ZR - 1) / NV_ZR > P.nbt) {  // dense: this task's stage-B tile of words
    const int64_t wb = ((int64_t)t << NV_BT_LOG) + (int64_t)threadIdx.x * NV_BW;
#pragma unroll
    for (int i = 0; i < NV_BW; i += 2)
      if (wb + i + 1 < P.nw) *(ulonglong2*)(S.bm + wb + i) = make_ulonglong2(0ull, 0ull);
      else if (wb + i < P.nw) S.bm[wb + i] = 0ull;
    if (P.use_sum[l] && threadIdx.x < NV_BT / 32 && ((int64_t)t << (NV_BT_LOG - 5)) + threadIdx.x < P.nsw)
      S.sm[((int64_t)t << (NV_BT_LOG - 5)) + threadIdx.x] = 0u;
    return;
  }
  const int32_t* rows = P.row_map[l] + b * P.batch_size * P.K[l];
  const long long hi = min(R, (long long)(t + 1) * NV_ZR);
  for (long long i = (long long)t * NV_ZR + threadIdx.x; i < hi; i += NV_THREADS)
  {
    const uint32_t u = (uint32_t)__ldcg(rows + i);
    S.bm[u >> 5] = 0ull;
    if (P.use_sum[l]) S.sm[u >> 10] = 0u;
  }
}

// WEIGHTED: A-Res / PASS select (its own instantiation: the uniform kernel
// carries none of the weighted code, which would cost it registers / ILP).
template <bool WEIGHTED>
__global__ void __launch_bounds__(NV_THREADS, 2) nodewise_wave_kernel(NVParams P) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  using SM = NVSmemT<WEIGHTED ? NV_MAXSEG_W : NV_MAXSEG>;
  SM& sm = *reinterpret_cast<SM*>(smem_raw);
  cg::grid_group grid = cg::this_grid();
  for (int s = 0; s < P.S; ++s) {
    unsigned int* ctr = P.ctr + (int64_t)s * (4 + NV_MAXSEG);
    nv_segments(P, sm, s);
    if (P.trace && blockIdx.x == 0 && threadIdx.x == 0) P.trace[s * 4] = gtimer_ns();
    while (true) {
      if (threadIdx.x == 0) sm.work = (long long)atomicAdd(&ctr[0], 1u);
      __syncthreads();
      const long long c = sm.work;
      __syncthreads();
      if (c >= sm.ntasks) break;
      const int si = nv_find_seg(sm, c);
      const NVSeg sg = sm.seg[si];
      const int t = (int)(c - sg.task0);
      unsigned long long t_start = 0;
      if (P.trace2 && threadIdx.x == 0) t_start = gtimer_ns();
      switch (sg.st) {
        case ST_B: nv_stage_b(P, sm, sg, t, &ctr[4 + si]); break;
        case ST_A: nv_stage_a<WEIGHTED>(P, sm, sg, t); break;
        case ST_C: nv_stage_c(P, sm, sg, t); break;
        default: nv_stage_z(P, sg, t); break;
      }
      __syncthreads();
      if (P.trace2 && threadIdx.x == 0 && c < 4096) {
        unsigned long long* e = P.trace2 + ((int64_t)s * 4096 + c) * 3;
        e[0] = t_start;
        e[1] = gtimer_ns();
        e[2] = (unsigned long long)sg.st | ((unsigned long long)sg.l << 8) | ((unsigned long long)blockIdx.x << 16);
      }
    }
    if (P.trace && blockIdx.x == 0 && threadIdx.x == 0) P.trace[s * 4 + 1] = gtimer_ns();
    grid.sync();
    if (P.trace && blockIdx.x == 0 && threadIdx.x == 0) P.trace[s * 4 + 2] = P.trace[s * 4 + 3] = gtimer_ns();
  }
}

// ---------------------------------------------------------------------------
// Host side
// ---------------------------------------------------------------------------
static int64_t a256(int64_t x) { return (x + 255) & ~int64_t(255); }

gs_status run_nodewise_wave(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                            int64_t batch_size, int64_t batch_base, const int32_t* fanouts, int L,
                            int replace, int bias, uint64_t key, cudaStream_t stream,
                            gs_blocks* blk) {
  const Allocator& al = blk->al;
  NVParams P = {};
  P.core.indptr = g->indptr;
  P.core.indices = g->indices;
  P.core.weights = g->weights;
  P.core.ptab = g->ptab;
  P.core.cidx = g->cidx;
  P.core.cw = g->cw;
  P.core.cpsh = g->cpsh;
  P.core.colsum = g->colsum;
  P.core.N = g->num_nodes;
  P.core.replace = replace;
  P.core.bias = bias;
  P.core.key = key;
  P.seeds = seeds;
  P.num_seeds = num_seeds;
  P.batch_size = batch_size;
  P.num_batches = (num_seeds + batch_size - 1) / batch_size;
  P.batch_base = batch_base;
  P.L = L;
  int64_t prod = 1;
  for (int l = 0; l < L; ++l) {
    P.k[l] = fanouts[l];
    prod *= fanouts[l];
    P.K[l] = prod;
  }
  const int64_t nbatch = P.num_batches;
  P.nw = ((g->num_nodes + 31) / 32 + 1) & ~int64_t(1);  // even: 16-byte aligned bitmaps
  P.nbt = (int)((P.nw + NV_BT - 1) / NV_BT);
  // batches per group: ~16 M padded slots in the deepest hop (measured on the
  // PD-shaped GraphSAGE epoch: 64 batches of 1024 1.47 ms, 48 1.49, 32 1.54,
  // 16 2.7), <= 4 GB of bitmaps, <= NV_MAXSEG live segments
  {
    const int64_t deep = std::max<int64_t>(1, batch_size * P.K[L - 1]);
    const bool wsel = !replace && bias != GS_W_UNIFORM;  // A-Res: measured best at <= 32 (PASS PD 7.3 ms vs 8.5 at 64)
    int64_t wb = std::max<int64_t>(1, (int64_t(wsel ? 8 : 16) << 20) / deep);
    if (wsel) wb = std::min<int64_t>(wb, 32);
    wb = std::min<int64_t>(wb, std::max<int64_t>(1, (int64_t(4) << 30) / (4 * L * P.nw * 8)));
    const int maxseg = wsel ? NV_MAXSEG_W : NV_MAXSEG;
    wb = std::min<int64_t>(wb, maxseg / (4 * L));
    if (const char* e = getenv("GS_WAVE")) wb = std::max(1, std::min(atoi(e), maxseg / (4 * L)));
    wb = std::min<int64_t>(wb, std::max<int64_t>(1, nbatch));
    // (balancing the groups -- 49+48+48+48 instead of 64+64+64+1 for the PD
    // epoch -- measured 1.53 ms vs 1.51: the short last group is cheap)
    P.WB = (int)wb;
  }
  P.G = (int)((nbatch + P.WB - 1) / P.WB);
  P.S = nbatch > 0 ? P.G + 3 * L : 0;  // the last step clears the last group's bitmaps
  blk->kind = gs_blocks::NODEWISE;
  blk->bptr_dev = nullptr;
  blk->num_seeds = num_seeds;
  blk->batch_size = batch_size;
  blk->num_batches = nbatch;
  blk->num_layers = L;
  blk->stream = stream;
  blk->synced = false;

  auto need = [&](DevBuf& b, int64_t bytes) -> bool {
    return b.ensure(al, (size_t)std::max<int64_t>(bytes, 256), stream);
  };
  bool ok = need(blk->b_col[0], num_seeds * 4);
  for (int l = 0; l < L && ok; ++l) {
    const int64_t rows = num_seeds * P.K[l];
    const int64_t cols = num_seeds * (l == 0 ? 1 : P.K[l - 1]);
    ok = ok && need(blk->b_row[l], rows * 4) && need(blk->b_indptr[l], (cols + nbatch) * 8) &&
         need(blk->b_rowl[l], rows * 4) && need(blk->b_eid[l], rows * 8);
    if (bias == GS_W_PASS_COLNORM) ok = ok && need(blk->b_val[l], rows * 4);
  }
  const int64_t ctr_bytes = a256((int64_t)std::max(P.S, 1) * (4 + NV_MAXSEG) * 4);
  const int64_t t_bytes = a256(std::max<int64_t>(nbatch, 1) * L * 8);
  ok = ok && need(blk->b_meta, nbatch * L * 8 * 8) && need(blk->b_err, 16) &&
       need(blk->b_sched, ctr_bytes + t_bytes);
  if (!ok) return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (blocks buffers)");

  // workspace: 4 * L * WB row bitmaps (rotating over groups), then staging
  // hops whose rows are sparse in N keep a summary bit per bitmap word, so
  // stage B reads only the non-empty words (slots < nw/2; measured: A-Res PP
  // 197 ms vs 217 at slots < nw/8, PD GraphSAGE unchanged)
  P.nsw = (P.nw + 31) / 32;
  for (int l = 0; l < L; ++l) P.use_sum[l] = batch_size * P.K[l] * 2 < P.nw ? 1 : 0;
  const int64_t sm_off = a256((int64_t)4 * L * P.WB * P.nw * 8);
  const int64_t bm_bytes = a256(sm_off + (int64_t)4 * L * P.WB * P.nsw * 4);
  int64_t o = bm_bytes;
  for (int l = 0; l < L; ++l) {
    const int64_t slots = batch_size * P.K[l] + 64;
    const int64_t cols = batch_size * (l == 0 ? 1 : P.K[l - 1]) + 64;
    const int64_t tiles = cols / NV_TC + 2;
    int64_t q = 0;
    P.o_u[l] = q; q = a256(q + slots * 4);
    P.o_pos[l] = q; q = a256(q + slots * 4);
    if (bias == GS_W_PASS_COLNORM) { P.o_val[l] = q; q = a256(q + slots * 4); }
    else P.o_val[l] = -1;
    P.o_coff[l] = q; q = a256(q + cols * 8);
    P.o_cnt[l] = q; q = a256(q + cols * 4);
    P.o_tcnt[l] = q; q = a256(q + tiles * 8);
    P.o_tx[l] = q; q = a256(q + tiles * 8);
    P.o_bcnt[l] = q; q = a256(q + (int64_t)P.nbt * 4);
    P.o_bx[l] = q; q = a256(q + (int64_t)P.nbt * 4);
    P.stg_stride[l] = q;
    P.stg_off[l] = o - bm_bytes;
    o += q * 4 * P.WB;
  }
  const size_t ws_bytes = (size_t)o;
  const bool fresh = blk->b_ws.bytes < ws_bytes || blk->ws_kind_prev != 7 ||
                     blk->ws_stride_prev != bm_bytes;
  if (!blk->b_ws.ensure(al, ws_bytes, stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (workspace)");
  // bitmaps are left clear by every launch (stage Z); a fresh layout is cleared here
  if (fresh) GS_CUDA_TRY(cudaMemsetAsync(blk->b_ws.ptr, 0, (size_t)bm_bytes, stream));
  blk->ws_stride_prev = bm_bytes;
  blk->ws_kind_prev = 7;
  P.bm = (unsigned long long*)blk->b_ws.ptr;
  P.stg = (char*)blk->b_ws.ptr + bm_bytes;
  P.sm = (uint32_t*)((char*)blk->b_ws.ptr + sm_off);
  P.ctr = (unsigned int*)blk->b_sched.ptr;
  P.T = (long long*)((char*)blk->b_sched.ptr + ctr_bytes);

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
  if (nbatch == 0) return GS_OK;

  // dynamic shared memory: the A-Res candidate buffers only in weighted mode;
  // cooperative grid = every CTA co-resident
  const bool weighted = !replace && bias != GS_W_UNIFORM;
  const size_t smem = weighted ? sizeof(NVSmemT<NV_MAXSEG_W>) + sizeof(NVWeighted) : sizeof(NVSmemT<NV_MAXSEG>);
  static int grid_for[2] = {0, 0};
  int& grid = grid_for[weighted ? 1 : 0];
  void* kfn = weighted ? (void*)nodewise_wave_kernel<true> : (void*)nodewise_wave_kernel<false>;
  GS_CUDA_TRY(cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)smem));
  if (grid == 0) {
    int per_sm = 0, dev = 0, sms = 148;
    GS_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kfn,
                                                              NV_THREADS, smem));
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    grid = std::max(1, per_sm) * sms;
    if (getenv("GS_VERBOSE"))
      fprintf(stderr, "nodewise_wave: smem %zu B, %d CTAs/SM, grid %d\n", smem, per_sm, grid);
  }
  const char* trace_path = getenv("GS_TRACE");
  const size_t tr2 = (size_t)P.S * 4096 * 24;
  if (trace_path) {
    GS_CUDA_TRY(cudaMalloc(&P.trace, (size_t)P.S * 32));
    GS_CUDA_TRY(cudaMalloc(&P.trace2, tr2));
    GS_CUDA_TRY(cudaMemsetAsync(P.trace2, 0, tr2, stream));
  }
  void* args[] = {&P};
  GS_CUDA_TRY(cudaLaunchCooperativeKernel(kfn, dim3(grid),
                                          dim3(NV_THREADS), args, smem, stream)); count_launch();
  if (trace_path) {  // tracing aid: per-super-step timestamps
    std::vector<unsigned long long> h((size_t)P.S * 4);
    GS_CUDA_TRY(cudaStreamSynchronize(stream));
    GS_CUDA_TRY(cudaMemcpy(h.data(), P.trace, h.size() * 8, cudaMemcpyDeviceToHost));
    cudaFree(P.trace);
    std::vector<unsigned long long> h2(tr2 / 8);
    GS_CUDA_TRY(cudaMemcpy(h2.data(), P.trace2, tr2, cudaMemcpyDeviceToHost));
    cudaFree(P.trace2);
    if (FILE* f = fopen((std::string(trace_path) + ".tasks").c_str(), "wb")) {
      fwrite(h2.data(), 8, h2.size(), f);
      fclose(f);
    }
    if (FILE* f = fopen(trace_path, "a")) {
      for (int s = 0; s < P.S; ++s)
        fprintf(f, "%d %llu %llu %llu %llu\n", s, h[s * 4], h[s * 4 + 1], h[s * 4 + 2], h[s * 4 + 3]);
      fclose(f);
    }
  }
  return GS_OK;
}

}  // namespace gsb
