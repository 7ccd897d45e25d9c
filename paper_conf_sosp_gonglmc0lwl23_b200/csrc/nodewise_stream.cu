// nodewise_stream.cu -- node-wise ECSF sampling (GraphSAGE, KGCN, weighted
// A-Res, PASS-style A3) as ONE persistent software-pipelined kernel per epoch.
//
// Work is cut into tiles of 512 frontier columns of one (batch, hop).  Tiles
// are handed out by a single global ticket counter in a fixed order: step s
// holds hop l of mini-batch s - l*D for every l (deepest hop first), so a
// batch's hop l+1 is issued D steps after its hop l (software pipelining
// across the super-batch) and only ~L*D batches are live at once:
// their hash tables and slot staging (a few MB each) stay in the 126 MB L2.
// Each tile runs one fused pass (no phase barriers):
//   1. Extract + Select (Extract-Select fusion P:289):
//      Floyd / replacement / A-Res positions, gather of the sampled rows,
//      staging and an ordered-hash insert keeping every row's first slot;
//   2. wait until every EARLIER tile of the same (batch, hop) has inserted
//      (first occurrence only depends on smaller slots);
//   3. first-occurrence bitmap of its own slots + tile-local prefix counts;
//   4. decoupled look-back over the tiles of the (batch, hop) for the
//      exclusive (edges, rows) prefix;
//   5. Finalize: row id = rank of the row's first slot (the
//      first slot is in this or an earlier tile), compaction into the block
//      (CSC indptr + COO row_local/eid) and row_map (the next frontier, R2).
// The CTA completing the last tile of a hop writes the block's meta, clears
// the table and releases the next hop (or the batch) -- all on the device.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "gs_internal.h"
#include "nodewise_common.cuh"

namespace gsb {

constexpr int NS_THREADS = 512;
constexpr int NS_WARPS = NS_THREADS / 32;
constexpr int NS_COLS = NS_WARPS * 32;  // columns per tile
constexpr int NS_LAG = 8;               // steps between consecutive hops of a batch
constexpr int NS_MAXW = 512;            // bitmap words per tile (NS_COLS * MAX_FANOUT / 32)

struct NSBatch {                  // per mini-batch (device), zeroed per launch
  long long T[MAX_LAYERS];        // frontier columns of every hop
  unsigned int ready[MAX_LAYERS]; // unused (kept for layout)
  unsigned int cnt[MAX_LAYERS];   // tiles of hop l finished
  unsigned int done;              // every hop finished: the window slot is free
  unsigned int pad;
};

// A hop job: hop l of batch b, ntiles tiles, occupying tickets [start, start + nt).
struct NSJob {
  long long start;
  int b, l, nt;
  unsigned int ready;
};

struct NSParams {
  NWCore core;
  const int32_t* seeds;
  int64_t num_seeds, batch_size, num_batches, batch_base;
  int L;
  int k[MAX_LAYERS];
  int64_t K[MAX_LAYERS];
  int maxtiles[MAX_LAYERS];  // bound on the tiles of hop l (frontier bound / NS_COLS)
  int win;                   // window slots = mini-batches in flight
  int32_t* col0;
  int32_t* row_map[MAX_LAYERS];
  int64_t* indptr_out[MAX_LAYERS];
  int32_t* row_local[MAX_LAYERS];
  int64_t* eid[MAX_LAYERS];
  float* val[MAX_LAYERS];
  int64_t* meta;
  NSBatch* bs;
  unsigned long long* ticket;   // [0] head (claimed tickets), [1] tail (jobs << 40 | tickets),
                                // [2] finished batches
  NSJob* jobs;
  char* ws;
  int64_t ws_stride;
  int64_t o_u, o_pos, o_val, o_coff, o_ccnt, o_ceoff, o_bits, o_wpre, o_tab;
  int64_t o_sel, o_agg, o_rx;  // per (hop, tile) look-back state
  int64_t o_first;             // direct first-slot array [N]
  int max_tiles_all;           // max over l of maxtiles[l]
  unsigned int launch;         // per-call id (tags of the look-back state)
  unsigned long long* trace;   // optional: [tickets][8] globaltimer checkpoints (GS_TRACE)
  unsigned long long* trace2;  // optional: [tickets][4] select sub-steps of warp 0
  int log_tab_cap;
};

struct NSSlot {
  NWStage stg;
  int32_t* ceoff;
  uint32_t* bits;
  int32_t* wpre;
  uint32_t* first;          // [N] first slot of every row in the current hop (~0 = none)
  unsigned long long* sel;  // [L][maxt] = batch + 1 once the tile's inserts are done
  unsigned long long* lbs;  // [L][maxt] look-back status word
  unsigned long long* lba;  // [L][maxt] aggregate (edges, rows)
  unsigned long long* lbp;  // [L][maxt] inclusive (edges, rows)
  long long* rx;            // [L][maxt] exclusive row prefix of the tile
};

__device__ __forceinline__ NSSlot ns_slot(const NSParams& P, int64_t b) {
  char* base = P.ws + (b % P.win) * P.ws_stride;
  NSSlot s;
  s.stg.u = (int32_t*)(base + P.o_u);
  s.stg.pos = (uint32_t*)(base + P.o_pos);
  s.stg.val = P.o_val >= 0 ? (float*)(base + P.o_val) : nullptr;
  s.stg.coff = (int64_t*)(base + P.o_coff);
  s.stg.ccnt = (int32_t*)(base + P.o_ccnt);
  s.stg.tab = (unsigned long long*)(base + P.o_tab);
  s.ceoff = (int32_t*)(base + P.o_ceoff);
  s.bits = (uint32_t*)(base + P.o_bits);
  s.wpre = (int32_t*)(base + P.o_wpre);
  s.first = (uint32_t*)(base + P.o_first);
  s.sel = (unsigned long long*)(base + P.o_sel);
  s.lbs = (unsigned long long*)(base + P.o_agg);
  s.lba = s.lbs + (int64_t)P.L * P.max_tiles_all;
  s.lbp = s.lba + (int64_t)P.L * P.max_tiles_all;
  s.rx = (long long*)(base + P.o_rx);
  return s;
}

// decoupled look-back state of a tile: status word (batch + 1) << 2 | status,
// aggregate value and inclusive value (edges << 32 | rows), written before the
// status that announces them.
constexpr unsigned long long LB_A = 1, LB_P = 2;
__device__ __forceinline__ unsigned long long lb_status_word(unsigned long long tag,
                                                             unsigned long long st) {
  return (tag << 2) | st;
}
__device__ __forceinline__ unsigned long long lb_pack(int64_t e, int64_t r) {
  return ((unsigned long long)e << 32) | (unsigned long long)r;
}
__device__ __forceinline__ int64_t lb_e(unsigned long long v) { return (int64_t)(v >> 32); }
__device__ __forceinline__ int64_t lb_r(unsigned long long v) { return (int64_t)(v & 0xFFFFFFFFull); }

constexpr int NS_SLOTS = 6144;            // slots of one tile kept in shared memory
constexpr int NS_SROW = NS_SLOTS + 512;   // padded rows (odd stride) of the tile's slots

struct NSSmem {
  uint32_t su[NS_SROW];     // sampled row of tile slot q = column * ks + rank
  uint32_t spos[NS_SROW];   // position inside the column
  uint32_t sp0[NS_SROW];    // first slot (batch-hop slot id) of the slot's row
  int64_t scoff[NS_COLS];   // indptr[v] of the tile's columns
  int32_t scnt[NS_COLS];    // sampled edges per column
  int32_t sceo[NS_COLS];    // tile-local edge offset per column
  float scsum[NS_COLS];     // PASS column sums
  uint32_t sbits[NS_MAXW];  // first-occurrence bitmap of the tile's words
  int32_t swpre[NS_MAXW];   // tile-local count of first slots before each word
  int32_t spre[NS_WARPS][32];
  int wtot[NS_WARPS];
  long long x[4];
  long long job[4];
  int flag;
};

__device__ __forceinline__ unsigned int ld_acq_u32(const unsigned int* p) {
  unsigned int v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_acq_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_rel_u32(unsigned int* p, unsigned int v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_rel_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Polling with exponential backoff: spinning threads must not turn a flag's
// L2 slice into a hot spot that every other request queues behind.
struct Backoff {
  unsigned int ns = 64;
  __device__ __forceinline__ void wait() {
    __nanosleep(ns);
    ns = ns < 4096u ? ns * 2u : 4096u;
  }
};

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

struct NSSmem;
__device__ void ns_hop_done(const NSParams& P, NSSmem& sm, int64_t b, int l, int64_t T, int64_t E, int64_t R);

// Tile geometry of a hop with fanout k: rows of the shared-memory slot arrays
// have an odd stride ks (conflict-free per-lane rows), and a tile has as many
// 32-column chunks as fit NS_SLOTS slots (at most NS_COLS columns).
__device__ __forceinline__ int ns_ks(int k) { return k | 1; }
__device__ __forceinline__ int ns_tile_cols(int k) {
  const int chunks = NS_SLOTS / (ns_ks(k) * 32);
  return min(NS_COLS, max(1, chunks) * 32);
}

__device__ __forceinline__ int ns_log_cap(const NSParams& P, int64_t T, int k) {
  const int lc = log2_pow2ceil64((T * k * 4) / 3 + 64);
  return lc > P.log_tab_cap ? P.log_tab_cap : lc;
}

struct RowOut {  // A-Res output into the tile's shared-memory rows
  uint32_t* spos;
  int32_t* scnt;
  float* scsum;
  int base, ks;
  __device__ void pos(int c, int r, uint32_t v) const { spos[(base + c) * ks + r] = v; }
  __device__ void col(int c, int cnt, float cs) const {
    scnt[base + c] = cnt;
    scsum[base + c] = cs;
  }
};

// The tile: (batch b, hop l, tile t).  All threads of the CTA.
__device__ void ns_tile(const NSParams& P, NSSmem& sm, int64_t b, int l, int t, unsigned long long tk) {
  unsigned long long* trc = P.trace ? P.trace + tk * 8 : nullptr;
  if (trc && threadIdx.x == 0) { trc[0] = gtimer(); trc[7] = ((unsigned long long)b << 16) | ((unsigned long long)l << 12) | (unsigned long long)t; }
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t bstart = b * P.batch_size;
  NSBatch& B = P.bs[b];
  if (trc && threadIdx.x == 0) trc[1] = gtimer();
  // the job was appended only once its inputs were complete: no waiting here
  const int64_t T = __ldcg(&B.T[l]);
  const int k = P.k[l];
  const int ks = ns_ks(k);
  const int TC = ns_tile_cols(k);
  const int ntiles = (int)((T + TC - 1) / TC);
  const NSSlot S = ns_slot(P, b);
  const uint64_t pf = pol_first(), pl = pol_last();
  // (launch, batch) tag of the per-tile flags: stale values from earlier
  // batches in this window slot or from earlier launches never match
  const unsigned long long btag = ((unsigned long long)P.launch << 32) | (unsigned long long)(b + 1);
  const uint32_t gb = (uint32_t)(P.batch_base + b);
  const int32_t* F = l == 0 ? P.seeds + bstart : P.row_map[l - 1] + bstart * P.K[l - 1];
  const int64_t c0 = (int64_t)t * TC;                 // first column of the tile
  const int ncols = (int)min((int64_t)TC, T - c0);    // columns of this tile
  const int64_t p_base = c0 * k;                      // first batch-hop slot of the tile
  const int nslots = ncols * k;
  const int nwords = (nslots + 31) >> 5;
  const bool weighted = !P.core.replace && P.core.bias != GS_W_UNIFORM;

  // ---- 1. Extract + Select: positions into shared memory rows ----
  const int nchunks = (ncols + 31) >> 5;
  for (int ch = warp; ch < nchunks; ch += NS_WARPS) {
    const int jl = ch * 32 + lane;
    const bool active = jl < ncols;
    const int32_t v = active ? ldh(F + c0 + jl, pl) : -1;
    const bool valid = active && v >= 0 && (int64_t)v < P.core.N;
    if (active && !valid) atomicOr(P.core.err, ERR_SEED_RANGE);
    int64_t off = 0, d = 0;
    if (valid) {
      off = __ldg(P.core.indptr + v);
      d = __ldg(P.core.indptr + v + 1) - off;
    }
    uint32_t* row = &sm.spos[jl * ks];
    int cnt = 0;
    if (weighted) {
      ares_chunk_t(P.core, RowOut{sm.spos, sm.scnt, sm.scsum, ch * 32, ks}, l, gb, k, v, valid,
                   off, d);
      __syncwarp();
      cnt = active ? sm.scnt[jl] : 0;
    } else if (P.core.replace) {  // KGCN (R10): k i.i.d. positions in slot order
      cnt = d > 0 ? k : 0;
      for (int s = 0; s < cnt; ++s) {
        const U4 r = philox((uint32_t)v, (uint32_t)s, ctr2(l, TAG_REPLACE), gb, P.core.key);
        row[s] = (uint32_t)draw_below((uint64_t)d, r.x, r.y);
      }
    } else if (d <= k) {  // GraphSAGE, d <= k: every neighbour (R5)
      cnt = (int)d;
      for (int s = 0; s < cnt; ++s) row[s] = (uint32_t)s;
    } else {  // GraphSAGE (R5): Floyd, the row kept sorted (m is always appended)
      cnt = k;
      int nn = 0;
      for (int s = 0; s < k; ++s) {
        const U4 r = philox((uint32_t)v, (uint32_t)s, ctr2(l, TAG_FLOYD), gb, P.core.key);
        const uint32_t m = (uint32_t)(d - k + s);
        const uint32_t tt = (uint32_t)draw_below((uint64_t)m + 1, r.x, r.y);
        int lo = 0, hi = nn;
        while (lo < hi) {
          const int mid = (lo + hi) >> 1;
          if (row[mid] < tt) lo = mid + 1;
          else hi = mid;
        }
        if (lo < nn && row[lo] == tt) {
          row[nn] = m;
        } else {
          for (int q = nn; q > lo; --q) row[q] = row[q - 1];
          row[lo] = tt;
        }
        ++nn;
      }
    }
    if (active) {
      sm.scoff[jl] = off;
      sm.scnt[jl] = cnt;
    }
    int total;
    const int pre = warp_excl(cnt, &total);
    sm.spre[warp][lane] = pre;
    if (active) sm.sceo[jl] = pre;  // chunk-local edge offset of the column
    __syncwarp();
    // flattened gather: every sampled row of the chunk is requested at once
    // with cp.async straight into shared memory (no register cap on the
    // number of random HBM sectors in flight)
    for (int f = lane; f < total; f += 32) {
      const int c = chunk_col(sm.spre[warp], f);
      const int s = f - sm.spre[warp][c];
      const int jc = ch * 32 + c;
      const int qq = jc * ks + s;
      const int32_t* src = P.core.indices + sm.scoff[jc] + sm.spos[qq];
      const unsigned dst = (unsigned)__cvta_generic_to_shared(&sm.su[qq]);
      asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 4, %2;" ::"r"(dst),
                   "l"(src), "l"(pf)
                   : "memory");
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
    asm volatile("cp.async.wait_all;" ::: "memory");
    __syncwarp();
    // first occurrence: first[u] = min over the slots holding row u.  A
    // fire-and-forget red.min (no return, no probing); inside a warp only the
    // lowest lane (= smallest slot) of each row issues it (hub rows recur).
    for (int f = lane; f - lane < total; f += 32) {
      const bool ok = f < total;
      uint32_t u = 0xFFFFFFFFu, pslot = 0;
      if (ok) {
        const int c = chunk_col(sm.spre[warp], f);
        const int s = f - sm.spre[warp][c];
        const int jc = ch * 32 + c;
        pslot = (uint32_t)(p_base + (int64_t)jc * k + s);
        u = sm.su[jc * ks + s];
      }
      const uint32_t peers = __match_any_sync(0xffffffffu, u);
      if (ok && (__ffs(peers) - 1) == lane)
        asm volatile("red.global.min.u32 [%0], %1;" ::"l"(S.first + u), "r"(pslot) : "memory");
    }
    if (lane == 0) sm.wtot[warp] = total;
  }
  if (warp >= nchunks && lane == 0) sm.wtot[warp] = 0;  // nchunks <= NS_WARPS
  __syncthreads();
  if (warp == 0) {  // chunk edge totals -> tile-local column offsets
    const int v = lane < NS_WARPS ? sm.wtot[lane] : 0;
    int tot;
    const int ex = warp_excl(v, &tot);
    if (lane < NS_WARPS) sm.wtot[lane] = ex;
    if (lane == 0) sm.x[2] = tot;  // tile edges
  }
  __syncthreads();
  for (int jl = threadIdx.x; jl < ncols; jl += blockDim.x) sm.sceo[jl] += sm.wtot[jl >> 5];
  const int maxt = P.max_tiles_all;
  unsigned long long* sel = S.sel + (int64_t)l * maxt;
  unsigned long long* lbs = S.lbs + (int64_t)l * maxt;
  unsigned long long* lba = S.lba + (int64_t)l * maxt;
  unsigned long long* lbp = S.lbp + (int64_t)l * maxt;
  long long* rx = S.rx + (int64_t)l * maxt;
  if (threadIdx.x == 0) {
    __threadfence();
    st_rel_u64(&sel[t], btag);
    if (trc) trc[2] = gtimer();
  }
  // ---- 2. wait for the inserts of every earlier tile ----
  if (threadIdx.x == 0) {  // newest first: when t-1 is done, older ones usually are
    for (int t0 = t - 1; t0 >= 0; --t0) {
      Backoff bo;
      while (ld_acq_u64(&sel[t0]) != btag) bo.wait();
    }
  }
  __syncthreads();
  if (trc && threadIdx.x == 0) trc[3] = gtimer();
  // ---- 3. first-occurrence bitmap of this tile's slots (word-major) ----
  // every first[u] lookup of the warp's words is issued at once (<= 12 per lane)
  constexpr int NS_WPW = NS_SLOTS / 32 / NS_WARPS;  // words per warp, upper bound
  const int wpw = (nwords + NS_WARPS - 1) / NS_WARPS;
  const int wa = warp * wpw, wz = min(nwords, wa + wpw);
  uint32_t p0r[NS_WPW];
  bool vr[NS_WPW];
#pragma unroll
  for (int i = 0; i < NS_WPW; ++i) {
    const int r = (wa + i) * 32 + lane;
    vr[i] = false;
    p0r[i] = 0u;
    if (wa + i < wz && r < nslots) {
      const int jl = r / k, s = r - jl * k;
      if (s < sm.scnt[jl]) {
        vr[i] = true;
        p0r[i] = ldh(S.first + sm.su[jl * ks + s], pl);
      }
    }
  }
  int wrun = 0;
#pragma unroll
  for (int i = 0; i < NS_WPW; ++i) {
    const int wl = wa + i;
    const int r = wl * 32 + lane;
    const int64_t p = p_base + r;
    bool first = false;
    if (vr[i]) {
      const int jl = r / k, s = r - jl * k;
      sm.sp0[jl * ks + s] = p0r[i];
      if (p0r[i] > (uint32_t)p) atomicOr(P.core.err, ERR_INTERNAL);
      first = p0r[i] == (uint32_t)p;
    }
    const uint32_t word = __ballot_sync(0xffffffffu, first);
    if (wl < wz) {
      if (lane == 0) {
        sm.sbits[wl] = word;
        sm.swpre[wl] = __popc(word);
        sth(S.bits + (p_base >> 5) + wl, word, pl);
      }
      wrun += __popc(word);
    }
  }
  if (lane == 0) sm.wtot[warp] = wrun;
  __syncthreads();
  if (warp == 0) {
    const int v = lane < NS_WARPS ? sm.wtot[lane] : 0;
    int tot;
    const int ex = warp_excl(v, &tot);
    if (lane < NS_WARPS) sm.wtot[lane] = ex;
    if (lane == 0) sm.x[3] = tot;  // tile rows (first occurrences)
  }
  __syncthreads();
  {  // per-word tile-local prefix (shared + global for later tiles)
    int run = sm.wtot[warp];
    for (int i0 = wa; i0 < wz; i0 += 32) {
      const int i = i0 + lane;
      const int c = i < wz ? sm.swpre[i] : 0;
      int tot;
      const int ex = warp_excl(c, &tot);
      if (i < wz) {
        sm.swpre[i] = run + ex;
        sth(S.wpre + (p_base >> 5) + i, run + ex, pl);
      }
      run += tot;
    }
  }
  // ---- 4. decoupled look-back over the hop's tiles ----
  if (threadIdx.x == 0) {
    if (trc) trc[4] = gtimer();
    const int64_t te = sm.x[2], tr = sm.x[3];
    __threadfence();
    int64_t xe = 0, xr = 0;
    if (t > 0) {
      lba[t] = lb_pack(te, tr);
      __threadfence();
      st_rel_u64(&lbs[t], lb_status_word(btag, LB_A));
      Backoff bo;
      for (int t0 = t - 1; t0 >= 0;) {
        const unsigned long long w = ld_acq_u64(&lbs[t0]);
        if (w == lb_status_word(btag, LB_P)) {
          const unsigned long long v = __ldcg(&lbp[t0]);
          xe += lb_e(v);
          xr += lb_r(v);
          break;
        }
        if (w == lb_status_word(btag, LB_A)) {
          const unsigned long long v = __ldcg(&lba[t0]);
          xe += lb_e(v);
          xr += lb_r(v);
          --t0;
          continue;
        }
        bo.wait();
      }
    }
    rx[t] = xr;
    lbp[t] = lb_pack(xe + te, xr + tr);
    __threadfence();
    st_rel_u64(&lbs[t], lb_status_word(btag, LB_P));
    sm.x[0] = xe;
    sm.x[1] = xr;
    if (trc) trc[5] = gtimer();
  }
  __syncthreads();
  // ---- 5. relabel + compaction (word-major over the tile's slots) ----
  {
    const int64_t xe = sm.x[0], xr = sm.x[1];
    const int64_t colbase = l == 0 ? bstart : bstart * P.K[l - 1];
    const int64_t rbase = bstart * P.K[l];
    const int64_t ibase = colbase + b;
    int32_t* row_map = P.row_map[l] + rbase;
    int32_t* row_local = P.row_local[l] + rbase;
    int64_t* eid_out = P.eid[l] + rbase;
    float* val_out = P.val[l] ? P.val[l] + rbase : nullptr;
    const int tile_slots = TC * k;
    for (int jl = threadIdx.x; jl < ncols; jl += blockDim.x) {
      sth(P.indptr_out[l] + ibase + c0 + jl, (int64_t)(xe + sm.sceo[jl]), pf);
      if (l == 0) sth(P.col0 + bstart + c0 + jl, __ldcg(P.seeds + bstart + c0 + jl), pf);
    }
    for (int r = threadIdx.x; r < nslots; r += blockDim.x) {
      const int jl = r / k, s = r - jl * k;
      if (s >= sm.scnt[jl]) continue;
      const int q = jl * ks + s;
      const int64_t p = p_base + r;
      const uint32_t p0 = sm.sp0[q];
      const int64_t e = xe + sm.sceo[jl] + s;
      const int64_t eid = sm.scoff[jl] + sm.spos[q];
      int64_t lid;
      if ((int64_t)p0 >= p_base) {
        const int wl = (int)((p0 - p_base) >> 5);
        lid = xr + sm.swpre[wl] + __popc(sm.sbits[wl] & ((1u << (p0 & 31)) - 1u));
      } else {  // first occurrence in an earlier tile: wait for its prefix
        const int t0 = (int)(p0 / (uint32_t)tile_slots);
        Backoff bo;
        while (ld_acq_u64(&lbs[t0]) != lb_status_word(btag, LB_P)) bo.wait();
        const int64_t wd = p0 >> 5;
        lid = __ldcg(rx + t0) + ldh(S.wpre + wd, pl) +
              __popc(ldh(S.bits + wd, pl) & ((1u << (p0 & 31)) - 1u));
      }
      sth(row_local + e, (int32_t)lid, pf);
      sth(eid_out + e, eid, pf);
      if (val_out) {
        const float w = P.core.weights ? __ldg(P.core.weights + eid) : 1.0f;
        sth(val_out + e, w / sm.scsum[jl], pf);
      }
      if ((int64_t)p0 == p) sth(row_map + lid, (int32_t)sm.su[q], pf);
    }
  }
  // ---- 6. completion of the hop ----
  __syncthreads();
  if (trc && threadIdx.x == 0) trc[6] = gtimer();
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned int d = atomicAdd(&B.cnt[l], 1u) + 1u;
    sm.flag = (d == (unsigned int)ntiles);
    if (sm.flag) {
      __threadfence();
      const int64_t i = (int64_t)l * P.max_tiles_all + ntiles - 1;
      Backoff bo;
      while (ld_acq_u64(&S.lbs[i]) != lb_status_word(btag, LB_P)) bo.wait();
      const unsigned long long v = __ldcg(&S.lbp[i]);
      sm.x[2] = lb_e(v);
      sm.x[3] = lb_r(v);
    }
  }
  __syncthreads();
  if (sm.flag) ns_hop_done(P, sm, b, l, T, sm.x[2], sm.x[3]);
}

// Appends hop job (b, l) with nt tiles (thread 0).
__device__ void ns_append(const NSParams& P, int64_t b, int l, int nt) {
  const unsigned long long old = atomicAdd(P.ticket + 1, (1ull << 40) | (unsigned long long)nt);
  const int64_t j = (int64_t)(old >> 40);
  NSJob& J = P.jobs[j];
  J.start = (long long)(old & ((1ull << 40) - 1));
  J.b = (int)b;
  J.l = l;
  J.nt = nt;
  __threadfence();
  st_rel_u32(&J.ready, 1u);
}

// Makes hop l of batch b (T columns) runnable, finishing empty hops on the spot.
__device__ void ns_start_hop(const NSParams& P, NSSmem& sm, int64_t b, int l, int64_t T);

// Hop l of batch b is complete (CTA-wide): write the block's meta, scrub the
// scratch (clear the table, discard dead staging lines from L2 without
// write-back) and release the next hop or the next batch of the window slot.
__device__ void ns_hop_done(const NSParams& P, NSSmem& sm, int64_t b, int l, int64_t T,
                            int64_t E, int64_t R) {
  const NSSlot S = ns_slot(P, b);
  const int k = P.k[l];
  const uint64_t pl = pol_last();
  // reset first[u] of exactly the rows this hop touched (its row_map), so the
  // array is all ~0 for the next hop / the next batch of this window slot
  if (R > 0) {
    const int32_t* rows = P.row_map[l] + b * P.batch_size * P.K[l];
    for (int64_t i = threadIdx.x; i < R; i += blockDim.x)
      sth(S.first + __ldcg(rows + i), 0xFFFFFFFFu, pl);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    const int64_t bstart = b * P.batch_size;
    const int64_t colbase = l == 0 ? bstart : bstart * P.K[l - 1];
    const int64_t rbase = bstart * P.K[l];
    const int64_t ibase = colbase + b;
    P.indptr_out[l][ibase + T] = E;
    long long* m = (long long*)(P.meta + (b * P.L + l) * 8);
    m[0] = T; m[1] = R; m[2] = E; m[3] = colbase; m[4] = rbase; m[5] = ibase; m[6] = rbase;
    m[7] = 0;
    __threadfence();
  }
  if (l + 1 < P.L) {
    ns_start_hop(P, sm, b, l + 1, R);
  } else {
    if (threadIdx.x == 0) {
      st_rel_u32(&P.bs[b].done, 1u);
      atomicAdd((unsigned int*)(P.ticket + 2), 1u);
    }
    const int64_t nb = b + P.win;  // the window slot is free: admit the next batch
    if (nb < P.num_batches)
      ns_start_hop(P, sm, nb, 0, min(P.batch_size, P.num_seeds - nb * P.batch_size));
  }
}

__device__ void ns_start_hop(const NSParams& P, NSSmem& sm, int64_t b, int l, int64_t T) {
  const int nt = (int)((T + ns_tile_cols(P.k[l]) - 1) / ns_tile_cols(P.k[l]));
  if (threadIdx.x == 0) {
    P.bs[b].T[l] = T;
    __threadfence();
    if (nt > 0) ns_append(P, b, l, nt);
  }
  __syncthreads();
  if (nt == 0) {  // empty frontier: the hop (and every later one) is empty
    if (threadIdx.x == 0) {
      const int64_t bstart = b * P.batch_size;
      const int64_t colbase = l == 0 ? bstart : bstart * P.K[l - 1];
      const int64_t ibase = colbase + b;
      P.indptr_out[l][ibase] = 0;
    }
    ns_hop_done(P, sm, b, l, 0, 0, 0);
  }
}

__global__ void stream_admit_kernel(NSParams P) {
  // admit the first window of batches (hop 0 of batch b has min(bs, rest) columns)
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  const int64_t n = min((int64_t)P.win, P.num_batches);
  for (int64_t b = 0; b < n; ++b) {
    const int64_t T = min(P.batch_size, P.num_seeds - b * P.batch_size);
    P.bs[b].T[0] = T;
    ns_append(P, b, 0, (int)((T + ns_tile_cols(P.k[0]) - 1) / ns_tile_cols(P.k[0])));
  }
}

__global__ void __launch_bounds__(NS_THREADS, 2) nodewise_stream_kernel(NSParams P) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  NSSmem& sm = *reinterpret_cast<NSSmem*>(smem_raw);
  int64_t hint = 0;  // job index cursor (this CTA's tickets only increase)
  while (true) {
    if (threadIdx.x == 0) {
      const unsigned long long t = atomicAdd(P.ticket, 1ull);
      long long kind = 0;  // 0 exit, 1 work
      Backoff bo;
      while (true) {
        const unsigned long long tail = ld_acq_u64(P.ticket + 1);
        if (t < (tail & ((1ull << 40) - 1))) {
          kind = 1;
          break;
        }
        if ((int64_t)ld_acq_u32((const unsigned int*)(P.ticket + 2)) >= P.num_batches) break;
        bo.wait();
      }
      if (kind) {
        while (true) {
          NSJob& J = P.jobs[hint];
          Backoff bj;
          while (ld_acq_u32(&J.ready) == 0u) bj.wait();
          if ((long long)t < J.start + J.nt) break;
          ++hint;
        }
        const NSJob& J = P.jobs[hint];
        sm.job[1] = J.b;
        sm.job[2] = J.l;
        sm.job[3] = (long long)t - J.start;
      }
      sm.job[0] = kind;
      sm.job[0] |= (long long)t << 1;
    }
    __syncthreads();
    const long long w0 = sm.job[0], b = sm.job[1], l = sm.job[2], t = sm.job[3];
    __syncthreads();
    if ((w0 & 1) == 0) break;
    ns_tile(P, sm, b, (int)l, (int)t, (unsigned long long)(w0 >> 1));
  }
}

// ---------------------------------------------------------------------------
// Host side
// ---------------------------------------------------------------------------
static int64_t align256(int64_t x) { return (x + 255) & ~int64_t(255); }

gs_status run_nodewise_stream(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                              int64_t batch_size, int64_t batch_base, const int32_t* fanouts,
                              int L, int replace, int bias, uint64_t key, cudaStream_t stream,
                              gs_blocks* blk) {
  const Allocator& al = blk->al;
  NSParams P = {};
  P.core.indptr = g->indptr;
  P.core.indices = g->indices;
  P.core.weights = g->weights;
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
  int64_t prod = 1, slot_cap = 64, col_cap = 64;
  int max_t = 1;
  for (int l = 0; l < L; ++l) {
    P.k[l] = fanouts[l];
    const int64_t cols = batch_size * prod;  // bound on the hop's frontier
    col_cap = std::max(col_cap, cols);
    const int ks = fanouts[l] | 1;  // = ns_tile_cols() on the device
    const int tcols = std::min(NS_COLS, std::max(1, NS_SLOTS / (ks * 32)) * 32);
    P.maxtiles[l] = (int)((cols + tcols - 1) / tcols);
    max_t = std::max(max_t, P.maxtiles[l]);
    prod *= fanouts[l];
    P.K[l] = prod;
    slot_cap = std::max(slot_cap, cols * fanouts[l]);
  }
  P.max_tiles_all = max_t;
  {
    const char* w = getenv("GS_WINDOW");
    P.win = w ? std::max(1, atoi(w)) : 48;  // mini-batches in flight
  }
  const int64_t nbatch = P.num_batches;
  int64_t tiles_bound = 0;
  for (int l = 0; l < L; ++l) tiles_bound += P.maxtiles[l];
  tiles_bound *= std::max<int64_t>(nbatch, 1);
  col_cap += NS_COLS;
  slot_cap += (int64_t)NS_COLS * MAX_FANOUT;
  blk->kind = gs_blocks::NODEWISE;
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
  const int64_t jobs_off = align256(nbatch * (int64_t)sizeof(NSBatch) + 64);
  const int64_t sched_bytes = jobs_off + (nbatch * L + 16) * (int64_t)sizeof(NSJob);
  ok = ok && need(blk->b_meta, nbatch * L * 8 * 8) && need(blk->b_err, 16) &&
       need(blk->b_ctr, 8 * (MAX_LAYERS + 2)) && need(blk->b_sched, sched_bytes);
  if (!ok) return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (blocks buffers)");

  int log_tab = 6;
  while ((int64_t(1) << log_tab) < (slot_cap * 4) / 3 + 64) ++log_tab;
  const int64_t words = (slot_cap + 31) / 32 + 64;
  int64_t o = 0;
  P.o_u = o; o = align256(o + slot_cap * 4);
  P.o_pos = o; o = align256(o + slot_cap * 4);
  if (bias == GS_W_PASS_COLNORM) {
    P.o_val = o;
    o = align256(o + slot_cap * 4);
  } else {
    P.o_val = -1;
  }
  P.o_coff = o; o = align256(o + col_cap * 8);
  P.o_ccnt = o; o = align256(o + col_cap * 4);
  P.o_ceoff = o; o = align256(o + col_cap * 4);
  P.o_bits = o; o = align256(o + words * 4);
  P.o_wpre = o; o = align256(o + words * 4);
  P.o_sel = o; o = align256(o + (int64_t)L * max_t * 8);
  P.o_agg = o; o = align256(o + (int64_t)3 * L * max_t * 8);
  P.o_rx = o; o = align256(o + (int64_t)L * max_t * 8);
  P.o_tab = o; o = align256(o + 256);  // (hash table unused: direct first[] array)
  P.o_first = o; o = align256(o + g->num_nodes * 4);
  P.ws_stride = o;
  P.log_tab_cap = log_tab;
  const size_t ws_bytes = (size_t)P.ws_stride * P.win;
  const bool fresh = blk->b_ws.bytes < ws_bytes || blk->ws_stride_prev != P.ws_stride ||
                     blk->ws_kind_prev != 4;
  if (!blk->b_ws.ensure(al, ws_bytes, stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (workspace)");
  if (fresh)  // empty tables (~0) and no stale look-back state
    GS_CUDA_TRY(cudaMemsetAsync(blk->b_ws.ptr, 0xFF, blk->b_ws.bytes, stream));
  blk->ws_stride_prev = P.ws_stride;
  blk->ws_kind_prev = 4;
  P.ws = (char*)blk->b_ws.ptr;
  P.launch = (++blk->launch_id) & 0x3FFFFFFFu;
  P.bs = (NSBatch*)blk->b_sched.ptr;
  P.ticket = (unsigned long long*)((char*)blk->b_sched.ptr + nbatch * sizeof(NSBatch));
  P.jobs = (NSJob*)((char*)blk->b_sched.ptr + jobs_off);

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
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_sched.ptr, 0, sched_bytes, stream));
  if (nbatch == 0) return GS_OK;

  static int grid = 0;
  if (grid == 0) {
    GS_CUDA_TRY(cudaFuncSetAttribute(nodewise_stream_kernel,
                                     cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)sizeof(NSSmem)));
    int per_sm = 0, dev = 0, sms = 148;
    GS_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, nodewise_stream_kernel,
                                                              NS_THREADS, sizeof(NSSmem)));
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    grid = std::max(1, per_sm) * sms;  // every CTA co-resident: waits only point backwards
  }
  const char* trace_path = getenv("GS_TRACE");
  unsigned long long* dtrace = nullptr;
  const size_t ntk = (size_t)tiles_bound + 1024;
  if (trace_path) {
    GS_CUDA_TRY(cudaMalloc(&dtrace, ntk * 96));
    GS_CUDA_TRY(cudaMemsetAsync(dtrace, 0, ntk * 96, stream));
    P.trace = dtrace;
    P.trace2 = dtrace + ntk * 8;
  }
  stream_admit_kernel<<<1, 32, 0, stream>>>(P);
  nodewise_stream_kernel<<<grid, NS_THREADS, sizeof(NSSmem), stream>>>(P);
  GS_CUDA_TRY(cudaGetLastError());
  if (trace_path) {  // tracing aid: per-tile timestamps to a binary file
    std::vector<unsigned long long> h(ntk * 12);
    GS_CUDA_TRY(cudaStreamSynchronize(stream));
    GS_CUDA_TRY(cudaMemcpy(h.data(), dtrace, ntk * 96, cudaMemcpyDeviceToHost));
    cudaFree(dtrace);
    if (FILE* f = fopen(trace_path, "wb")) {
      fwrite(h.data(), 8, h.size(), f);
      fclose(f);
    }
  }
  return GS_OK;
}

}  // namespace gsb
