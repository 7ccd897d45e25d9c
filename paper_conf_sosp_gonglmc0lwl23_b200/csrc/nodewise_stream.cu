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
  unsigned int ready[MAX_LAYERS]; // hop l may start (T[l] valid, table clear)
  unsigned int cnt[MAX_LAYERS];   // tiles of hop l finished (including empty ones)
  unsigned int done;              // every hop finished: the window slot is free
  unsigned int pad;
};

struct NSParams {
  NWCore core;
  const int32_t* seeds;
  int64_t num_seeds, batch_size, num_batches, batch_base;
  int L;
  int k[MAX_LAYERS];
  int64_t K[MAX_LAYERS];
  int maxtiles[MAX_LAYERS];  // tile budget of hop l (bound on its frontier / NS_COLS)
  int tile_off[MAX_LAYERS];  // position of hop l's tiles inside a step (deepest first)
  int tps;                   // tickets per step
  int64_t nsteps;
  int win;                   // window slots (> (L-1) * NS_LAG)
  int32_t* col0;
  int32_t* row_map[MAX_LAYERS];
  int64_t* indptr_out[MAX_LAYERS];
  int32_t* row_local[MAX_LAYERS];
  int64_t* eid[MAX_LAYERS];
  float* val[MAX_LAYERS];
  int64_t* meta;
  NSBatch* bs;
  unsigned long long* ticket;
  char* ws;
  int64_t ws_stride;
  int64_t o_u, o_pos, o_val, o_coff, o_ccnt, o_ceoff, o_bits, o_wpre, o_tab;
  int64_t o_sel, o_agg, o_rx;  // per (hop, tile) look-back state
  int max_tiles_all;           // max over l of maxtiles[l]
  unsigned int launch;         // per-call id (tags of the look-back state)
  int log_tab_cap;
};

struct NSSlot {
  NWStage stg;
  int32_t* ceoff;
  uint32_t* bits;
  int32_t* wpre;
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

struct NSSmem {
  WarpChunk wc[NS_WARPS];
  int wtot[NS_WARPS];
  int wcnt[NS_MAXW];
  long long x[4];   // exclusive edges / rows of this tile, totals
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

__device__ __forceinline__ int ns_log_cap(const NSParams& P, int64_t T, int k) {
  const int lc = log2_pow2ceil64((T * k * 4) / 3 + 64);
  return lc > P.log_tab_cap ? P.log_tab_cap : lc;
}

// The tile: (batch b, hop l, tile t).  All threads of the CTA.
__device__ void ns_tile(const NSParams& P, NSSmem& sm, int64_t b, int l, int t) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t bstart = b * P.batch_size;
  NSBatch& B = P.bs[b];
  // ---- 0. wait for the inputs of this hop ----
  if (threadIdx.x == 0) {
    if (l == 0) {
      if (b >= P.win) {  // the window slot must be free
        while (ld_acq_u32(&P.bs[b - P.win].done) == 0u) __nanosleep(64);
      }
    } else {
      while (ld_acq_u32(&B.ready[l]) == 0u) __nanosleep(64);
    }
  }
  __syncthreads();
  const int64_t T = l == 0 ? min(P.batch_size, P.num_seeds - bstart) : __ldcg(&B.T[l]);
  const int k = P.k[l];
  const int ntiles = (int)((T + NS_COLS - 1) / NS_COLS);
  const NSSlot S = ns_slot(P, b);
  const int log_cap = ns_log_cap(P, T, k);
  const uint32_t tag = 0u;  // tables are cleared after every hop
  // (launch, batch) tag of the per-tile flags: stale values from earlier
  // batches in this window slot or from earlier launches never match
  const unsigned long long btag = ((unsigned long long)P.launch << 32) | (unsigned long long)(b + 1);
  if (t < ntiles) {
    const uint32_t gb = (uint32_t)(P.batch_base + b);
    const int32_t* F = l == 0 ? P.seeds + bstart : P.row_map[l - 1] + bstart * P.K[l - 1];
    const int64_t tend = min(T, (int64_t)(t + 1) * NS_COLS);
    const int64_t jb = (int64_t)t * NS_COLS + warp * 32;
    // ---- 1. Extract + Select + stage + insert ----
    int e = 0, pre = 0;
    if (jb < tend) {
      e = select_chunk<true>(P.core, S.stg, sm.wc[warp], l, k, log_cap, tag, F, jb, tend, gb);
      pre = sm.wc[warp].pre[lane];
    }
    if (lane == 0) sm.wtot[warp] = e;
    __syncthreads();
    if (warp == 0) {
      const int v = lane < NS_WARPS ? sm.wtot[lane] : 0;
      int tot;
      const int ex = warp_excl(v, &tot);
      if (lane < NS_WARPS) sm.wtot[lane] = ex;
      if (lane == 0) sm.x[2] = tot;  // tile edges
    }
    __syncthreads();
    if (jb + lane < tend) S.ceoff[jb + lane] = sm.wtot[warp] + pre;
    __syncthreads();
    const int maxt = P.max_tiles_all;
    unsigned long long* sel = S.sel + (int64_t)l * maxt;
    unsigned long long* lbs = S.lbs + (int64_t)l * maxt;
    unsigned long long* lba = S.lba + (int64_t)l * maxt;
    unsigned long long* lbp = S.lbp + (int64_t)l * maxt;
    long long* rx = S.rx + (int64_t)l * maxt;
    if (threadIdx.x == 0) {
      __threadfence();
      st_rel_u64(&sel[t], btag);
    }
    // ---- 2. wait for the inserts of every earlier tile ----
    if (warp == 0) {
      for (int t0 = lane; t0 < t; t0 += 32)
        while (ld_acq_u64(&sel[t0]) != btag) __nanosleep(32);
      __syncwarp();
    }
    __syncthreads();
    // ---- 3. first-occurrence bitmap of this tile's slots ----
    const int64_t PT = T * k;
    const int64_t wbase = ((int64_t)t * NS_COLS * k) >> 5;   // first word of the tile
    const int64_t wend = min((PT + 31) >> 5, wbase + (int64_t)NS_COLS * k / 32);
    const int wpw = k;                                        // words per warp
    const int64_t w0 = wbase + (int64_t)warp * wpw;
    int wrun = 0;
    for (int i0 = 0; i0 < wpw; i0 += NW_ILP) {
      uint32_t uu[NW_ILP];
      bool vv[NW_ILP];
      int64_t hh[NW_ILP];
#pragma unroll
      for (int i = 0; i < NW_ILP; ++i) {
        const int64_t wd = w0 + i0 + i;
        const int64_t p = wd * 32 + lane;
        vv[i] = false;
        if (i0 + i < wpw && wd < wend && p < PT) {
          const int64_t j = p / k;
          vv[i] = (p - j * k) < __ldcg(S.stg.ccnt + j);
        }
        uu[i] = vv[i] ? (uint32_t)__ldcg(S.stg.u + p) : 0u;
      }
#pragma unroll
      for (int i = 0; i < NW_ILP; ++i)
        hh[i] = vv[i] ? ct_find(S.stg.tab, log_cap, uu[i]) : -1;
#pragma unroll
      for (int i = 0; i < NW_ILP; ++i) {
        const int64_t wd = w0 + i0 + i;
        const int64_t p = wd * 32 + lane;
        bool first = false;
        if (vv[i]) {
          if (hh[i] < 0) atomicOr(P.core.err, ERR_INTERNAL);
          else first = tab_val(__ldcg(S.stg.tab + hh[i])) == (uint32_t)p;
        }
        const uint32_t word = __ballot_sync(0xffffffffu, first);
        if (i0 + i < wpw) {
          if (wd < wend && lane == 0) S.bits[wd] = word;
          if (lane == 0) sm.wcnt[warp * wpw + i0 + i] = __popc(word);
          wrun += __popc(word);
        }
      }
    }
    if (lane == 0) sm.wtot[warp] = wrun;
    __syncthreads();
    if (warp == 0) {
      const int v = lane < NS_WARPS ? sm.wtot[lane] : 0;
      int tot;
      const int ex = warp_excl(v, &tot);
      if (lane < NS_WARPS) sm.wtot[lane] = ex;
      if (lane == 0) sm.x[3] = tot;  // tile rows
    }
    __syncthreads();
    {  // per-word tile-local prefix
      int run = sm.wtot[warp];
      for (int i0 = 0; i0 < wpw; i0 += 32) {
        const int i = i0 + lane;
        const int c = i < wpw ? sm.wcnt[warp * wpw + i] : 0;
        int tot;
        const int ex = warp_excl(c, &tot);
        if (i < wpw && w0 + i < wend) S.wpre[w0 + i] = run + ex;
        run += tot;
      }
    }
    // ---- 4. decoupled look-back over the hop's tiles ----
    if (threadIdx.x == 0) {
      const int64_t te = sm.x[2], tr = sm.x[3];
      __threadfence();
      int64_t xe = 0, xr = 0;
      if (t > 0) {
        lba[t] = lb_pack(te, tr);
        __threadfence();
        st_rel_u64(&lbs[t], lb_status_word(btag, LB_A));
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
          __nanosleep(32);
        }
      }
      rx[t] = xr;
      lbp[t] = lb_pack(xe + te, xr + tr);
      __threadfence();
      st_rel_u64(&lbs[t], lb_status_word(btag, LB_P));
      sm.x[0] = xe;
      sm.x[1] = xr;
    }
    __syncthreads();
    // ---- 5. relabel + compaction ----
    const int64_t xe = sm.x[0], xr = sm.x[1];
    const int64_t colbase = l == 0 ? bstart : bstart * P.K[l - 1];
    const int64_t rbase = bstart * P.K[l];
    const int64_t ibase = colbase + b;
    int32_t* row_map = P.row_map[l] + rbase;
    int32_t* row_local = P.row_local[l] + rbase;
    int64_t* eid_out = P.eid[l] + rbase;
    float* val_out = P.val[l] ? P.val[l] + rbase : nullptr;
    const int tile_slots = NS_COLS * k;
    if (jb < tend) {
      WarpChunk& C = sm.wc[warp];
      const int64_t j = jb + lane;
      const bool act = j < tend;
      const int cnt = act ? __ldcg(S.stg.ccnt + j) : 0;
      const int eo = act ? __ldcg(S.ceoff + j) : 0;
      const int64_t off = act ? __ldcg(S.stg.coff + j) : 0;
      int total;
      const int cpre = warp_excl(cnt, &total);
      C.pre[lane] = cpre;
      C.coff[lane] = off;
      C.cnt_all[lane] = eo;
      if (act) {
        P.indptr_out[l][ibase + j] = xe + eo;
        if (l == 0) P.col0[bstart + j] = __ldcg(P.seeds + bstart + j);
      }
      __syncwarp();
      for (int f0 = 0; f0 < total; f0 += 32 * NW_ILP) {
        int64_t p[NW_ILP], ee[NW_ILP], hh[NW_ILP];
        uint32_t uu[NW_ILP], ps[NW_ILP];
        int cc[NW_ILP];
        bool ok[NW_ILP];
#pragma unroll
        for (int i = 0; i < NW_ILP; ++i) {
          const int f = f0 + i * 32 + lane;
          ok[i] = f < total;
          cc[i] = 0;
          p[i] = ee[i] = 0;
          uu[i] = ps[i] = 0;
          if (ok[i]) {
            const int c = chunk_col(C.pre, f);
            const int s = f - C.pre[c];
            p[i] = (jb + c) * k + s;
            ee[i] = xe + C.cnt_all[c] + s;
            uu[i] = (uint32_t)__ldcg(S.stg.u + p[i]);
            ps[i] = __ldcg(S.stg.pos + p[i]);
            cc[i] = c;
          }
        }
#pragma unroll
        for (int i = 0; i < NW_ILP; ++i) {
          hh[i] = -1;
          if (ok[i]) {
            eid_out[ee[i]] = C.coff[cc[i]] + ps[i];
            if (val_out) val_out[ee[i]] = __ldcg(S.stg.val + p[i]);
            hh[i] = ct_find(S.stg.tab, log_cap, uu[i]);
          }
        }
#pragma unroll
        for (int i = 0; i < NW_ILP; ++i) {
          if (ok[i]) {
            const uint32_t p0 = hh[i] >= 0 ? tab_val(__ldcg(S.stg.tab + hh[i])) : 0u;
            const int t0 = (int)(p0 / (uint32_t)tile_slots);
            long long base;
            if (t0 == t) {
              base = xr;
            } else {  // the first slot is in an earlier tile: wait for its prefix
              while (ld_acq_u64(&lbs[t0]) != lb_status_word(btag, LB_P)) __nanosleep(32);
              base = __ldcg(rx + t0);
            }
            const int64_t wd = p0 >> 5;
            const uint32_t bw = __ldcg(S.bits + wd);
            const int64_t lid = base + __ldcg(S.wpre + wd) + __popc(bw & ((1u << (p0 & 31)) - 1u));
            row_local[ee[i]] = (int32_t)lid;
            if (p0 == (uint32_t)p[i]) row_map[lid] = (int32_t)uu[i];
          }
        }
      }
      __syncwarp();
    }
  }
  // ---- 6. completion of the hop ----
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned int d = atomicAdd(&B.cnt[l], 1u) + 1u;
    sm.flag = (d == (unsigned int)P.maxtiles[l]);
    if (sm.flag) {
      __threadfence();
      int64_t E = 0, R = 0;
      if (ntiles > 0) {
        const int64_t i = (int64_t)l * P.max_tiles_all + ntiles - 1;
        while (ld_acq_u64(&S.lbs[i]) != lb_status_word(btag, LB_P)) __nanosleep(32);
        const unsigned long long v = __ldcg(&S.lbp[i]);
        E = lb_e(v);
        R = lb_r(v);
      }
      sm.x[2] = E;
      sm.x[3] = R;
    }
  }
  __syncthreads();
  if (sm.flag) {
    // clear this hop's part of the table for the next user of the slot
    const int64_t cap = 1ll << log_cap;
    for (int64_t i = threadIdx.x; i < cap; i += blockDim.x) S.stg.tab[i] = ~0ull;
    __syncthreads();
    if (threadIdx.x == 0) {
      const int64_t E = sm.x[2], R = sm.x[3];
      const int64_t colbase = l == 0 ? bstart : bstart * P.K[l - 1];
      const int64_t rbase = bstart * P.K[l];
      const int64_t ibase = colbase + b;
      P.indptr_out[l][ibase + T] = E;
      long long* m = (long long*)(P.meta + (b * P.L + l) * 8);
      m[0] = T; m[1] = R; m[2] = E; m[3] = colbase; m[4] = rbase; m[5] = ibase; m[6] = rbase;
      m[7] = 0;
      __threadfence();
      if (l + 1 < P.L) {
        B.T[l + 1] = R;
        __threadfence();
        st_rel_u32(&B.ready[l + 1], 1u);
      } else {
        st_rel_u32(&B.done, 1u);
      }
    }
  }
}

__global__ void __launch_bounds__(NS_THREADS, 2) nodewise_stream_kernel(NSParams P) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  NSSmem& sm = *reinterpret_cast<NSSmem*>(smem_raw);
  const unsigned long long total = (unsigned long long)P.nsteps * P.tps;
  while (true) {
    if (threadIdx.x == 0) sm.job[0] = (long long)atomicAdd(P.ticket, 1ull);
    __syncthreads();
    const unsigned long long tk = (unsigned long long)sm.job[0];
    __syncthreads();
    if (tk >= total) break;
    const int64_t step = (int64_t)(tk / P.tps);
    const int r = (int)(tk % P.tps);
    int l = 0;
    while (l + 1 < P.L && r >= P.tile_off[l + 1]) ++l;  // tile_off is increasing in l's order
    // hops are laid out deepest first: map the range index back to the hop
    const int hop = P.L - 1 - l;
    const int t = r - P.tile_off[l];
    const int64_t b = step - (int64_t)hop * NS_LAG;
    if (b < 0 || b >= P.num_batches) continue;
    ns_tile(P, sm, b, hop, t);
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
    P.maxtiles[l] = (int)((cols + NS_COLS - 1) / NS_COLS);
    max_t = std::max(max_t, P.maxtiles[l]);
    prod *= fanouts[l];
    P.K[l] = prod;
    slot_cap = std::max(slot_cap, cols * fanouts[l]);
  }
  // deepest hop first inside a step
  int off = 0;
  for (int i = 0; i < L; ++i) {
    const int hop = L - 1 - i;
    P.tile_off[i] = off;
    off += P.maxtiles[hop];
  }
  P.tps = off;
  P.max_tiles_all = max_t;
  P.win = (L - 1) * NS_LAG + NS_LAG + 2;
  const int64_t nbatch = P.num_batches;
  P.nsteps = nbatch + (int64_t)(L - 1) * NS_LAG;
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
  const int64_t sched_bytes = nbatch * (int64_t)sizeof(NSBatch) + 256;
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
  P.o_tab = o; o = align256(o + (int64_t(8) << log_tab));
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
  nodewise_stream_kernel<<<grid, NS_THREADS, sizeof(NSSmem), stream>>>(P);
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

}  // namespace gsb
