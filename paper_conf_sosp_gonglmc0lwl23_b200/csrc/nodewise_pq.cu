// nodewise_pq.cu -- node-wise ECSF sampling (GraphSAGE, KGCN, weighted A-Res,
// PASS-style A3) as ONE persistent, barrier-free work-queue kernel per epoch.
//
// Why: per mini-batch work is microseconds, so any
// per-batch barrier structure is latency bound.  Here every resident CTA pulls
// TILES of (batch, hop, phase) work from a window of PQ_WIN in-flight
// mini-batches (super-batch sampling); a batch's phases advance
// when its last tile completes ("last block done"), and different batches'
// phases overlap, so the whole GPU works on the few batches whose hash tables
// and slot staging are live in L2.  Phases of one hop of one batch:
//   CLEAR  (only every 255 hops of a window slot) reset the table to ~0;
//   SEL    Extract + Select (Extract-Select fusion P:289):
//          tiles of 512 columns, one 32-column chunk per warp
//          (nodewise_common.cuh: Floyd / replacement / A-Res, flattened gather,
//          staging, ordered-hash insert keeping the first slot of every row);
//   FLAG   Finalize-1: first-occurrence bitmap over the padded slots, tiles of
//          64 words (2048 slots), per-word tile-local prefix counts;
//   EMIT   Finalize-2: row id = rank of the row's first slot,
//          compaction into the block (CSC indptr + COO row_local/eid) and
//          row_map (the next frontier, R2).
// The tile-total prefixes are computed by the finalising CTA (one warp).
#include <algorithm>
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "gs_internal.h"
#include "nodewise_common.cuh"

namespace gsb {

constexpr int PQ_THREADS = 512;
constexpr int PQ_WARPS = PQ_THREADS / 32;
constexpr int PQ_COLS = PQ_WARPS * 32;      // columns per SEL / EMIT tile
constexpr int PQ_WPT = PQ_WARPS * NW_ILP;   // bitmap words per FLAG tile
constexpr int PQ_WIN = 16;                  // mini-batches in flight (workspace slots)
constexpr int PQ_CLEAR = 1 << 16;           // table entries per CLEAR tile

constexpr uint32_t ST_IDLE = 0, ST_INIT = 0xFFFE, ST_DONE = 0xFFFF;
enum { PH_CLEAR = 0, PH_SEL = 1, PH_FLAG = 2, PH_EMIT = 3 };

__host__ __device__ constexpr uint32_t stage_of(int hop, int ph) { return 1u + hop * 4u + ph; }
__device__ __forceinline__ int stage_hop(uint32_t s) { return (int)((s - 1u) >> 2); }
__device__ __forceinline__ int stage_ph(uint32_t s) { return (int)((s - 1u) & 3u); }

__device__ __forceinline__ unsigned long long make_word(uint32_t stage, uint32_t ntiles) {
  return ((unsigned long long)stage << 48) | ((unsigned long long)ntiles << 28);
}
__device__ __forceinline__ uint32_t w_stage(unsigned long long w) { return (uint32_t)(w >> 48); }
__device__ __forceinline__ uint32_t w_ntiles(unsigned long long w) {
  return (uint32_t)((w >> 28) & 0xFFFFFu);
}
__device__ __forceinline__ uint32_t w_claimed(unsigned long long w) {
  return (uint32_t)(w & 0xFFFFFFFu);
}

struct BState {                 // one per mini-batch (64 B)
  unsigned long long word;      // stage(16) | ntiles(20) | claimed(28)
  unsigned int done;            // tiles completed in the current stage
  unsigned int gen;             // table generation of the current hop (1..255)
  long long T;                  // frontier columns of the current hop
  long long E;                  // edges of the current hop (after SEL)
  long long R;                  // rows of the current hop (after FLAG)
  long long colbase;            // column region of the current hop
  long long pad[2];
};

struct PQParams {
  NWCore core;
  const int32_t* seeds;
  int64_t num_seeds, batch_size, num_batches, batch_base;
  int L;
  int k[MAX_LAYERS];
  int64_t K[MAX_LAYERS];
  int32_t* col0;
  int32_t* row_map[MAX_LAYERS];
  int64_t* indptr_out[MAX_LAYERS];
  int32_t* row_local[MAX_LAYERS];
  int64_t* eid[MAX_LAYERS];
  float* val[MAX_LAYERS];
  int64_t* meta;
  BState* st;
  unsigned long long* lo;       // first not-finished batch
  uint32_t* slot_gen;           // [PQ_WIN] generation counter of each workspace slot
  char* ws;
  int64_t ws_stride;
  int64_t o_u, o_pos, o_val, o_coff, o_ccnt, o_ceoff, o_bits, o_wpre, o_tte, o_ttr, o_tab;
  int log_tab_cap;
};

struct Slot {
  NWStage stg;
  int32_t* ceoff;
  uint32_t* bits;
  int32_t* wpre;
  long long* tte;   // SEL tile edge totals -> exclusive prefix
  long long* ttr;   // FLAG tile row totals -> exclusive prefix
};

__device__ __forceinline__ Slot slot_of(const PQParams& P, int64_t b) {
  char* base = P.ws + (b % PQ_WIN) * P.ws_stride;
  Slot s;
  s.stg.u = (int32_t*)(base + P.o_u);
  s.stg.pos = (uint32_t*)(base + P.o_pos);
  s.stg.val = P.o_val >= 0 ? (float*)(base + P.o_val) : nullptr;
  s.stg.coff = (int64_t*)(base + P.o_coff);
  s.stg.ccnt = (int32_t*)(base + P.o_ccnt);
  s.stg.tab = (unsigned long long*)(base + P.o_tab);
  s.ceoff = (int32_t*)(base + P.o_ceoff);
  s.bits = (uint32_t*)(base + P.o_bits);
  s.wpre = (int32_t*)(base + P.o_wpre);
  s.tte = (long long*)(base + P.o_tte);
  s.ttr = (long long*)(base + P.o_ttr);
  return s;
}

struct PQSmem {
  WarpChunk wc[PQ_WARPS];
  int wtot[PQ_WARPS];
  int wcnt[PQ_WPT];
  long long job[4];   // kind, batch, stage, tile
  int flag;
};

enum { JOB_NONE = 0, JOB_TILE = 1, JOB_INIT = 2, JOB_EXIT = 3 };

__device__ __forceinline__ int hop_log_cap(const PQParams& P, int64_t T, int k) {
  int lc = log2_pow2ceil64((T * k * 4) / 3 + 64);
  return lc > P.log_tab_cap ? P.log_tab_cap : lc;
}

__device__ __forceinline__ const int32_t* frontier(const PQParams& P, int64_t b, int l) {
  const int64_t bstart = b * P.batch_size;
  return l == 0 ? P.seeds + bstart : P.row_map[l - 1] + bstart * P.K[l - 1];
}

// Publishes (stage, ntiles) for batch b after its fields were written.
__device__ __forceinline__ void publish(const PQParams& P, int64_t b, uint32_t stage, uint32_t nt) {
  P.st[b].done = 0u;
  __threadfence();
  atomicExch(&P.st[b].word, make_word(stage, nt));
}

// Enters hop l of batch b (T columns): picks the table generation of the slot,
// a CLEAR stage when the generation wraps, else SEL.  Returns (stage, ntiles).
__device__ void enter_hop(const PQParams& P, int64_t b, int l, int64_t T, int64_t colbase,
                          uint32_t* stage, uint32_t* nt) {
  const int slot = (int)(b % PQ_WIN);
  uint32_t g = P.slot_gen[slot] + 1u;
  P.st[b].T = T;
  P.st[b].colbase = colbase;
  if (g > 255u) {
    g = 1u;
    *stage = stage_of(l, PH_CLEAR);
    *nt = (uint32_t)(((1ll << P.log_tab_cap) + PQ_CLEAR - 1) / PQ_CLEAR);
  } else {
    *stage = stage_of(l, PH_SEL);
    *nt = (uint32_t)((T + PQ_COLS - 1) / PQ_COLS);
  }
  P.slot_gen[slot] = g;
  P.st[b].gen = g;
}

// Finalises `stage` of batch b (all its tiles done) and publishes the next
// stage; zero-tile stages are finalised on the spot.  Run by warp 0.
__device__ void finalize(const PQParams& P, int64_t b, uint32_t stage) {
  const int lane = threadIdx.x & 31;
  const int64_t bstart = b * P.batch_size;
  while (true) {
    const int l = stage_hop(stage), ph = stage_ph(stage);
    const int k = P.k[l];
    const Slot S = slot_of(P, b);
    const int64_t T = __ldcg(&P.st[b].T);
    uint32_t next = 0, nt = 0;
    if (ph == PH_CLEAR) {
      next = stage_of(l, PH_SEL);
      nt = (uint32_t)((T + PQ_COLS - 1) / PQ_COLS);
    } else if (ph == PH_SEL || ph == PH_FLAG) {
      // exclusive prefix over the tile totals (in place)
      long long* tt = ph == PH_SEL ? S.tte : S.ttr;
      const int64_t ntiles = ph == PH_SEL ? (T + PQ_COLS - 1) / PQ_COLS
                                          : (((T * k + 31) >> 5) + PQ_WPT - 1) / PQ_WPT;
      long long run = 0;
      for (int64_t t0 = 0; t0 < ntiles; t0 += 32) {
        const int64_t t = t0 + lane;
        const long long v = t < ntiles ? __ldcg(tt + t) : 0;
        long long inc = v;
        for (int o = 1; o < 32; o <<= 1) {
          const long long n = __shfl_up_sync(0xffffffffu, inc, o);
          if (lane >= o) inc += n;
        }
        if (t < ntiles) tt[t] = run + inc - v;
        run += __shfl_sync(0xffffffffu, inc, 31);
      }
      if (lane == 0) {
        if (ph == PH_SEL) {
          P.st[b].E = run;
          next = stage_of(l, PH_FLAG);
          nt = (uint32_t)((((T * k + 31) >> 5) + PQ_WPT - 1) / PQ_WPT);
        } else {
          P.st[b].R = run;
          next = stage_of(l, PH_EMIT);
          nt = (uint32_t)((T + PQ_COLS - 1) / PQ_COLS);
        }
      }
    } else {  // EMIT done: block complete
      if (lane == 0) {
        const int64_t E = __ldcg(&P.st[b].E), R = __ldcg(&P.st[b].R);
        const int64_t colbase = __ldcg(&P.st[b].colbase);
        const int64_t rbase = bstart * P.K[l];
        const int64_t ibase = colbase + b;
        P.indptr_out[l][ibase + T] = E;
        long long* m = (long long*)(P.meta + (b * P.L + l) * 8);
        m[0] = T; m[1] = R; m[2] = E; m[3] = colbase; m[4] = rbase; m[5] = ibase; m[6] = rbase;
        m[7] = 0;
        if (l + 1 < P.L) {
          enter_hop(P, b, l + 1, R, rbase, &next, &nt);
        } else {
          next = ST_DONE;
          nt = 0;
        }
      }
    }
    if (lane == 0) __threadfence();
    __syncwarp();
    next = __shfl_sync(0xffffffffu, next, 0);
    nt = __shfl_sync(0xffffffffu, nt, 0);
    if (lane == 0) {
      if (next == ST_DONE) {
        publish(P, b, ST_DONE, 0);
        // advance the low-water mark over finished batches
        while (true) {
          const unsigned long long cur = *(volatile unsigned long long*)P.lo;
          if ((int64_t)cur >= P.num_batches) break;
          if (w_stage(__ldcg(&P.st[cur].word)) != ST_DONE) break;
          atomicCAS(P.lo, cur, cur + 1);
        }
      } else if (nt > 0) {
        publish(P, b, next, nt);
      }
    }
    if (next == ST_DONE || nt > 0) break;
    stage = next;  // empty stage: finalise it right away
  }
}

// Initialises batch b (stage ST_INIT, owned by this CTA).  Warp 0.
__device__ void init_batch(const PQParams& P, int64_t b) {
  const int lane = threadIdx.x & 31;
  uint32_t stage = 0, nt = 0;
  if (lane == 0) {
    const int64_t bstart = b * P.batch_size;
    const int64_t nb = min(P.batch_size, P.num_seeds - bstart);
    enter_hop(P, b, 0, nb, bstart, &stage, &nt);
    if (nt > 0) publish(P, b, stage, nt);
  }
  stage = __shfl_sync(0xffffffffu, stage, 0);
  nt = __shfl_sync(0xffffffffu, nt, 0);
  if (nt == 0) finalize(P, b, stage);
}

// ---------------------------------------------------------------------------
// Tiles
// ---------------------------------------------------------------------------
__device__ void tile_clear(const PQParams& P, int64_t b, int64_t t) {
  const Slot S = slot_of(P, b);
  const int64_t cap = 1ll << P.log_tab_cap;
  const int64_t a = t * PQ_CLEAR, e = min(cap, a + PQ_CLEAR);
  for (int64_t i = a + threadIdx.x; i < e; i += blockDim.x) S.stg.tab[i] = ~0ull;
}

__device__ void tile_sel(const PQParams& P, PQSmem& sm, int64_t b, int l, int64_t t) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const Slot S = slot_of(P, b);
  const int64_t T = __ldcg(&P.st[b].T);
  const uint32_t tag = otag(__ldcg(&P.st[b].gen));
  const int k = P.k[l];
  const int log_cap = hop_log_cap(P, T, k);
  const uint32_t gb = (uint32_t)(P.batch_base + b);
  const int32_t* F = frontier(P, b, l);
  const int64_t tend = min(T, (t + 1) * PQ_COLS);
  const int64_t jb = t * PQ_COLS + warp * 32;
  int e = 0, pre = 0;
  if (jb < tend) {
    e = select_chunk(P.core, S.stg, sm.wc[warp], l, k, log_cap, tag, F, jb, tend, gb);
    pre = sm.wc[warp].pre[lane];
  }
  if (lane == 0) sm.wtot[warp] = e;
  __syncthreads();
  if (warp == 0) {
    const int v = lane < PQ_WARPS ? sm.wtot[lane] : 0;
    int tot;
    const int ex = warp_excl(v, &tot);
    if (lane < PQ_WARPS) sm.wtot[lane] = ex;
    if (lane == 0) S.tte[t] = tot;
  }
  __syncthreads();
  if (jb + lane < tend) S.ceoff[jb + lane] = sm.wtot[warp] + pre;
}

__device__ void tile_flag(const PQParams& P, PQSmem& sm, int64_t b, int l, int64_t t) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const Slot S = slot_of(P, b);
  const int64_t T = __ldcg(&P.st[b].T);
  const uint32_t tag = otag(__ldcg(&P.st[b].gen));
  const int k = P.k[l];
  const int log_cap = hop_log_cap(P, T, k);
  const int64_t PT = T * k, NWD = (PT + 31) >> 5;
  const int64_t wb = t * PQ_WPT + warp * NW_ILP;
  uint32_t uu[NW_ILP];
  bool vv[NW_ILP];
  int64_t hh[NW_ILP];
#pragma unroll
  for (int i = 0; i < NW_ILP; ++i) {
    const int64_t wd = wb + i;
    const int64_t p = wd * 32 + lane;
    vv[i] = false;
    if (wd < NWD && p < PT) {
      const int64_t j = p / k;
      vv[i] = (p - j * k) < __ldcg(S.stg.ccnt + j);
    }
    uu[i] = vv[i] ? (uint32_t)__ldcg(S.stg.u + p) : 0u;
  }
#pragma unroll
  for (int i = 0; i < NW_ILP; ++i) hh[i] = vv[i] ? otab_find(S.stg.tab, log_cap, tag, uu[i]) : -1;
#pragma unroll
  for (int i = 0; i < NW_ILP; ++i) {
    const int64_t wd = wb + i;
    const int64_t p = wd * 32 + lane;
    bool first = false;
    if (vv[i]) {
      if (hh[i] < 0) atomicOr(P.core.err, ERR_INTERNAL);
      else first = tab_val(__ldcg(S.stg.tab + hh[i])) == (uint32_t)p;
    }
    const uint32_t word = __ballot_sync(0xffffffffu, first);
    if (wd < NWD && lane == 0) S.bits[wd] = word;
    if (lane == 0) sm.wcnt[warp * NW_ILP + i] = __popc(word);
  }
  __syncthreads();
  if (warp == 0) {  // tile-local exclusive prefix over the tile's 64 words
    const int a = sm.wcnt[2 * lane], c = sm.wcnt[2 * lane + 1];
    int tot;
    const int ex = warp_excl(a + c, &tot);
    const int64_t w0 = t * PQ_WPT + 2 * lane;
    if (w0 < NWD) S.wpre[w0] = ex;
    if (w0 + 1 < NWD) S.wpre[w0 + 1] = ex + a;
    if (lane == 0) S.ttr[t] = tot;
  }
}

__device__ void tile_emit(const PQParams& P, PQSmem& sm, int64_t b, int l, int64_t t) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const Slot S = slot_of(P, b);
  const int64_t T = __ldcg(&P.st[b].T);
  const uint32_t tag = otag(__ldcg(&P.st[b].gen));
  const int k = P.k[l];
  const int log_cap = hop_log_cap(P, T, k);
  const int64_t bstart = b * P.batch_size;
  const int64_t colbase = __ldcg(&P.st[b].colbase);
  const int64_t rbase = bstart * P.K[l];
  const int64_t ibase = colbase + b;
  const int64_t tend = min(T, (t + 1) * PQ_COLS);
  const int64_t jb = t * PQ_COLS + warp * 32;
  if (jb >= tend) return;
  const long long tbase = __ldcg(S.tte + t);
  int32_t* row_map = P.row_map[l] + rbase;
  int32_t* row_local = P.row_local[l] + rbase;
  int64_t* eid_out = P.eid[l] + rbase;
  float* val_out = P.val[l] ? P.val[l] + rbase : nullptr;
  WarpChunk& C = sm.wc[warp];
  const int64_t j = jb + lane;
  const bool act = j < tend;
  const int cnt = act ? __ldcg(S.stg.ccnt + j) : 0;
  const int eo = act ? __ldcg(S.ceoff + j) : 0;
  const int64_t off = act ? __ldcg(S.stg.coff + j) : 0;
  int total;
  const int pre = warp_excl(cnt, &total);
  C.pre[lane] = pre;
  C.coff[lane] = off;
  C.cnt_all[lane] = eo;
  if (act) {
    P.indptr_out[l][ibase + j] = tbase + eo;
    if (l == 0) P.col0[bstart + j] = __ldcg(P.seeds + bstart + j);
  }
  __syncwarp();
  for (int f0 = 0; f0 < total; f0 += 32 * NW_ILP) {
    int64_t p[NW_ILP], e[NW_ILP], hh[NW_ILP];
    uint32_t uu[NW_ILP], ps[NW_ILP];
    int cc[NW_ILP];
    bool ok[NW_ILP];
#pragma unroll
    for (int i = 0; i < NW_ILP; ++i) {
      const int f = f0 + i * 32 + lane;
      ok[i] = f < total;
      cc[i] = 0;
      p[i] = e[i] = 0;
      uu[i] = ps[i] = 0;
      if (ok[i]) {
        const int c = chunk_col(C.pre, f);
        const int s = f - C.pre[c];
        p[i] = (jb + c) * k + s;
        e[i] = tbase + C.cnt_all[c] + s;
        uu[i] = (uint32_t)__ldcg(S.stg.u + p[i]);
        ps[i] = __ldcg(S.stg.pos + p[i]);
        cc[i] = c;
      }
    }
#pragma unroll
    for (int i = 0; i < NW_ILP; ++i) {
      hh[i] = -1;
      if (ok[i]) {
        eid_out[e[i]] = C.coff[cc[i]] + ps[i];
        if (val_out) val_out[e[i]] = __ldcg(S.stg.val + p[i]);
        hh[i] = otab_find(S.stg.tab, log_cap, tag, uu[i]);
      }
    }
#pragma unroll
    for (int i = 0; i < NW_ILP; ++i) {
      if (ok[i]) {
        const uint32_t p0 = hh[i] >= 0 ? tab_val(__ldcg(S.stg.tab + hh[i])) : 0u;
        const int64_t wd = p0 >> 5;
        const uint32_t bw = __ldcg(S.bits + wd);
        const int64_t lid = __ldcg(S.ttr + wd / PQ_WPT) + __ldcg(S.wpre + wd) +
                            __popc(bw & ((1u << (p0 & 31)) - 1u));
        row_local[e[i]] = (int32_t)lid;
        if (p0 == (uint32_t)p[i]) row_map[lid] = (int32_t)uu[i];
      }
    }
  }
  __syncwarp();
}

// ---------------------------------------------------------------------------
// Scheduler: warp 0 finds the oldest claimable tile in the window.
// ---------------------------------------------------------------------------
__device__ void find_work(const PQParams& P, PQSmem& sm) {
  const int lane = threadIdx.x & 31;
  const unsigned long long lo = *(volatile unsigned long long*)P.lo;
  if ((int64_t)lo >= P.num_batches) {
    if (lane == 0) sm.job[0] = JOB_EXIT;
    return;
  }
  const int64_t b = (int64_t)lo + lane;
  const bool in = lane < PQ_WIN && b < P.num_batches;
  const unsigned long long w = in ? __ldcg(&P.st[b].word) : 0ull;
  const uint32_t s = w_stage(w);
  const bool cand = in && (s == ST_IDLE || (s != ST_INIT && s != ST_DONE &&
                                            w_claimed(w) < w_ntiles(w)));
  uint32_t m = __ballot_sync(0xffffffffu, cand);
  long long kind = JOB_NONE, st = 0, tile = 0, bb = 0;
  while (m) {
    const int c = __ffs(m) - 1;
    int got = 0;
    long long gs = 0, gt = 0;
    if (lane == c) {
      if (s == ST_IDLE) {
        if (atomicCAS(&P.st[b].word, w, make_word(ST_INIT, 0)) == w) got = JOB_INIT;
      } else {
        const unsigned long long old = atomicAdd(&P.st[b].word, 1ull);
        const uint32_t s2 = w_stage(old);
        if (s2 != ST_INIT && s2 != ST_DONE && s2 != ST_IDLE && w_claimed(old) < w_ntiles(old)) {
          got = JOB_TILE;
          gs = s2;
          gt = w_claimed(old);
        }
      }
    }
    got = __shfl_sync(0xffffffffu, got, c);
    if (got) {
      kind = got;
      bb = (int64_t)lo + c;
      st = __shfl_sync(0xffffffffu, gs, c);
      tile = __shfl_sync(0xffffffffu, gt, c);
      break;
    }
    m &= m - 1u;
  }
  if (lane == 0) {
    sm.job[0] = kind;
    sm.job[1] = bb;
    sm.job[2] = st;
    sm.job[3] = tile;
  }
  __threadfence();
}

__global__ void __launch_bounds__(PQ_THREADS, 2) nodewise_pq_kernel(PQParams P) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  PQSmem& sm = *reinterpret_cast<PQSmem*>(smem_raw);
  const int warp = threadIdx.x >> 5;
  while (true) {
    if (warp == 0) find_work(P, sm);
    __syncthreads();
    const long long kind = sm.job[0], b = sm.job[1], st = sm.job[2], tile = sm.job[3];
    __syncthreads();
    if (kind == JOB_EXIT) break;
    if (kind == JOB_NONE) {
      __nanosleep(200);
      continue;
    }
    if (kind == JOB_INIT) {
      if (warp == 0) init_batch(P, b);
      __syncthreads();
      continue;
    }
    const uint32_t stage = (uint32_t)st;
    const int l = stage_hop(stage), ph = stage_ph(stage);
    if (ph == PH_CLEAR) tile_clear(P, b, tile);
    else if (ph == PH_SEL) tile_sel(P, sm, b, l, tile);
    else if (ph == PH_FLAG) tile_flag(P, sm, b, l, tile);
    else tile_emit(P, sm, b, l, tile);
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence();
      const unsigned int ntiles = w_ntiles(__ldcg(&P.st[b].word));
      const unsigned int d = atomicAdd(&P.st[b].done, 1u) + 1u;
      sm.flag = (d == ntiles);
      __threadfence();
    }
    __syncthreads();
    if (sm.flag && warp == 0) finalize(P, b, stage);
    __syncthreads();
  }
}

// ---------------------------------------------------------------------------
// Host side
// ---------------------------------------------------------------------------
static int64_t align256(int64_t x) { return (x + 255) & ~int64_t(255); }

gs_status run_nodewise_pq(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                          int64_t batch_size, int64_t batch_base, const int32_t* fanouts, int L,
                          int replace, int bias, uint64_t key, cudaStream_t stream,
                          gs_blocks* blk) {
  const Allocator& al = blk->al;
  PQParams P = {};
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
  for (int l = 0; l < L; ++l) {
    P.k[l] = fanouts[l];
    col_cap = std::max(col_cap, batch_size * prod);
    prod *= fanouts[l];
    P.K[l] = prod;
    slot_cap = std::max(slot_cap, batch_size * prod);
  }
  col_cap += PQ_COLS;
  slot_cap += 64 * 32;
  const int64_t nbatch = P.num_batches;
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
  ok = ok && need(blk->b_meta, nbatch * L * 8 * 8) && need(blk->b_err, 16) &&
       need(blk->b_ctr, 8 * (MAX_LAYERS + 2)) && need(blk->b_sched, nbatch * sizeof(BState) + 256);
  if (!ok) return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (blocks buffers)");

  int log_tab = 6;
  while ((int64_t(1) << log_tab) < (slot_cap * 4) / 3 + 64) ++log_tab;
  const int64_t words = (slot_cap + 31) / 32 + PQ_WPT;
  const int64_t sel_tiles = (col_cap + PQ_COLS - 1) / PQ_COLS + 1;
  const int64_t flag_tiles = (words + PQ_WPT - 1) / PQ_WPT + 1;
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
  P.o_tte = o; o = align256(o + sel_tiles * 8);
  P.o_ttr = o; o = align256(o + flag_tiles * 8);
  P.o_tab = o; o = align256(o + (int64_t(8) << log_tab));
  P.ws_stride = o;
  P.log_tab_cap = log_tab;
  const size_t ws_bytes = (size_t)P.ws_stride * PQ_WIN;
  const bool fresh = blk->b_ws.bytes < ws_bytes || blk->ws_stride_prev != P.ws_stride ||
                     blk->ws_kind_prev != 3;
  if (!blk->b_ws.ensure(al, ws_bytes, stream) || !blk->b_gen.ensure(al, 4096 * 4, stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (workspace)");
  if (fresh) {  // tables start cleared (~0 = the oldest generation)
    GS_CUDA_TRY(cudaMemsetAsync(blk->b_ws.ptr, 0xFF, blk->b_ws.bytes, stream));
    GS_CUDA_TRY(cudaMemsetAsync(blk->b_gen.ptr, 0, 4096 * 4, stream));
  }
  blk->ws_stride_prev = P.ws_stride;
  blk->ws_kind_prev = 3;
  P.ws = (char*)blk->b_ws.ptr;
  P.slot_gen = (uint32_t*)blk->b_gen.ptr;
  P.st = (BState*)blk->b_sched.ptr;
  P.lo = (unsigned long long*)((char*)blk->b_sched.ptr + nbatch * sizeof(BState));

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
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_sched.ptr, 0, nbatch * sizeof(BState) + 256, stream));
  if (nbatch == 0) return GS_OK;

  static int grid = 0;
  if (grid == 0) {
    GS_CUDA_TRY(cudaFuncSetAttribute(nodewise_pq_kernel,
                                     cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)sizeof(PQSmem)));
    int per_sm = 0, dev = 0, sms = 148;
    GS_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, nodewise_pq_kernel,
                                                              PQ_THREADS, sizeof(PQSmem)));
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    grid = std::max(1, per_sm) * sms;  // all CTAs co-resident (persistent)
  }
  nodewise_pq_kernel<<<grid, PQ_THREADS, sizeof(PQSmem), stream>>>(P);
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

}  // namespace gsb
