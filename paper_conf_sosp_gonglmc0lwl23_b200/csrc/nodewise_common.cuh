// nodewise_common.cuh -- device building blocks of the node-wise select
// (Extract + Select fused): per-warp chunks of 32 frontier columns,
// Floyd / replacement / A-Res positions in shared memory, flattened gather of
// the sampled rows with NW_ILP loads in flight per lane, staging and the
// ordered-hash first-occurrence insert.
#pragma once
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include "common.cuh"
#include "gs_internal.h"

namespace gsb {

constexpr int NW_ILP = 4;  // independent slots per lane in flight

// Read-only graph + sampling parameters shared by the node-wise kernels.
struct NWCore {
  const int64_t* indptr;
  const int32_t* indices;
  const float* weights;
  int64_t N;
  int* err;
  int replace, bias;
  uint64_t key;
};

// Per-batch-hop staging written by the select step.
struct NWStage {
  int32_t* u;      // [slot] sampled row
  uint32_t* pos;   // [slot] position inside the column
  float* val;      // [slot] PASS prob (or NULL)
  int64_t* coff;   // [col] indptr[v]
  int32_t* ccnt;   // [col] sampled edges of the column
  unsigned long long* tab;
};

// Shared memory of one warp's chunk of 32 columns.
struct WarpChunk {
  uint32_t list[MAX_FANOUT][32];  // positions, [rank][column lane]
  int64_t coff[32];
  int32_t pre[32];                // exclusive prefix of the chunk's counts
  float csum[32];                 // PASS column sums
  int32_t cnt_all[32];            // count; bit 30: positions are 0..cnt-1
};

__device__ __forceinline__ int pow2ceil_int(int k) { return k <= 1 ? 1 : 1 << (32 - __clz(k - 1)); }

__device__ __forceinline__ int log2_pow2ceil64(int64_t x) {
  int l = 0;
  while ((1ll << l) < x) ++l;
  return l;
}

__device__ __forceinline__ uint32_t sel_word(const U4& r, int i) {
  return i == 0 ? r.x : (i == 1 ? r.y : (i == 2 ? r.z : r.w));
}

// Warp-level exclusive scan of an int; *total = warp sum.
__device__ __forceinline__ int warp_excl(int v, int* total) {
  const int lane = threadIdx.x & 31;
  int inc = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int n = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += n;
  }
  *total = __shfl_sync(0xffffffffu, inc, 31);
  return inc - v;
}

// Last column c of the chunk with pre[c] <= f (the column holding flat slot f).
__device__ __forceinline__ int chunk_col(const int32_t* pre, int f) {
  int lo = 0, hi = 31;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (pre[mid] <= f) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

// A-Res top-k for the chunk's columns (R6): groups of G = pow2ceil(k) lanes
// stream a column's weights, keep the k smallest (key, position), and write
// the selected positions (ascending) into list[.][c] and the count into
// cnt_all[c]; csum[c] = fp32(sum_fp64 w over the whole column) (PASS A3).
template <typename Out>
__device__ inline void ares_chunk_t(const NWCore& P, Out out, int l, uint32_t gb, int k,
                                    int32_t my_v, bool my_valid, int64_t my_off, int64_t my_d) {
  const int G = pow2ceil_int(k);
  const int lane = threadIdx.x & 31;
  const int s = lane & (G - 1), gbase = lane & ~(G - 1);
  const int gpw = 32 / G;
  const uint32_t FULL = 0xffffffffu;
  const uint32_t gbits = (G == 32) ? FULL : (((1u << G) - 1u) << gbase);
  for (int cb = 0; cb < 32; cb += gpw) {
    const int c = cb + lane / G;
    const int32_t v = __shfl_sync(FULL, my_v, c);
    const bool valid = __shfl_sync(FULL, my_valid ? 1 : 0, c) != 0;
    const int64_t off = __shfl_sync(FULL, my_off, c);
    const int64_t dsh = __shfl_sync(FULL, my_d, c);
    const int64_t d = valid ? dsh : 0;
    double bk = INFINITY, mk = INFINITY, csum = 0.0;
    int64_t bp = INT64_MAX, mp = INT64_MAX;
    int ml = 0;
    int rounds = valid ? (int)((d + G - 1) / G) : 0;
    rounds = (int)__reduce_max_sync(FULL, (unsigned)rounds);
    for (int rd = 0; rd < rounds; ++rd) {
      const int64_t i = (int64_t)rd * G + s;
      const bool in = valid && i < d;
      const float w = in ? (P.weights ? __ldg(P.weights + off + i) : 1.0f) : 0.0f;
      csum += in ? (double)w : 0.0;
      const bool elig = in && w > 0.0f;
      double kk = INFINITY;
      if (elig) {
        const U4 r = philox((uint32_t)v, (uint32_t)(i >> 2), ctr2(l, TAG_ARES_NODE), gb, P.key);
        kk = ares_key(sel_word(r, (int)(i & 3)), (double)w);
      }
      uint32_t cand = __ballot_sync(FULL, elig && key_less(kk, i, mk, mp)) & gbits;
      while (__any_sync(FULL, cand != 0u)) {
        const int cl = cand ? (__ffs(cand) - 1) : 0;
        const double ck = __shfl_sync(FULL, kk, cl);
        const int64_t cp = __shfl_sync(FULL, i, cl);
        const bool ins = cand != 0u && key_less(ck, cp, mk, mp);
        if (ins && s == ml) {
          bk = ck;
          bp = cp;
        }
        if (cand) cand &= cand - 1u;
        // new group maximum over the k held entries: (key, pos, lane) lexicographic
        double tk = (s < k) ? bk : -INFINITY;
        int64_t tp = (s < k) ? bp : -1;
        int tl = s;
        for (int o = G >> 1; o > 0; o >>= 1) {
          const double ok = __shfl_xor_sync(FULL, tk, o);
          const int64_t op = __shfl_xor_sync(FULL, tp, o);
          const int ol = __shfl_xor_sync(FULL, tl, o);
          if (key_less(tk, tp, ok, op) || (tk == ok && tp == op && ol > tl)) {
            tk = ok;
            tp = op;
            tl = ol;
          }
        }
        if (ins) {
          mk = tk;
          mp = tp;
          ml = tl;
        }
      }
    }
    const bool sel = s < k && bp != INT64_MAX;
    const uint32_t selb = __ballot_sync(FULL, sel) & gbits;
    int rnk = 0;
    for (int i = 0; i < G; ++i) {
      const int64_t pi = __shfl_sync(FULL, bp, gbase + i);
      rnk += (((selb >> (gbase + i)) & 1u) && pi < bp) ? 1 : 0;
    }
    for (int o = G >> 1; o > 0; o >>= 1) csum += __shfl_xor_sync(FULL, csum, o);
    if (sel) out.pos(c, rnk, (uint32_t)bp);
    if (s == 0) out.col(c, __popc(selb), (float)csum);
  }
  __syncwarp();
}

struct ChunkOut {
  WarpChunk* C;
  __device__ void pos(int c, int r, uint32_t v) const { C->list[r][c] = v; }
  __device__ void col(int c, int cnt, float cs) const {
    C->cnt_all[c] = cnt;
    C->csum[c] = cs;
  }
};
__device__ inline void ares_chunk(const NWCore& P, WarpChunk& C, int l, uint32_t gb, int k,
                                  int32_t my_v, bool my_valid, int64_t my_off, int64_t my_d) {
  ares_chunk_t(P, ChunkOut{&C}, l, gb, k, my_v, my_valid, my_off, my_d);
}

// Select for one warp chunk of up to 32 columns [jb, min(jb + 32, jend)) of
// frontier F (batch-local column j -> padded slots j*k .. j*k+k-1), stage the
// sampled edges and insert every (u, slot) into the ordered hash (first
// occurrence = minimum slot; kFixed: fixed-position CAS table, safe for
// lookups concurrent with later inserts).  Returns the chunk's edge count (warp-uniform);
// C.pre / C.cnt_all describe the chunk afterwards.
template <bool kFixed = false>
__device__ inline int select_chunk(const NWCore& P, const NWStage& W, WarpChunk& C, int l, int k,
                                   int log_cap, uint32_t tag, const int32_t* F, int64_t jb,
                                   int64_t jend, uint32_t gb, unsigned long long* dbg = nullptr) {
  const int lane = threadIdx.x & 31;
  const uint64_t pf = pol_first(), pl = pol_last();
  const int64_t j = jb + lane;
  const bool active = j < jend;
  const int32_t v = active ? (kFixed ? ldh(F + j, pl) : __ldcg(F + j)) : -1;
  const bool valid = active && v >= 0 && (int64_t)v < P.N;
  if (active && !valid) atomicOr(P.err, ERR_SEED_RANGE);
  int64_t off = 0, d = 0;
  if (valid) {
    off = __ldg(P.indptr + v);
    d = __ldg(P.indptr + v + 1) - off;
  }
  int cnt = 0;
  bool all = false;
  const bool weighted = !P.replace && P.bias != GS_W_UNIFORM;
  if (dbg && lane == 0) {
    unsigned long long tt;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(tt));
    dbg[0] = tt + (unsigned long long)(d & 0);
  }
  if (weighted) {
    ares_chunk(P, C, l, gb, k, v, valid, off, d);
    cnt = C.cnt_all[lane];
  } else if (P.replace) {
    // KGCN (R10): k i.i.d. uniform positions in slot order.
    cnt = d > 0 ? k : 0;
    for (int s = 0; s < cnt; ++s) {
      const U4 r = philox((uint32_t)v, (uint32_t)s, ctr2(l, TAG_REPLACE), gb, P.key);
      C.list[s][lane] = (uint32_t)draw_below((uint64_t)d, r.x, r.y);
    }
  } else if (d <= k) {
    // GraphSAGE, d <= k: every neighbour, no randomness (R5)
    cnt = (int)d;
    all = true;
  } else {
    // GraphSAGE (R5): Floyd's algorithm; the list is kept sorted (m exceeds
    // every element chosen so far, so it is appended).
    cnt = k;
    int n = 0;
    for (int s = 0; s < k; ++s) {
      const U4 r = philox((uint32_t)v, (uint32_t)s, ctr2(l, TAG_FLOYD), gb, P.key);
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
  if (dbg && lane == 0) {
    unsigned long long tt;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(tt));
    dbg[1] = tt;
  }
  C.coff[lane] = off;
  C.pre[lane] = pre;
  if (!weighted) C.cnt_all[lane] = cnt | (all ? (1 << 30) : 0);
  if (active) {
    if (kFixed) {
      sth(W.coff + j, off, pl);
      sth(W.ccnt + j, cnt, pl);
    } else {
      W.coff[j] = off;
      W.ccnt[j] = cnt;
    }
  }
  __syncwarp();
  // Flattened gather + stage + insert: flat slot f of the chunk -> column c, rank s.
  const uint32_t mask = (1u << log_cap) - 1u;
  for (int f0 = 0; f0 < total; f0 += 32 * NW_ILP) {
    int32_t u[NW_ILP];
    int64_t p[NW_ILP];
    uint32_t ps[NW_ILP];
    int cc[NW_ILP];
    bool ok[NW_ILP];
#pragma unroll
    for (int i = 0; i < NW_ILP; ++i) {
      const int f = f0 + i * 32 + lane;
      ok[i] = f < total;
      cc[i] = 0;
      p[i] = 0;
      ps[i] = 0;
      u[i] = 0;
      if (ok[i]) {
        const int c = chunk_col(C.pre, f);
        const int s = f - C.pre[c];
        ps[i] = (C.cnt_all[c] & (1 << 30)) ? (uint32_t)s : C.list[s][c];
        p[i] = (jb + c) * k + s;
        u[i] = kFixed ? ldg_h(P.indices + C.coff[c] + ps[i], pf)
                      : __ldg(P.indices + C.coff[c] + ps[i]);
        cc[i] = c;
      }
    }
    unsigned long long old[NW_ILP], carry[NW_ILP];
    uint32_t h[NW_ILP];
#pragma unroll
    for (int i = 0; i < NW_ILP; ++i) {
      h[i] = 0;
      carry[i] = 0;
      if (ok[i]) {
        if (kFixed) {
          sth(W.u + p[i], u[i], pl);
          sth(W.pos + p[i], ps[i], pl);
        } else {
          W.u[p[i]] = u[i];
          W.pos[p[i]] = ps[i];
        }
        if (W.val) {
          const float w = P.weights ? __ldg(P.weights + C.coff[cc[i]] + ps[i]) : 1.0f;
          W.val[p[i]] = w / C.csum[cc[i]];
        }
        h[i] = tab_hash((uint32_t)u[i], log_cap);
        carry[i] = kFixed ? ct_entry((uint32_t)u[i], (uint32_t)p[i])
                          : tab_entry(tag, (uint32_t)u[i], (uint32_t)p[i]);
      }
    }
    if (kFixed) {
      // Hot rows (hubs) recur in many columns: a CAS per occurrence would
      // serialise on one L2 address.  Only the first occurrence inside the
      // warp (lowest lane = smallest slot) proceeds, and it first reads the
      // home slot: a row already holding a smaller slot needs no atomic.
      bool go[NW_ILP];
#pragma unroll
      for (int i = 0; i < NW_ILP; ++i) {
        const uint32_t peers = __match_any_sync(0xffffffffu, ok[i] ? (uint32_t)u[i] : 0xFFFFFFFFu);
        go[i] = ok[i] && (__ffs(peers) - 1) == lane;
        old[i] = go[i] ? ldh(&W.tab[h[i]], pl) : 0ull;
      }
#pragma unroll
      for (int i = 0; i < NW_ILP; ++i) {
        if (!go[i]) continue;
        if (old[i] != CT_EMPTY && (old[i] >> TAB_VAL_BITS) == (carry[i] >> TAB_VAL_BITS) &&
            old[i] <= carry[i]) {
          go[i] = false;  // present with an earlier slot
          continue;
        }
        old[i] = atom_cas_h(&W.tab[h[i]], CT_EMPTY, carry[i], pl);
      }
#pragma unroll
      for (int i = 0; i < NW_ILP; ++i)
        if (go[i]) ct_finish(W.tab, mask, h[i], carry[i], old[i], pl);
    } else {
#pragma unroll
      for (int i = 0; i < NW_ILP; ++i)
        if (ok[i]) old[i] = atomicMin(&W.tab[h[i]], carry[i]);
#pragma unroll
      for (int i = 0; i < NW_ILP; ++i)
        if (ok[i]) otab_finish(W.tab, mask, tag, h[i], carry[i], old[i]);
    }
  }
  __syncwarp();
  if (dbg && lane == 0) {
    unsigned long long tt;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(tt));
    dbg[2] = tt;
  }
  return total;
}

}  // namespace gsb
