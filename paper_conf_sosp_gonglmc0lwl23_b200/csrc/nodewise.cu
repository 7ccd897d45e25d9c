// nodewise.cu -- node-wise ECSF sampling (GraphSAGE, KGCN, weighted A-Res,
// PASS-style A3 probabilities) and the ShaDow induced subgraph, as ONE
// persistent thread-block-cluster kernel per call.
//
// Design:
//   * one cluster (CS CTAs) owns one mini-batch at a time (super-batch):
//     every hop of the batch -- Extract, Select and
//     Finalize -- runs inside the cluster, separated by cluster
//     barriers, so per-batch state (hash table, slot staging) stays in L2 and
//     the epoch needs no host synchronisation and one launch;
//   * P1 select: a group of G = pow2ceil(k) lanes per frontier column
//     (Extract-Select fusion): gather the indptr pair, draw positions
//     (Floyd / with replacement / A-Res top-k), gather the sampled rows, stage
//     (u, eid) in padded slots [T][k] and insert (u, slot) into a
//     generation-tagged hash keeping the minimum slot (first occurrence);
//   * P2 finalize-1, slot-parallel: first-occurrence flag, CTA scan of
//     (valid, first) -> CTA-local edge index and local row id;
//   * P3 finalize-2, slot-parallel: cluster offsets from DSMEM totals,
//     relabel, compaction into the block (CSC indptr + COO row_local/eid) and
//     row_map (A.row(), next frontier).
#include <cooperative_groups.h>
#include <algorithm>
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include "common.cuh"
#include "gs_internal.h"

namespace cg = cooperative_groups;

namespace gsb {

struct NWParams {
  const int64_t* indptr;
  const int32_t* indices;
  const float* weights;
  int64_t N;
  const int32_t* seeds;
  int64_t num_seeds, batch_size, num_batches, batch_base;
  int L;
  int k[MAX_LAYERS];
  int64_t K[MAX_LAYERS];  // prod k[0..l]
  int replace, bias;
  uint64_t key;
  // outputs (row_local/eid/indptr may be NULL: ShaDow keeps only row_map)
  int32_t* col0;
  int32_t* row_map[MAX_LAYERS];
  int64_t* indptr_out[MAX_LAYERS];
  int32_t* row_local[MAX_LAYERS];
  int64_t* eid[MAX_LAYERS];
  float* val[MAX_LAYERS];
  int64_t* meta;  // [num_batches][meta_layers][8]
  int meta_layers;
  int* err;
  // per-cluster workspace
  char* ws;
  int64_t ws_stride;
  int64_t o_u, o_e, o_p0, o_lid, o_eidx, o_val, o_cnt, o_eoff, o_tab;
  int log_tab_cap;
  uint32_t* gen;
  // ShaDow: induced subgraph on U
  int shadow;
  int64_t sh_stride;  // 1 + sum K[l]: node capacity per seed
  int32_t* sh_nodes;
  int64_t* sh_indptr;
  int32_t* sh_row_local;
  int64_t* sh_eid;
  int64_t sh_edge_cap;
  unsigned long long* sh_edge_ctr;
};

struct Ws {
  int32_t* u;
  int64_t* e;
  int32_t* p0;
  int32_t* lid;
  int32_t* eidx;
  float* val;
  int32_t* cnt;
  int32_t* eoff;
  unsigned long long* tab;
};

__device__ __forceinline__ int pow2ceil_int(int k) { return k <= 1 ? 1 : 1 << (32 - __clz(k - 1)); }

__device__ __forceinline__ int log2_pow2ceil64(int64_t x) {
  int l = 0;
  while ((1ll << l) < x) ++l;
  return l;
}

// next generation tag 1..255; returns true when the table must be cleared.
__device__ __forceinline__ bool next_gen(uint32_t& gen) {
  bool wrap = (gen == 255u);
  gen = (gen % 255u) + 1u;
  return wrap;
}

template <int CS>
__device__ void clear_table(const NWParams& P, Ws& W, int crank) {
  const int64_t cap = 1ll << P.log_tab_cap;
  for (int64_t i = (int64_t)crank * blockDim.x + threadIdx.x; i < cap; i += (int64_t)CS * blockDim.x)
    W.tab[i] = 0ull;
}

__device__ __forceinline__ uint32_t sel_word(const U4& r, int i) {
  return i == 0 ? r.x : (i == 1 ? r.y : (i == 2 ? r.z : r.w));
}

// ---------------------------------------------------------------------------
// P1: select for the columns [c0, c1) of frontier F (batch-local indices).
// ---------------------------------------------------------------------------
__device__ void nw_select(const NWParams& P, Ws& W, int l, int log_cap, uint32_t gen,
                          const int32_t* F, int64_t c0, int64_t c1, uint32_t gb) {
  const int k = P.k[l];
  const int G = pow2ceil_int(k);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
  const int s = lane & (G - 1), gbase = lane & ~(G - 1);
  const uint32_t gbits = (G == 32) ? 0xffffffffu : (((1u << G) - 1u) << gbase);
  const int gpw = 32 / G;
  const uint32_t FULL = 0xffffffffu;
  const int64_t N = P.N;
  const bool weighted_sel = !P.replace && P.bias != GS_W_UNIFORM;

  for (int64_t jb = c0 + (int64_t)warp * gpw; jb < c1; jb += (int64_t)nwarps * gpw) {
    const int64_t j = jb + lane / G;
    const bool active = j < c1;
    int32_t v = active ? __ldcg(F + j) : 0;
    const bool valid = active && v >= 0 && (int64_t)v < N;
    if (active && !valid && s == 0) atomicOr(P.err, ERR_SEED_RANGE);
    int64_t off = 0, d = 0;
    if (valid) {
      off = __ldg(P.indptr + v);
      d = __ldg(P.indptr + v + 1) - off;
    }
    int cnt = 0;
    int64_t pos = 0;
    int slot = s;
    float pval = 0.f;

    if (P.replace) {
      // KGCN (R10): k i.i.d. uniform positions, slot order.
      cnt = d > 0 ? k : 0;
      if (s < cnt) {
        U4 r = philox((uint32_t)v, (uint32_t)s, ctr2(l, TAG_REPLACE), gb, P.key);
        pos = (int64_t)draw_below((uint64_t)d, r.x, r.y);
      }
    } else if (!weighted_sel) {
      // GraphSAGE (R5): d <= k -> all positions; else Floyd, positions ascending.
      const bool need = valid && d > k;
      cnt = (int)(d < k ? d : k);
      pos = s;
      if (__ballot_sync(FULL, need)) {
        const int64_t m = d - k + s;
        int64_t t = 0;
        if (need && s < k) {
          U4 r = philox((uint32_t)v, (uint32_t)s, ctr2(l, TAG_FLOYD), gb, P.key);
          t = (int64_t)draw_below((uint64_t)(m + 1), r.x, r.y);
        }
        int64_t x = -1;
        for (int i = 0; i < k; ++i) {
          const int64_t ti = __shfl_sync(FULL, t, gbase + i);
          const uint32_t b = __ballot_sync(FULL, s < i && x == ti) & gbits;
          if (s == i) x = b ? m : t;
        }
        int rnk = 0;
        for (int i = 0; i < k; ++i) {
          const int64_t xi = __shfl_sync(FULL, x, gbase + i);
          rnk += (xi < x) ? 1 : 0;
        }
        if (need) {
          pos = x;
          slot = s < k ? rnk : k;  // lanes beyond k (G > k) hold nothing
        }
      }
    } else {
      // Weighted without replacement (R6): the k smallest A-Res keys over the
      // eligible positions (w > 0), ties -> smaller position.
      double bk = INFINITY;
      int64_t bp = INT64_MAX;
      double mk = INFINITY;
      int64_t mp = INT64_MAX;
      int ml = 0;
      double csum = 0.0;
      int rounds = valid ? (int)((d + G - 1) / G) : 0;
      rounds = __reduce_max_sync(FULL, (unsigned)rounds);
      for (int rd = 0; rd < rounds; ++rd) {
        const int64_t i = (int64_t)rd * G + s;
        const bool in = valid && i < d;
        const float w = in ? (P.weights ? __ldg(P.weights + off + i) : 1.0f) : 0.0f;
        csum += in ? (double)w : 0.0;
        const bool elig = in && w > 0.0f;
        double kk = INFINITY;
        if (elig) {
          U4 r = philox((uint32_t)v, (uint32_t)(i >> 2), ctr2(l, TAG_ARES_NODE), gb, P.key);
          kk = ares_key(sel_word(r, (int)(i & 3)), (double)w);
        }
        uint32_t cand = __ballot_sync(FULL, elig && key_less(kk, i, mk, mp)) & gbits;
        while (__any_sync(FULL, cand != 0u)) {
          const int c = cand ? (__ffs(cand) - 1) : 0;
          const double ck = __shfl_sync(FULL, kk, c);
          const int64_t cp = __shfl_sync(FULL, i, c);
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
            const bool other_bigger = key_less(tk, tp, ok, op) || (tk == ok && tp == op && ol > tl);
            if (other_bigger) {
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
      cnt = __popc(selb);
      int rnk = 0;
      for (int i = 0; i < G; ++i) {
        const int64_t pi = __shfl_sync(FULL, bp, gbase + i);
        const bool si = (selb >> (gbase + i)) & 1u;
        rnk += (si && pi < bp) ? 1 : 0;
      }
      pos = bp;
      slot = rnk;
      if (P.bias == GS_W_PASS_COLNORM) {
        for (int o = G >> 1; o > 0; o >>= 1) csum += __shfl_xor_sync(FULL, csum, o);
        if (sel) {
          const float w = P.weights ? __ldg(P.weights + off + bp) : 1.0f;
          pval = w / (float)csum;
        }
      }
      if (!sel) slot = k;  // not taken
    }

    // Stage the sampled edges and insert their rows (first slot wins).
    if (valid && slot < cnt) {
      const int64_t e = off + pos;
      const int32_t u = __ldg(P.indices + e);
      const int64_t p = j * k + slot;
      W.u[p] = u;
      W.e[p] = e;
      if (W.val) W.val[p] = pval;
      tab_insert_min(W.tab, log_cap, gen, (uint32_t)u, (uint32_t)p);
    }
    if (active && s == 0) W.cnt[j] = valid ? cnt : 0;
  }
}

// ---------------------------------------------------------------------------
// ShaDow induce for batch b (R12).
// Z = seeds ++ row_map_0 ++ ... ++ row_map_{L-1}; U = first-occurrence unique
// of Z; block = every edge u -> v of A with u, v in U, columns in U order.
//   S1 insert (Z[z], z) keeping the minimum z;  S2 first flags + CTA scan;
//   S3 write U and replace each entry's value by the local id;
//   S4 warp-per-column count of in-U rows + CTA scan;  S5 emit.
// ---------------------------------------------------------------------------
template <int CS>
__device__ void shadow_induce(const NWParams& P, Ws& W, cg::cluster_group& cluster, int crank,
                              int64_t b, int64_t bstart, int64_t nb, const int64_t* rows_l,
                              uint32_t gen, unsigned long long* s_scan, unsigned long long* s_tot,
                              long long* s_base_e, long long* s_base_r) {
  __shared__ long long s_ebase;
  // segment starts of Z
  int64_t seg_start[MAX_LAYERS + 2];
  seg_start[0] = 0;
  seg_start[1] = nb;
  for (int l = 0; l < P.L; ++l) seg_start[l + 2] = seg_start[l + 1] + rows_l[l];
  const int64_t Zn = seg_start[P.L + 1];
  auto zval = [&](int64_t z) -> uint32_t {
    if (z < nb) return (uint32_t)__ldcg(P.seeds + bstart + z);
    int l = 0;
    while (z >= seg_start[l + 2]) ++l;
    return (uint32_t)__ldcg(P.row_map[l] + bstart * P.K[l] + (z - seg_start[l + 1]));
  };
  int log_cap = log2_pow2ceil64((Zn * 4) / 3 + 64);
  if (log_cap > P.log_tab_cap) log_cap = P.log_tab_cap;
  const int64_t zchunk = (Zn + CS - 1) / CS;
  const int64_t z0 = min(Zn, (int64_t)crank * zchunk), z1 = min(Zn, z0 + zchunk);
  const int64_t ubase = bstart * P.sh_stride;
  const int64_t uibase = ubase + b;

  // S1
  for (int64_t z = z0 + threadIdx.x; z < z1; z += blockDim.x)
    tab_insert_min(W.tab, log_cap, gen, zval(z), (uint32_t)z);
  cluster.sync();
  // S2
  unsigned long long carry = 0;
  for (int64_t zt = z0; zt < z1; zt += blockDim.x) {
    const int64_t z = zt + threadIdx.x;
    bool first = false;
    if (z < z1) {
      const int64_t h = tab_find(W.tab, log_cap, gen, zval(z));
      first = tab_val(__ldcg(W.tab + h)) == (uint32_t)z;
    }
    unsigned long long tot;
    const unsigned long long ex = block_exclusive_scan((unsigned long long)(first ? 1 : 0), s_scan, &tot) + carry;
    if (first) W.lid[z] = (int32_t)ex;
    carry += tot;
  }
  if (threadIdx.x == 0) *s_tot = carry;
  cluster.sync();
  if (threadIdx.x == 0) {
    long long a = 0;
    for (int r = 0; r < CS; ++r) {
      s_base_r[r] = a;
      a += (long long)*cluster.map_shared_rank(s_tot, r);
    }
    s_base_r[CS] = a;
  }
  __syncthreads();
  const int64_t nU = s_base_r[CS];
  // S3
  for (int64_t z = z0 + threadIdx.x; z < z1; z += blockDim.x) {
    const uint32_t u = zval(z);
    const int64_t h = tab_find(W.tab, log_cap, gen, u);
    if (tab_val(__ldcg(W.tab + h)) == (uint32_t)z) {
      const int64_t lid = s_base_r[crank] + __ldcg(W.lid + z);
      P.sh_nodes[ubase + lid] = (int32_t)u;
      W.tab[h] = tab_entry(gen, u, (uint32_t)lid);
    }
  }
  cluster.sync();
  // S4: count in-U rows of every column of U (warp per column)
  const int64_t uchunk = (nU + CS - 1) / CS;
  const int64_t u0 = min(nU, (int64_t)crank * uchunk), u1 = min(nU, u0 + uchunk);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
  for (int64_t c = u0 + warp; c < u1; c += nwarps) {
    const int32_t v = __ldcg(P.sh_nodes + ubase + c);
    const int64_t off = __ldg(P.indptr + v), d = __ldg(P.indptr + v + 1) - off;
    int cnt = 0;
    for (int64_t i = lane; i < d; i += 32) {
      const uint32_t u = (uint32_t)__ldg(P.indices + off + i);
      cnt += tab_find(W.tab, log_cap, gen, u) >= 0 ? 1 : 0;
    }
    cnt = __reduce_add_sync(0xffffffffu, (unsigned)cnt);
    if (lane == 0) W.cnt[c] = cnt;
  }
  __syncthreads();
  carry = 0;
  for (int64_t ct = u0; ct < u1; ct += blockDim.x) {
    const int64_t c = ct + threadIdx.x;
    const unsigned long long cv = c < u1 ? (unsigned long long)__ldcg(W.cnt + c) : 0ull;
    unsigned long long tot;
    const unsigned long long ex = block_exclusive_scan(cv, s_scan, &tot) + carry;
    if (c < u1) W.eoff[c] = (int32_t)ex;
    carry += tot;
  }
  if (threadIdx.x == 0) *s_tot = carry;
  cluster.sync();
  if (threadIdx.x == 0) {
    long long a = 0;
    for (int r = 0; r < CS; ++r) {
      s_base_e[r] = a;
      a += (long long)*cluster.map_shared_rank(s_tot, r);
    }
    s_base_e[CS] = a;
    if (crank == 0) s_ebase = (long long)atomicAdd(P.sh_edge_ctr, (unsigned long long)a);
  }
  cluster.sync();
  if (threadIdx.x == 0) s_ebase = *cluster.map_shared_rank(&s_ebase, 0);
  __syncthreads();
  const int64_t nE = s_base_e[CS];
  const int64_t ebase = s_ebase;
  const bool fits = ebase + nE <= P.sh_edge_cap;
  if (!fits && crank == 0 && threadIdx.x == 0) atomicOr(P.err, ERR_CAPACITY);
  // S5: emit (warp per column, ballot compaction keeps CSC order)
  for (int64_t c = u0 + warp; c < u1; c += nwarps) {
    const int32_t v = __ldcg(P.sh_nodes + ubase + c);
    const int64_t off = __ldg(P.indptr + v), d = __ldg(P.indptr + v + 1) - off;
    int64_t e = s_base_e[crank] + __ldcg(W.eoff + c);
    if (lane == 0) P.sh_indptr[uibase + c] = e;
    if (!fits) continue;
    for (int64_t i0 = 0; i0 < d; i0 += 32) {
      const int64_t i = i0 + lane;
      int64_t h = -1;
      uint32_t u = 0;
      if (i < d) {
        u = (uint32_t)__ldg(P.indices + off + i);
        h = tab_find(W.tab, log_cap, gen, u);
      }
      const uint32_t m = __ballot_sync(0xffffffffu, h >= 0);
      if (h >= 0) {
        const int64_t o = ebase + e + __popc(m & ((1u << lane) - 1u));
        P.sh_row_local[o] = (int32_t)tab_val(__ldcg(W.tab + h));
        P.sh_eid[o] = off + i;
      }
      e += __popc(m);
    }
  }
  if (crank == 0 && threadIdx.x == 0) {
    P.sh_indptr[uibase + nU] = nE;
    long long* m = (long long*)(P.meta + b * 8);
    m[0] = nU; m[1] = nU; m[2] = nE; m[3] = ubase; m[4] = ubase; m[5] = uibase; m[6] = ebase;
    m[7] = 0;
  }
  cluster.sync();
}

// ---------------------------------------------------------------------------
// The kernel: one cluster per batch, all hops (and the ShaDow induce) inside.
// ---------------------------------------------------------------------------
template <int CS>
__global__ void __launch_bounds__(512, 2) nodewise_kernel(NWParams P) {
  cg::cluster_group cluster = cg::this_cluster();
  const int crank = (int)cluster.block_rank();
  const int64_t cid = blockIdx.x / CS;
  const int64_t nclusters = gridDim.x / CS;

  __shared__ unsigned long long s_scan[33];
  __shared__ unsigned long long s_tot;        // this CTA: (edges << 32) | rows
  __shared__ long long s_base_e[CS + 1], s_base_r[CS + 1];

  Ws W;
  char* base = P.ws + cid * P.ws_stride;
  W.u = (int32_t*)(base + P.o_u);
  W.e = (int64_t*)(base + P.o_e);
  W.p0 = (int32_t*)(base + P.o_p0);
  W.lid = (int32_t*)(base + P.o_lid);
  W.eidx = (int32_t*)(base + P.o_eidx);
  W.val = P.o_val >= 0 ? (float*)(base + P.o_val) : nullptr;
  W.cnt = (int32_t*)(base + P.o_cnt);
  W.eoff = (int32_t*)(base + P.o_eoff);
  W.tab = (unsigned long long*)(base + P.o_tab);

  uint32_t gen = P.gen[cid];

  for (int64_t b = cid; b < P.num_batches; b += nclusters) {
    const int64_t bstart = b * P.batch_size;
    const int64_t nb = min(P.batch_size, P.num_seeds - bstart);
    const uint32_t gb = (uint32_t)(P.batch_base + b);
    const int32_t* F = P.seeds + bstart;
    int64_t T = nb;
    int64_t colbase = bstart;      // region of this layer's columns
    int64_t rows_l[MAX_LAYERS];

    for (int l = 0; l < P.L; ++l) {
      const int k = P.k[l];
      const int64_t rbase = bstart * P.K[l];
      const int64_t ibase = colbase + b;
      if (next_gen(gen)) {
        clear_table<CS>(P, W, crank);
        cluster.sync();
      }
      int64_t want = (T * k * 4) / 3 + 64;
      int log_cap = log2_pow2ceil64(want);
      if (log_cap > P.log_tab_cap) log_cap = P.log_tab_cap;
      const int64_t chunk = (T + CS - 1) / CS;
      const int64_t c0 = min(T, (int64_t)crank * chunk), c1 = min(T, c0 + chunk);

      // ---- P1: select + insert ----
      nw_select(P, W, l, log_cap, gen, F, c0, c1, gb);
      cluster.sync();

      // ---- P2: first-occurrence flags, CTA scan over slots ----
      unsigned long long carry = 0;
      const int64_t p_lo = c0 * k, p_hi = c1 * k;
      for (int64_t pt = p_lo; pt < p_hi; pt += blockDim.x) {
        const int64_t p = pt + threadIdx.x;
        bool valid = false, first = false;
        int64_t j = 0;
        int s = 0;
        if (p < p_hi) {
          j = p / k;
          s = (int)(p - j * k);
          valid = s < __ldcg(W.cnt + j);
          if (valid) {
            const uint32_t u = (uint32_t)__ldcg(W.u + p);
            const int64_t h = tab_find(W.tab, log_cap, gen, u);
            if (h < 0) atomicOr(P.err, ERR_INTERNAL);
            const uint32_t p0 = h < 0 ? 0xffffffffu : tab_val(__ldcg(W.tab + h));
            W.p0[p] = (int32_t)p0;
            first = (p0 == (uint32_t)p);
          }
        }
        const unsigned long long packed = ((unsigned long long)(valid ? 1 : 0) << 32) | (first ? 1ull : 0ull);
        unsigned long long tot;
        const unsigned long long ex = block_exclusive_scan(packed, s_scan, &tot) + carry;
        if (p < p_hi) {
          if (s == 0) W.eoff[j] = (int32_t)(ex >> 32);
          if (valid) W.eidx[p] = (int32_t)(ex >> 32);
          if (first) W.lid[p] = (int32_t)(ex & 0xffffffffu);
        }
        carry += tot;
      }
      if (threadIdx.x == 0) s_tot = carry;
      cluster.sync();

      // ---- P3: cluster offsets, relabel, compaction ----
      if (threadIdx.x == 0) {
        long long ae = 0, ar = 0;
        for (int r = 0; r < CS; ++r) {
          s_base_e[r] = ae;
          s_base_r[r] = ar;
          const unsigned long long t = *cluster.map_shared_rank(&s_tot, r);
          ae += (long long)(t >> 32);
          ar += (long long)(t & 0xffffffffu);
        }
        s_base_e[CS] = ae;
        s_base_r[CS] = ar;
      }
      __syncthreads();
      const int64_t baseE = s_base_e[crank], baseR = s_base_r[crank];
      const int64_t totE = s_base_e[CS], totR = s_base_r[CS];
      int32_t* row_map = P.row_map[l];
      int32_t* row_local = P.row_local[l];
      int64_t* eid_out = P.eid[l];
      float* val_out = P.val[l];
      int64_t* indptr_out = P.indptr_out[l];
      for (int64_t pt = p_lo; pt < p_hi; pt += blockDim.x) {
        const int64_t p = pt + threadIdx.x;
        if (p >= p_hi) continue;
        const int64_t j = p / k;
        const int s = (int)(p - j * k);
        if (s == 0) {
          if (indptr_out) indptr_out[ibase + j] = baseE + __ldcg(W.eoff + j);
          if (l == 0 && P.col0) P.col0[bstart + j] = F[j];
        }
        if (s >= __ldcg(W.cnt + j)) continue;
        const int32_t p0 = __ldcg(W.p0 + p);
        int64_t lid;
        if (p0 == (int32_t)p) {
          lid = baseR + __ldcg(W.lid + p);
          row_map[rbase + lid] = __ldcg(W.u + p);
        } else {
          const int64_t j0 = p0 / k;
          const int r0 = (int)(j0 / chunk);
          lid = s_base_r[r0] + __ldcg(W.lid + p0);
        }
        const int64_t e = rbase + baseE + __ldcg(W.eidx + p);
        if (row_local) row_local[e] = (int32_t)lid;
        if (eid_out) eid_out[e] = __ldcg(W.e + p);
        if (val_out) val_out[e] = __ldcg(W.val + p);
      }
      if (crank == 0 && threadIdx.x == 0) {
        if (indptr_out) indptr_out[ibase + T] = totE;
        if (!P.shadow) {
          long long* m = (long long*)(P.meta + (b * P.meta_layers + l) * 8);
          m[0] = T; m[1] = totR; m[2] = totE; m[3] = colbase; m[4] = rbase; m[5] = ibase;
          m[6] = rbase; m[7] = 0;
        }
      }
      cluster.sync();
      F = row_map + rbase;
      T = totR;
      colbase = rbase;
      rows_l[l] = totR;
    }

    if (P.shadow) {
      if (next_gen(gen)) {
        clear_table<CS>(P, W, crank);
        cluster.sync();
      }
      shadow_induce<CS>(P, W, cluster, crank, b, bstart, nb, rows_l, gen, s_scan, &s_tot,
                        s_base_e, s_base_r);
    }
  }
  if (crank == 0 && threadIdx.x == 0) P.gen[cid] = gen;
}

}  // namespace gsb

// ---------------------------------------------------------------------------
// Host side
// ---------------------------------------------------------------------------
namespace gsb {

static int64_t align256(int64_t x) { return (x + 255) & ~int64_t(255); }

template <int CS>
static int max_active_clusters(int threads) {
  static int cached = -1;
  if (cached > 0) return cached;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(CS * 1024);
  cfg.blockDim = dim3(threads);
  cfg.dynamicSmemBytes = 0;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = CS;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, nodewise_kernel<CS>, &cfg) != cudaSuccess || n <= 0) {
    cudaGetLastError();
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    n = sms / CS;
  }
  cached = n;
  return n;
}

constexpr int NW_CS = 8;
constexpr int NW_THREADS = 512;
constexpr int MAX_CLUSTERS = 4096;

gs_status run_nodewise(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                       int64_t batch_size, int64_t batch_base, const int32_t* fanouts, int L,
                       int replace, int bias, uint64_t key, bool shadow, cudaStream_t stream,
                       gs_blocks* blk) {
  const Allocator& al = blk->al;
  NWParams P = {};
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
  P.replace = replace;
  P.bias = bias;
  P.key = key;
  int64_t prod = 1, sum_K = 0;
  int64_t slot_cap = 1, col_cap = 1;
  for (int l = 0; l < L; ++l) {
    P.k[l] = fanouts[l];
    col_cap = std::max(col_cap, batch_size * prod);
    prod *= fanouts[l];
    P.K[l] = prod;
    sum_K += prod;
    slot_cap = std::max(slot_cap, batch_size * prod);
  }
  P.shadow = shadow ? 1 : 0;
  P.sh_stride = 1 + sum_K;
  if (shadow) {
    slot_cap = std::max(slot_cap, batch_size * P.sh_stride);
    col_cap = std::max(col_cap, batch_size * P.sh_stride);
  }
  const int64_t nbatch = P.num_batches;
  blk->kind = shadow ? gs_blocks::SHADOW : gs_blocks::NODEWISE;
  blk->num_batches = nbatch;
  blk->num_layers = shadow ? 1 : L;
  blk->stream = stream;
  blk->synced = false;

  // ---- outputs ----
  auto need = [&](DevBuf& b, int64_t bytes) -> bool {
    return b.ensure(al, (size_t)std::max<int64_t>(bytes, 256), stream);
  };
  bool ok = need(blk->b_col[0], num_seeds * 4);
  for (int l = 0; l < L && ok; ++l) {
    const int64_t rows = num_seeds * P.K[l];
    const int64_t cols = num_seeds * (l == 0 ? 1 : P.K[l - 1]);
    ok = ok && need(blk->b_row[l], rows * 4);
    if (!shadow) {
      ok = ok && need(blk->b_indptr[l], (cols + nbatch) * 8) && need(blk->b_rowl[l], rows * 4) &&
           need(blk->b_eid[l], rows * 8);
      if (bias == GS_W_PASS_COLNORM) ok = ok && need(blk->b_val[l], rows * 4);
    }
  }
  int64_t sh_nodes = 0, sh_edges = 0;
  if (shadow && ok) {
    sh_nodes = num_seeds * P.sh_stride;
    sh_edges = std::max<int64_t>(std::max<int64_t>(int64_t(1) << 20, blk->sh_edge_hint), sh_nodes * 4);
    ok = need(blk->b_col[1], sh_nodes * 4) && need(blk->b_indptr[0], (sh_nodes + nbatch) * 8) &&
         need(blk->b_rowl[0], sh_edges * 4) && need(blk->b_eid[0], sh_edges * 8);
    sh_edges = (int64_t)std::min(blk->b_rowl[0].bytes / 4, blk->b_eid[0].bytes / 8);
  }
  const int meta_layers = shadow ? 1 : L;
  ok = ok && need(blk->b_meta, nbatch * meta_layers * 8 * 8) && need(blk->b_err, 16) &&
       need(blk->b_ctr, 16);
  if (!ok) return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (blocks buffers)");

  // ---- workspace (per cluster) ----
  int log_tab = 6;
  while ((int64_t(1) << log_tab) < (slot_cap * 4) / 3 + 64) ++log_tab;
  int64_t o = 0;
  P.o_u = o; o = align256(o + slot_cap * 4);
  P.o_e = o; o = align256(o + slot_cap * 8);
  P.o_p0 = o; o = align256(o + slot_cap * 4);
  P.o_lid = o; o = align256(o + slot_cap * 4);
  P.o_eidx = o; o = align256(o + slot_cap * 4);
  if (bias == GS_W_PASS_COLNORM && !shadow) {
    P.o_val = o;
    o = align256(o + slot_cap * 4);
  } else {
    P.o_val = -1;
  }
  P.o_cnt = o; o = align256(o + col_cap * 4);
  P.o_eoff = o; o = align256(o + col_cap * 4);
  P.o_tab = o; o = align256(o + (int64_t(8) << log_tab));
  P.ws_stride = o;
  P.log_tab_cap = log_tab;
  const int nclusters =
      (int)std::max<int64_t>(1, std::min<int64_t>(nbatch, max_active_clusters<NW_CS>(NW_THREADS)));
  const size_t ws_bytes = (size_t)P.ws_stride * nclusters;
  const bool grow = blk->b_ws.bytes < ws_bytes;
  if (!blk->b_ws.ensure(al, ws_bytes, stream, true) ||
      !blk->b_gen.ensure(al, MAX_CLUSTERS * 4, stream, true))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (workspace)");
  if (grow) {
    // a regrown workspace starts with an all-empty table: restart the tags
    GS_CUDA_TRY(cudaMemsetAsync(blk->b_gen.ptr, 0, MAX_CLUSTERS * 4, stream));
  } else if (blk->ws_stride_prev != P.ws_stride) {
    // the layout moved: old tags could alias inside the new table region
    GS_CUDA_TRY(cudaMemsetAsync(blk->b_ws.ptr, 0, blk->b_ws.bytes, stream));
    GS_CUDA_TRY(cudaMemsetAsync(blk->b_gen.ptr, 0, MAX_CLUSTERS * 4, stream));
  }
  blk->ws_stride_prev = P.ws_stride;
  P.ws = (char*)blk->b_ws.ptr;
  P.gen = (uint32_t*)blk->b_gen.ptr;

  // ---- layer views ----
  P.col0 = shadow ? nullptr : (int32_t*)blk->b_col[0].ptr;
  for (int l = 0; l < L; ++l) {
    P.row_map[l] = (int32_t*)blk->b_row[l].ptr;
    if (!shadow) {
      P.indptr_out[l] = (int64_t*)blk->b_indptr[l].ptr;
      P.row_local[l] = (int32_t*)blk->b_rowl[l].ptr;
      P.eid[l] = (int64_t*)blk->b_eid[l].ptr;
      P.val[l] = bias == GS_W_PASS_COLNORM ? (float*)blk->b_val[l].ptr : nullptr;
      gs_layer_buffers& lb = blk->layers[l];
      lb = gs_layer_buffers{};
      lb.col_map = l == 0 ? (int32_t*)blk->b_col[0].ptr : (int32_t*)blk->b_row[l - 1].ptr;
      lb.col_capacity = num_seeds * (l == 0 ? 1 : P.K[l - 1]);
      lb.row_map = P.row_map[l];
      lb.row_capacity = num_seeds * P.K[l];
      lb.indptr = P.indptr_out[l];
      lb.indptr_capacity = lb.col_capacity + nbatch;
      lb.row_local = P.row_local[l];
      lb.eid = P.eid[l];
      lb.val = P.val[l];
      lb.edge_capacity = num_seeds * P.K[l];
      lb.row_prob = nullptr;
    }
  }
  if (shadow) {
    P.sh_nodes = (int32_t*)blk->b_col[1].ptr;
    P.sh_indptr = (int64_t*)blk->b_indptr[0].ptr;
    P.sh_row_local = (int32_t*)blk->b_rowl[0].ptr;
    P.sh_eid = (int64_t*)blk->b_eid[0].ptr;
    P.sh_edge_cap = sh_edges;
    P.sh_edge_ctr = (unsigned long long*)blk->b_ctr.ptr;
    gs_layer_buffers& lb = blk->layers[0];
    lb = gs_layer_buffers{};
    lb.col_map = P.sh_nodes;
    lb.row_map = P.sh_nodes;
    lb.col_capacity = lb.row_capacity = sh_nodes;
    lb.indptr = P.sh_indptr;
    lb.indptr_capacity = sh_nodes + nbatch;
    lb.row_local = P.sh_row_local;
    lb.eid = P.sh_eid;
    lb.edge_capacity = sh_edges;
  }
  P.meta = (int64_t*)blk->b_meta.ptr;
  P.meta_layers = meta_layers;
  P.err = (int*)blk->b_err.ptr;
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_err.ptr, 0, 16, stream));
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_ctr.ptr, 0, 16, stream));
  if (nbatch == 0) return GS_OK;

  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(nclusters * NW_CS));
  cfg.blockDim = dim3(NW_THREADS);
  cfg.dynamicSmemBytes = 0;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = NW_CS;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  GS_CUDA_TRY(cudaLaunchKernelEx(&cfg, nodewise_kernel<NW_CS>, P));
  return GS_OK;
}

}  // namespace gsb
