// nodewise.cu -- node-wise ECSF sampling (GraphSAGE, KGCN, weighted A-Res,
// PASS-style A3 probabilities) and the ShaDow induced subgraph, as ONE
// persistent thread-block-cluster kernel per call (one launch per epoch).
//
// Design ("K-nodewise"):
//   * one cluster (8 CTAs x 1024 threads, one CTA per SM) owns one mini-batch
//     at a time (super-batch) and runs every hop of it -- Extract
//     (P:180), Select, Finalize -- with the
//     phases separated by cluster barriers, so a batch's hash table and slot
//     staging (~3 MB) stay in L2 and no host synchronisation is needed;
//   * every warp owns a contiguous range of frontier columns and works on
//     chunks of 32 columns (one per lane) with batched independent loads
//     (memory-level parallelism instead of per-column latency chains):
//       P1  Extract + Select: indptr pairs, positions (Floyd / replacement /
//           A-Res top-k) into shared memory, a flattened gather of the sampled
//           rows (NW_ILP loads in flight per lane), staging of (u, position)
//           and an ordered-hash atomicMin insert of (u, slot) -- Extract-Select
//           fusion;
//       P2  Finalize-1: first-occurrence bitmap over the batch's padded slots
//           (slot p is first iff the table holds p for its row) and per-word
//           prefix counts;
//       P3  Finalize-2: local id of every edge = rank of its row's first slot
//           (bitmap popcount), compaction into the block (CSC indptr + COO
//           row_local/eid) and row_map (A.row(), the next frontier).
#include <cooperative_groups.h>

#include <algorithm>
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include "common.cuh"
#include "gs_internal.h"
#include "nodewise_common.cuh"

namespace cg = cooperative_groups;

namespace gsb {

constexpr int NW_CS = 8;          // CTAs per cluster (= SMs per mini-batch)
constexpr int NW_THREADS = 1024;  // one CTA per SM
constexpr int NW_WARPS = NW_THREADS / 32;
constexpr int MAX_CLUSTERS = 4096;

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
  int64_t o_u, o_pos, o_val, o_coff, o_ccnt, o_ceoff, o_bits, o_wpre, o_tab;
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
  int32_t* u;      // [slot] sampled row
  uint32_t* pos;   // [slot] position inside the column (ShaDow: local id)
  float* val;      // [slot] PASS prob (or NULL)
  int64_t* coff;   // [col] indptr[v]
  int32_t* ccnt;   // [col] sampled edges of the column
  int32_t* ceoff;  // [col] CTA-local edge offset
  uint32_t* bits;  // [slot/32] first-occurrence bitmap
  int32_t* wpre;   // [slot/32] CTA-local count of first slots before the word
  unsigned long long* tab;
};

// shared memory of one CTA (dynamic, ~150 KB)
struct NWSmem {
  WarpChunk wc[NW_WARPS];
  unsigned long long scan[33];
  long long wtot[NW_WARPS];
  unsigned long long tot;                   // this CTA: (edges << 32) | rows
  long long base_e[NW_CS + 1], base_r[NW_CS + 1];
  long long misc[4];
};
// next generation tag 1..255; returns true when the table must be cleared.
__device__ __forceinline__ bool next_gen(uint32_t& gen) {
  const bool wrap = (gen == 255u);
  gen = (gen % 255u) + 1u;
  return wrap;
}

__device__ void clear_table(const NWParams& P, Ws& W, int crank) {
  const int64_t cap = 1ll << P.log_tab_cap;
  for (int64_t i = (int64_t)crank * blockDim.x + threadIdx.x; i < cap;
       i += (int64_t)NW_CS * blockDim.x)
    W.tab[i] = ~0ull;
}

// Range of warp `w` inside [c0, c1) (contiguous split).
__device__ __forceinline__ void warp_range(int64_t c0, int64_t c1, int w, int64_t* a, int64_t* b) {
  const int64_t n = c1 - c0, per = (n + NW_WARPS - 1) / NW_WARPS;
  *a = min(c1, c0 + (int64_t)w * per);
  *b = min(c1, *a + per);
}

// ---------------------------------------------------------------------------
// ShaDow induce for batch b (R12).
// Z = seeds ++ row_map_0 ++ ... ++ row_map_{L-1}; U = first-occurrence unique
// of Z; block = every edge u -> v of A with u, v in U, columns in U order.
//   S1 insert (Z[z], z) keeping the minimum z;  S2 first flags + CTA scan;
//   S3 write U and replace each entry's value by the local id;
//   S4 warp-per-column count of in-U rows + CTA scan;  S5 emit.
// ---------------------------------------------------------------------------
__device__ void shadow_induce(const NWParams& P, Ws& W, NWSmem& S, cg::cluster_group& cluster,
                              int crank, int64_t b, int64_t bstart, int64_t nb,
                              const int64_t* rows_l, uint32_t tag) {
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
  const int64_t zchunk = (Zn + NW_CS - 1) / NW_CS;
  const int64_t z0 = min(Zn, (int64_t)crank * zchunk), z1 = min(Zn, z0 + zchunk);
  const int64_t ubase = bstart * P.sh_stride;
  const int64_t uibase = ubase + b;
  uint32_t* lidz = W.pos;  // reuse: local id of first occurrences

  // S1
  for (int64_t z = z0 + threadIdx.x; z < z1; z += blockDim.x)
    otab_insert_min(W.tab, log_cap, tag, zval(z), (uint32_t)z);
  cluster.sync();
  // S2
  unsigned long long carry = 0;
  for (int64_t zt = z0; zt < z1; zt += blockDim.x) {
    const int64_t z = zt + threadIdx.x;
    bool first = false;
    if (z < z1) {
      const int64_t h = otab_find(W.tab, log_cap, tag, zval(z));
      first = h >= 0 && tab_val(__ldcg(W.tab + h)) == (uint32_t)z;
    }
    unsigned long long tot;
    const unsigned long long ex =
        block_exclusive_scan((unsigned long long)(first ? 1 : 0), S.scan, &tot) + carry;
    if (first) lidz[z] = (uint32_t)ex;
    carry += tot;
  }
  if (threadIdx.x == 0) S.tot = carry;
  cluster.sync();
  if (threadIdx.x == 0) {
    long long a = 0;
    for (int r = 0; r < NW_CS; ++r) {
      S.base_r[r] = a;
      a += (long long)cluster.map_shared_rank(&S, r)->tot;
    }
    S.base_r[NW_CS] = a;
  }
  __syncthreads();
  const int64_t nU = S.base_r[NW_CS];
  // S3
  for (int64_t z = z0 + threadIdx.x; z < z1; z += blockDim.x) {
    const uint32_t u = zval(z);
    const int64_t h = otab_find(W.tab, log_cap, tag, u);
    if (h >= 0 && tab_val(__ldcg(W.tab + h)) == (uint32_t)z) {
      const int64_t lid = S.base_r[crank] + __ldcg(lidz + z);
      P.sh_nodes[ubase + lid] = (int32_t)u;
      W.tab[h] = tab_entry(tag, u, (uint32_t)lid);
    }
  }
  cluster.sync();
  // S4: count in-U rows of every column of U (warp per column)
  const int64_t uchunk = (nU + NW_CS - 1) / NW_CS;
  const int64_t u0 = min(nU, (int64_t)crank * uchunk), u1 = min(nU, u0 + uchunk);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int64_t c = u0 + warp; c < u1; c += NW_WARPS) {
    const int32_t v = __ldcg(P.sh_nodes + ubase + c);
    const int64_t off = __ldg(P.indptr + v), d = __ldg(P.indptr + v + 1) - off;
    int cnt = 0;
    for (int64_t i = lane; i < d; i += 32) {
      const uint32_t u = (uint32_t)__ldg(P.indices + off + i);
      cnt += otab_find(W.tab, log_cap, tag, u) >= 0 ? 1 : 0;
    }
    cnt = (int)__reduce_add_sync(0xffffffffu, (unsigned)cnt);
    if (lane == 0) W.ccnt[c] = cnt;
  }
  __syncthreads();
  carry = 0;
  for (int64_t ct = u0; ct < u1; ct += blockDim.x) {
    const int64_t c = ct + threadIdx.x;
    const unsigned long long cv = c < u1 ? (unsigned long long)__ldcg(W.ccnt + c) : 0ull;
    unsigned long long tot;
    const unsigned long long ex = block_exclusive_scan(cv, S.scan, &tot) + carry;
    if (c < u1) W.ceoff[c] = (int32_t)ex;
    carry += tot;
  }
  if (threadIdx.x == 0) S.tot = carry;
  cluster.sync();
  if (threadIdx.x == 0) {
    long long a = 0;
    for (int r = 0; r < NW_CS; ++r) {
      S.base_e[r] = a;
      a += (long long)cluster.map_shared_rank(&S, r)->tot;
    }
    S.base_e[NW_CS] = a;
    if (crank == 0) S.misc[0] = (long long)atomicAdd(P.sh_edge_ctr, (unsigned long long)a);
  }
  cluster.sync();
  if (threadIdx.x == 0) S.misc[1] = cluster.map_shared_rank(&S, 0)->misc[0];
  __syncthreads();
  const int64_t nE = S.base_e[NW_CS];
  const int64_t ebase = S.misc[1];
  const bool fits = ebase + nE <= P.sh_edge_cap;
  if (!fits && crank == 0 && threadIdx.x == 0) atomicOr(P.err, ERR_CAPACITY);
  // S5: emit (warp per column, ballot compaction keeps CSC order)
  for (int64_t c = u0 + warp; c < u1; c += NW_WARPS) {
    const int32_t v = __ldcg(P.sh_nodes + ubase + c);
    const int64_t off = __ldg(P.indptr + v), d = __ldg(P.indptr + v + 1) - off;
    int64_t e = S.base_e[crank] + __ldcg(W.ceoff + c);
    if (lane == 0) P.sh_indptr[uibase + c] = e;
    if (!fits) continue;
    for (int64_t i0 = 0; i0 < d; i0 += 32) {
      const int64_t i = i0 + lane;
      int64_t h = -1;
      if (i < d) h = otab_find(W.tab, log_cap, tag, (uint32_t)__ldg(P.indices + off + i));
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
__global__ void __cluster_dims__(NW_CS, 1, 1) __launch_bounds__(NW_THREADS, 1)
    nodewise_kernel(NWParams P) {
  cg::cluster_group cluster = cg::this_cluster();
  const int crank = (int)cluster.block_rank();
  const int64_t cid = blockIdx.x / NW_CS;
  const int64_t nclusters = gridDim.x / NW_CS;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  NWSmem& S = *reinterpret_cast<NWSmem*>(smem_raw);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;

  Ws W;
  char* base = P.ws + cid * P.ws_stride;
  W.u = (int32_t*)(base + P.o_u);
  W.pos = (uint32_t*)(base + P.o_pos);
  W.val = P.o_val >= 0 ? (float*)(base + P.o_val) : nullptr;
  W.coff = (int64_t*)(base + P.o_coff);
  W.ccnt = (int32_t*)(base + P.o_ccnt);
  W.ceoff = (int32_t*)(base + P.o_ceoff);
  W.bits = (uint32_t*)(base + P.o_bits);
  W.wpre = (int32_t*)(base + P.o_wpre);
  W.tab = (unsigned long long*)(base + P.o_tab);

  uint32_t gen = P.gen[cid];
  NWCore core;
  core.indptr = P.indptr;
  core.indices = P.indices;
  core.weights = P.weights;
  core.N = P.N;
  core.err = P.err;
  core.replace = P.replace;
  core.bias = P.bias;
  core.key = P.key;
  NWStage stage;
  stage.u = W.u;
  stage.pos = W.pos;
  stage.val = W.val;
  stage.coff = W.coff;
  stage.ccnt = W.ccnt;
  stage.tab = W.tab;

  for (int64_t b = cid; b < P.num_batches; b += nclusters) {
    const int64_t bstart = b * P.batch_size;
    const int64_t nb = min(P.batch_size, P.num_seeds - bstart);
    const uint32_t gb = (uint32_t)(P.batch_base + b);
    const int32_t* F = P.seeds + bstart;
    int64_t T = nb;
    int64_t colbase = bstart;
    int64_t rows_l[MAX_LAYERS];

    for (int l = 0; l < P.L; ++l) {
      const int k = P.k[l];
      const int64_t rbase = bstart * P.K[l];
      const int64_t ibase = colbase + b;
      if (next_gen(gen)) {
        clear_table(P, W, crank);
        cluster.sync();
      }
      const uint32_t tag = otag(gen);
      int log_cap = log2_pow2ceil64((T * k * 4) / 3 + 64);
      if (log_cap > P.log_tab_cap) log_cap = P.log_tab_cap;
      const int64_t chunk = (T + NW_CS - 1) / NW_CS;
      const int64_t c0 = min(T, (int64_t)crank * chunk), c1 = min(T, c0 + chunk);
      int64_t wa, wb;
      warp_range(c0, c1, warp, &wa, &wb);

      // ---- P1: Extract + Select + stage + insert ----
      int wedges = 0;
      for (int64_t jb = wa; jb < wb; jb += 32)
        wedges += select_chunk(core, stage, S.wc[warp], l, k, log_cap, tag, F, jb, wb, gb);
      if (lane == 0) S.wtot[warp] = wedges;
      __syncthreads();
      if (warp == 0) {  // exclusive scan of the warp totals
        const int t = lane < NW_WARPS ? (int)S.wtot[lane] : 0;
        int tot;
        const int ex = warp_excl(t, &tot);
        if (lane < NW_WARPS) S.wtot[lane] = ex;
        if (lane == 0) S.misc[2] = tot;
      }
      __syncthreads();
      {  // CTA-local edge offset of every column of this warp
        long long run = S.wtot[warp];
        for (int64_t jb = wa; jb < wb; jb += 32) {
          const int64_t j = jb + lane;
          const int c = j < wb ? __ldcg(W.ccnt + j) : 0;
          int tot;
          const int ex = warp_excl(c, &tot);
          if (j < wb) W.ceoff[j] = (int32_t)(run + ex);
          run += tot;
        }
      }
      const long long cta_edges = S.misc[2];
      cluster.sync();

      // ---- P2: first-occurrence bitmap over the batch's padded slots ----
      const int64_t PT = T * k;
      const int64_t NWD = (PT + 31) >> 5;
      const int64_t wchunk = (NWD + NW_CS - 1) / NW_CS;
      const int64_t w0 = min(NWD, (int64_t)crank * wchunk), w1 = min(NWD, w0 + wchunk);
      int64_t xa, xb;
      warp_range(w0, w1, warp, &xa, &xb);
      int wrows = 0;
      for (int64_t wd0 = xa; wd0 < xb; wd0 += NW_ILP) {
        uint32_t uu[NW_ILP];
        bool vv[NW_ILP];
        int64_t hh[NW_ILP];
#pragma unroll
        for (int i = 0; i < NW_ILP; ++i) {
          const int64_t wd = wd0 + i;
          const int64_t p = wd * 32 + lane;
          vv[i] = false;
          if (wd < xb && p < PT) {
            const int64_t j = p / k;
            vv[i] = (p - j * k) < __ldcg(W.ccnt + j);
          }
          uu[i] = vv[i] ? (uint32_t)__ldcg(W.u + p) : 0u;
        }
#pragma unroll
        for (int i = 0; i < NW_ILP; ++i)
          hh[i] = vv[i] ? otab_find(W.tab, log_cap, tag, uu[i]) : -1;
#pragma unroll
        for (int i = 0; i < NW_ILP; ++i) {
          const int64_t wd = wd0 + i;
          const int64_t p = wd * 32 + lane;
          bool first = false;
          if (vv[i]) {
            if (hh[i] < 0) atomicOr(P.err, ERR_INTERNAL);
            else first = tab_val(__ldcg(W.tab + hh[i])) == (uint32_t)p;
          }
          const uint32_t word = __ballot_sync(0xffffffffu, first);
          if (wd < xb && lane == 0) W.bits[wd] = word;
          wrows += __popc(word);
        }
      }
      if (lane == 0) S.wtot[warp] = wrows;
      __syncthreads();
      if (warp == 0) {
        const int t = lane < NW_WARPS ? (int)S.wtot[lane] : 0;
        int tot;
        const int ex = warp_excl(t, &tot);
        if (lane < NW_WARPS) S.wtot[lane] = ex;
        if (lane == 0) S.tot = ((unsigned long long)cta_edges << 32) | (unsigned)tot;
      }
      __syncthreads();
      {  // CTA-local count of first slots before every word of this warp
        long long run = S.wtot[warp];
        for (int64_t wd0 = xa; wd0 < xb; wd0 += 32) {
          const int64_t wd = wd0 + lane;
          const int c = wd < xb ? __popc(__ldcg(W.bits + wd)) : 0;
          int tot;
          const int ex = warp_excl(c, &tot);
          if (wd < xb) W.wpre[wd] = (int32_t)(run + ex);
          run += tot;
        }
      }
      cluster.sync();

      // ---- P3: relabel + compaction ----
      if (threadIdx.x == 0) {
        long long ae = 0, ar = 0;
        for (int r = 0; r < NW_CS; ++r) {
          S.base_e[r] = ae;
          S.base_r[r] = ar;
          const unsigned long long t = cluster.map_shared_rank(&S, r)->tot;
          ae += (long long)(t >> 32);
          ar += (long long)(t & 0xffffffffu);
        }
        S.base_e[NW_CS] = ae;
        S.base_r[NW_CS] = ar;
      }
      __syncthreads();
      const int64_t baseE = S.base_e[crank];
      const int64_t totE = S.base_e[NW_CS], totR = S.base_r[NW_CS];
      int32_t* row_map = P.row_map[l] + rbase;
      int32_t* row_local = P.row_local[l] ? P.row_local[l] + rbase : nullptr;
      int64_t* eid_out = P.eid[l] ? P.eid[l] + rbase : nullptr;
      float* val_out = P.val[l] ? P.val[l] + rbase : nullptr;
      int64_t* indptr_out = P.indptr_out[l] ? P.indptr_out[l] + ibase : nullptr;
      for (int64_t jb = wa; jb < wb; jb += 32) {
        const int64_t j = jb + lane;
        const bool act = j < wb;
        const int cnt = act ? __ldcg(W.ccnt + j) : 0;
        const int eo = act ? __ldcg(W.ceoff + j) : 0;
        const int64_t off = act ? __ldcg(W.coff + j) : 0;
        int total;
        const int pre = warp_excl(cnt, &total);
        S.wc[warp].pre[lane] = pre;
        S.wc[warp].coff[lane] = off;
        S.wc[warp].cnt_all[lane] = eo;  // P3: CTA-local edge offset of the column
        if (act) {
          if (indptr_out) indptr_out[j] = baseE + eo;
          if (l == 0 && P.col0) P.col0[bstart + j] = __ldcg(F + j);
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
            if (ok[i]) {
              const int c = chunk_col(S.wc[warp].pre, f);
              const int s = f - S.wc[warp].pre[c];
              p[i] = (jb + c) * k + s;
              e[i] = baseE + S.wc[warp].cnt_all[c] + s;
              uu[i] = (uint32_t)__ldcg(W.u + p[i]);
              ps[i] = __ldcg(W.pos + p[i]);
              cc[i] = c;
            }
          }
#pragma unroll
          for (int i = 0; i < NW_ILP; ++i) {
            hh[i] = -1;
            if (ok[i]) {
              if (eid_out) eid_out[e[i]] = S.wc[warp].coff[cc[i]] + ps[i];
              if (val_out) val_out[e[i]] = __ldcg(W.val + p[i]);
              hh[i] = otab_find(W.tab, log_cap, tag, uu[i]);
            }
          }
#pragma unroll
          for (int i = 0; i < NW_ILP; ++i) {
            if (ok[i]) {
              const uint32_t p0 = hh[i] >= 0 ? tab_val(__ldcg(W.tab + hh[i])) : 0u;
              const int64_t wd = p0 >> 5;
              const int r0 = (int)(wd / wchunk);
              const uint32_t bw = __ldcg(W.bits + wd);
              const int64_t lid = S.base_r[r0] + __ldcg(W.wpre + wd) +
                                  __popc(bw & ((1u << (p0 & 31)) - 1u));
              if (row_local) row_local[e[i]] = (int32_t)lid;
              if (p0 == (uint32_t)p[i]) row_map[lid] = (int32_t)uu[i];
            }
          }
        }
        __syncwarp();
      }
      if (crank == 0 && threadIdx.x == 0) {
        if (indptr_out) indptr_out[T] = totE;
        if (!P.shadow) {
          long long* m = (long long*)(P.meta + (b * P.meta_layers + l) * 8);
          m[0] = T; m[1] = totR; m[2] = totE; m[3] = colbase; m[4] = rbase; m[5] = ibase;
          m[6] = rbase; m[7] = 0;
        }
      }
      cluster.sync();
      F = P.row_map[l] + rbase;
      T = totR;
      colbase = rbase;
      rows_l[l] = totR;
    }

    if (P.shadow) {
      if (next_gen(gen)) {
        clear_table(P, W, crank);
        cluster.sync();
      }
      shadow_induce(P, W, S, cluster, crank, b, bstart, nb, rows_l, otag(gen));
    }
  }
  if (crank == 0 && threadIdx.x == 0) P.gen[cid] = gen;
}

// ---------------------------------------------------------------------------
// Host side
// ---------------------------------------------------------------------------
static int64_t align256(int64_t x) { return (x + 255) & ~int64_t(255); }

static int max_active_clusters() {
  static int cached = -1;
  if (cached > 0) return cached;
  cudaFuncSetAttribute(nodewise_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       (int)sizeof(NWSmem));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(NW_CS * 1024);
  cfg.blockDim = dim3(NW_THREADS);
  cfg.dynamicSmemBytes = sizeof(NWSmem);
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, nodewise_kernel, &cfg) != cudaSuccess || n <= 0) {
    cudaGetLastError();
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    n = sms / NW_CS;
  }
  cached = n;
  return n;
}

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
  int64_t slot_cap = 32, col_cap = 32;
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
  col_cap += 32;
  slot_cap += 64;
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
    sh_edges = std::max<int64_t>(std::max<int64_t>(int64_t(1) << 20, blk->sh_edge_hint),
                                 sh_nodes * 4);
    ok = need(blk->b_col[1], sh_nodes * 4) && need(blk->b_indptr[0], (sh_nodes + nbatch) * 8) &&
         need(blk->b_rowl[0], sh_edges * 4) && need(blk->b_eid[0], sh_edges * 8);
    sh_edges = (int64_t)std::min(blk->b_rowl[0].bytes / 4, blk->b_eid[0].bytes / 8);
  }
  const int meta_layers = shadow ? 1 : L;
  ok = ok && need(blk->b_meta, nbatch * meta_layers * 8 * 8) && need(blk->b_err, 16) &&
       need(blk->b_ctr, 8 * (MAX_LAYERS + 2));
  if (!ok) return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (blocks buffers)");

  // ---- workspace (per cluster) ----
  int log_tab = 6;
  while ((int64_t(1) << log_tab) < (slot_cap * 4) / 3 + 64) ++log_tab;
  const int64_t words = (slot_cap + 31) / 32 + 2;
  int64_t o = 0;
  P.o_u = o; o = align256(o + slot_cap * 4);
  P.o_pos = o; o = align256(o + slot_cap * 4);
  if (bias == GS_W_PASS_COLNORM && !shadow) {
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
  P.o_tab = o; o = align256(o + (int64_t(8) << log_tab));
  P.ws_stride = o;
  P.log_tab_cap = log_tab;
  const int nclusters =
      (int)std::max<int64_t>(1, std::min<int64_t>(nbatch, max_active_clusters()));
  const size_t ws_bytes = (size_t)P.ws_stride * nclusters;
  const bool fresh = blk->b_ws.bytes < ws_bytes || blk->ws_stride_prev != P.ws_stride ||
                     blk->ws_kind_prev != 1;
  if (!blk->b_ws.ensure(al, ws_bytes, stream) || !blk->b_gen.ensure(al, MAX_CLUSTERS * 4, stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (workspace)");
  if (fresh) {
    // tables start cleared (~0 = the oldest generation), tags restart at 1
    GS_CUDA_TRY(cudaMemsetAsync(blk->b_ws.ptr, 0xFF, blk->b_ws.bytes, stream));
    GS_CUDA_TRY(cudaMemsetAsync(blk->b_gen.ptr, 0, MAX_CLUSTERS * 4, stream));
  }
  blk->ws_stride_prev = P.ws_stride;
  blk->ws_kind_prev = 1;
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
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_ctr.ptr, 0, 8 * (MAX_LAYERS + 2), stream));
  if (nbatch == 0) return GS_OK;

  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(nclusters * NW_CS));
  cfg.blockDim = dim3(NW_THREADS);
  cfg.dynamicSmemBytes = sizeof(NWSmem);
  cfg.stream = stream;
  GS_CUDA_TRY(cudaLaunchKernelEx(&cfg, nodewise_kernel, P));
  return GS_OK;
}

}  // namespace gsb
