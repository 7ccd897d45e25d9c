// shadow.cu -- induced subgraphs: ShaDow (R12): node-wise
// sampling of every hop (nodewise_wave.cu), then per mini-batch the subgraph of
// A induced on U = unique(seeds, rows of every hop), ascending (R3/R12); and
// GraphSAINT-RW (R26): DeepWalk walks (walk.cu), then the subgraph
// induced on U = the nodes each batch's walks visited.
//
// Induce is one persistent kernel of thread-block CLUSTERS, one cluster per
// mini-batch at a time.  U's membership bitmap (N bits) is split across the
// cluster's shared memories (DSMEM): CTA r holds bits [r*bpc, (r+1)*bpc) plus
// a popcount prefix per 256 bits, so the membership test of every streamed
// edge -- the hot loop, Sum of in-degrees over U per batch -- and the rank of a
// kept row are shared-memory reads (local or a peer's), never L2/HBM probes.
// Per batch: mark U -> scan (U ascending) -> count kept edges per column
// (columns claimed dynamically by every warp of the cluster from a DSMEM
// counter), staging each kept edge (row rank, eid) in a per-warp region -> scan (CSC
// indptr, bump-allocated edge range) -> copy the staged edges to their CSC
// positions (a column whose edges did not fit the region is streamed again).
#include <algorithm>
#include <cstdlib>
#include <new>
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "gs_internal.h"

namespace cg = cooperative_groups;

namespace gsb {

gs_status run_nodewise(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                            int64_t batch_size, int64_t batch_base, const int32_t* fanouts, int L,
                            int replace, int bias, uint64_t key, cudaStream_t stream,
                            gs_blocks* blk);
gs_status launch_walk(const gs_graph* g, const int32_t* starts, int64_t num_walkers,
                      int64_t walker_base, int length, float p, float q, uint64_t key,
                      bool node2vec, bool plain, cudaStream_t stream, int32_t* traces,
                      int* err = nullptr);

constexpr int SH_THREADS = 512;
constexpr int SH_WARPS = SH_THREADS / 32;
constexpr int SH_MAX_CS = 8;                      // portable cluster size
constexpr int SH_ILP = 8;                         // column positions per lane in flight
constexpr int SH_CLAIM = 4;                       // columns per claim of the count pass
constexpr int64_t SH_SMEM_CAP = 220 * 1024;      // dynamic shared memory per CTA (bitmap + prefixes)

struct SHParams {
  const int64_t* indptr;
  const int32_t* indices;
  int64_t N;
  const int32_t* seeds;
  int64_t num_seeds, batch_size, num_batches;
  int L;
  const int32_t* rows[MAX_LAYERS];  // node-wise row_map of every hop
  int64_t K[MAX_LAYERS];
  const int64_t* nmeta;             // node-wise meta [b][L][8]
  const int32_t* traces;            // GraphSAINT-RW: walk traces [root][L1] (U source instead of seeds + rows)
  int64_t L1;                       // walk_length + 1
  int64_t stride;                   // U capacity per batch (fixed batches)
  const int64_t* bptr;              // [nb + 1] seed offsets (ragged batches) or NULL: b * batch_size
  int64_t mult;                     // U capacity per seed (region of batch b at bstart * mult)
  int32_t* U;                       // [b * stride] U ascending (col_map == row_map)
  int64_t* indptr_out;              // [b * stride + b] CSC over U
  int32_t* row_local;
  int64_t* eid;
  int64_t edge_cap;
  unsigned long long* edge_ctr;     // bump allocator of the edge range (total = need)
  int32_t* ucnt;                    // [b * stride] kept edges per column, then its prefix
  int64_t* meta;
  int* err;
  unsigned int* claim;
  int64_t* ustart;                  // [b * stride] staged start of a column's kept edges, -1: re-stream
  int32_t* stage_row;               // [CTA][warp][wcap] kept edges staged by the count pass
  int64_t* stage_eid;
  int64_t wcap;
  int64_t bpc;                      // bitmap bits per CTA (multiple of 256)
  uint32_t inv;                     // floor(2^32 / bpc)
  int load_first;                   // U column loads evict-first (else evict-normal)
};

struct SHShared {                   // static part; the bitmap + prefix are dynamic
  long long b;
  long long total, base[SH_MAX_CS];
  long long etotal, ebase, eoff, E, nU;
  unsigned long long next;          // rank 0: the cluster's column claim counter (count pass)
  long long scr64[40];
  int scr32[40];
};

// Owner CTA of bit u: u / bpc by a 32-bit reciprocal (inv = floor(2^32 / bpc))
// and one correction step (no 64-bit division on the per-edge path).
__device__ __forceinline__ unsigned sh_owner(uint32_t u, uint32_t bpc, uint32_t inv) {
  unsigned q = __umulhi(u, inv);
  if ((q + 1u) * bpc <= u) ++q;
  return q;
}

__device__ __forceinline__ bool sh_member(const cg::cluster_group& cl, uint32_t* bm, uint32_t bpc,
                                          uint32_t inv, uint32_t u) {
  const unsigned owner = sh_owner(u, bpc, inv);
  const uint32_t x = u - owner * bpc;
  const uint32_t* w = cl.map_shared_rank(bm, owner);
  return (w[x >> 5] >> (x & 31)) & 1u;
}

// Rank of u in U: the owner's base + its 256-bit group prefix + the word's
// offset inside the group (one byte per word) + the bits below u in its word.
__device__ __forceinline__ long long sh_rank(const cg::cluster_group& cl, uint32_t* bm, int32_t* gp,
                                             uint8_t* off8, const SHShared& ss, uint32_t bpc,
                                             uint32_t inv, uint32_t u) {
  const unsigned owner = sh_owner(u, bpc, inv);
  const uint32_t x = u - owner * bpc;
  const uint32_t* w = cl.map_shared_rank(bm, owner);
  const int32_t* p = cl.map_shared_rank(gp, owner);
  const uint8_t* o = cl.map_shared_rank(off8, owner);
  return ss.base[owner] + p[x >> 8] + o[x >> 5] + __popc(w[x >> 5] & ((1u << (x & 31)) - 1u));
}

// batch b's first seed, seed count and U region (fixed or ragged batches)
__device__ __forceinline__ int64_t sh_bstart(const SHParams& P, int64_t b) {
  return P.bptr ? __ldg(P.bptr + b) : b * P.batch_size;
}
__device__ __forceinline__ long long sh_T0(const SHParams& P, int64_t b) {
  return P.bptr ? (long long)(__ldg(P.bptr + b + 1) - __ldg(P.bptr + b))
                : min(P.batch_size, P.num_seeds - b * P.batch_size);
}

__global__ void __launch_bounds__(SH_THREADS, 1) shadow_induce_kernel(SHParams P) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ SHShared ss;
  cg::cluster_group cl = cg::this_cluster();
  const unsigned rank = cl.block_rank(), CS = cl.num_blocks();
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t bpc = P.bpc;
  const int nwords = (int)(bpc >> 5), ngroups = (int)(bpc >> 8);
  uint32_t* bm = (uint32_t*)smem_raw;
  int32_t* gp = (int32_t*)(smem_raw + (size_t)nwords * 4);
  uint8_t* off8 = (uint8_t*)(gp + ngroups);
  const uint32_t bpc32 = (uint32_t)bpc, inv = P.inv;
  // the output stores stream (evict-first); the U columns' index loads: evict-normal
  // (hub columns recur in the other batches' U) unless P.load_first
  const uint64_t pf = pol_first(), pg = P.load_first ? pol_first() : pol_normal();
  while (true) {
    if (rank == 0 && tid == 0) ss.b = (long long)atomicAdd(P.claim, 1u);
    cl.sync();
    const long long b = *cl.map_shared_rank(&ss.b, 0);
    cl.sync();  // no CTA may exit (or re-claim) while a peer still reads its shared memory
    if (b >= P.num_batches) break;
    // ---- mark U ----
    for (int i = tid; i < nwords; i += SH_THREADS) bm[i] = 0u;
    cl.sync();
    const int64_t bstart = sh_bstart(P, b);
    const long long T0 = sh_T0(P, b);
    const int64_t ub = bstart * P.mult;  // the batch's U region
    long long nitems = T0;
    long long cnt_l[MAX_LAYERS];
    if (P.traces) {
      nitems = T0 * P.L1;  // every visited node of the batch's walks (R26)
    } else {
      for (int l = 0; l < P.L; ++l) {
        cnt_l[l] = __ldcg(P.nmeta + (b * P.L + l) * 8 + 1);
        nitems += cnt_l[l];
      }
    }
    for (long long i = (long long)rank * SH_THREADS + tid; i < nitems; i += (long long)CS * SH_THREADS) {
      long long x = i;
      int32_t u;
      if (P.traces) {
        u = __ldcg(P.traces + bstart * P.L1 + x);
        if (u == -1 && x % P.L1 != 0) continue;  // padding after a dead end (R13)
      } else if (x < T0) {
        u = __ldg(P.seeds + bstart + x);
      } else {
        x -= T0;
        int l = 0;
        while (x >= cnt_l[l]) x -= cnt_l[l++];
        u = __ldcg(P.rows[l] + bstart * P.K[l] + x);
      }
      if (u < 0 || (int64_t)u >= P.N) {
        atomicOr(P.err, ERR_SEED_RANGE);
        continue;
      }
      const unsigned owner = sh_owner((uint32_t)u, bpc32, inv);
      const uint32_t xb = (uint32_t)u - owner * bpc32;
      atomicOr(cl.map_shared_rank(bm, owner) + (xb >> 5), 1u << (xb & 31));
    }
    cl.sync();
    // ---- local prefix per 256 bits, U ascending ----
    long long run = 0;
    for (int g0 = 0; g0 < ngroups; g0 += SH_THREADS) {
      const int g = g0 + tid;
      int c = 0;
      if (g < ngroups)
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          off8[g * 8 + i] = (uint8_t)c;
          c += __popc(bm[g * 8 + i]);
        }
      int tot;
      const int ex = block_exclusive_scan<int>(c, ss.scr32, &tot);
      if (g < ngroups) gp[g] = (int32_t)(run + ex);
      run += tot;
    }
    if (tid == 0) {
      ss.total = run;
      ss.next = 0;
    }
    cl.sync();
    if (tid < (int)CS) ss.base[tid] = 0;
    if (tid == 0) {
      long long acc = 0;
      for (unsigned r = 0; r < CS; ++r) {
        ss.base[r] = acc;
        acc += *cl.map_shared_rank(&ss.total, r);
      }
      ss.nU = acc;
    }
    __syncthreads();
    const long long nU = ss.nU;
    int32_t* U = P.U + ub;
    for (int g = tid; g < ngroups; g += SH_THREADS) {
      long long r = ss.base[rank] + gp[g];
      for (int i = 0; i < 8; ++i) {
        uint32_t m = bm[g * 8 + i];
        while (m) {
          const int bit = __ffs(m) - 1;
          m &= m - 1u;
          U[r++] = (int32_t)((int64_t)rank * bpc + (int64_t)(g * 8 + i) * 32 + bit);
        }
      }
    }
    __threadfence();
    cl.sync();
    // ---- count kept edges per column (this CTA's share of U), staging every
    // kept edge (row rank, eid) in this warp's private region so that the
    // emit below is a copy, not a second stream of the columns ----
    const long long c_lo = nU * rank / CS, c_hi = nU * (rank + 1) / CS;
    int32_t* ucnt = P.ucnt + ub;
    int64_t* ustart = P.ustart + ub;
    const int64_t wreg = ((int64_t)blockIdx.x * SH_WARPS + warp) * P.wcap;
    int32_t* wst_r = P.stage_row + wreg;
    int64_t* wst_e = P.stage_eid + wreg;
    long long wfill = 0;
    // columns are claimed dynamically, SH_CLAIM at a time, from a counter in
    // rank 0's shared memory by every warp of the cluster (hub columns no
    // longer pin one warp / one CTA while the others wait at the barrier)
    unsigned long long* next = cl.map_shared_rank(&ss.next, 0);
    for (;;) {
    long long cb = 0;
    if (lane == 0) cb = (long long)atomicAdd(next, (unsigned long long)SH_CLAIM);
    cb = __shfl_sync(0xffffffffu, cb, 0);
    if (cb >= nU) break;
    const long long ce = min(cb + SH_CLAIM, nU);
    for (long long c = cb; c < ce; ++c) {
      const int32_t v = __ldcg(U + c);
      const int64_t o = __ldg(P.indptr + v), d = __ldg(P.indptr + v + 1) - o;
      int cnt = 0;
      const long long start = wfill;
      bool staged = true;
      for (int64_t i0 = 0; i0 < d; i0 += 32 * SH_ILP) {  // SH_ILP loads, then tests, in flight
        uint32_t u[SH_ILP];
#pragma unroll
        for (int q = 0; q < SH_ILP; ++q) {
          const int64_t i = i0 + q * 32 + lane;
          u[q] = i < d ? (uint32_t)ldg_h(P.indices + o + i, pg) : 0xFFFFFFFFu;
        }
        bool m[SH_ILP];
#pragma unroll
        for (int q = 0; q < SH_ILP; ++q) m[q] = u[q] != 0xFFFFFFFFu && sh_member(cl, bm, bpc32, inv, u[q]);
#pragma unroll
        for (int q = 0; q < SH_ILP; ++q) {
          const uint32_t bal = __ballot_sync(0xffffffffu, m[q]);
          const int n = __popc(bal);
          cnt += n;
          if (staged && wfill + n > P.wcap) staged = false;  // this column is re-streamed below
          if (staged) {
            if (m[q]) {
              const long long idx = wfill + __popc(bal & ((1u << lane) - 1u));
              wst_r[idx] = (int32_t)sh_rank(cl, bm, gp, off8, ss, bpc32, inv, u[q]);
              wst_e[idx] = o + i0 + q * 32 + lane;
            }
            wfill += n;
          }
        }
      }
      if (!staged) wfill = start;
      if (lane == 0) {
        ucnt[c] = cnt;
        ustart[c] = staged ? wreg + start : -1;  // absolute staging index
      }
    }
    }
    __threadfence();
    cl.sync();
    // ---- scan: CSC indptr over U, the batch's edge range ----
    long long erun = 0;
    for (long long c0 = c_lo; c0 < c_hi; c0 += SH_THREADS) {
      const long long c = c0 + tid;
      const int x = c < c_hi ? __ldcg(ucnt + c) : 0;
      int tot;
      const int ex = block_exclusive_scan<int>(x, ss.scr32, &tot);
      if (c < c_hi) ucnt[c] = (int32_t)(erun + ex);  // CTA-local exclusive prefix
      erun += tot;
    }
    if (tid == 0) ss.etotal = erun;
    cl.sync();
    if (tid == 0) {
      long long acc = 0, mine = 0;
      for (unsigned r = 0; r < CS; ++r) {
        if (r == rank) mine = acc;
        acc += *cl.map_shared_rank(&ss.etotal, r);
      }
      ss.ebase = mine;
      ss.E = acc;
      if (rank == 0) ss.eoff = (long long)atomicAdd(P.edge_ctr, (unsigned long long)acc);
    }
    cl.sync();
    const long long E = ss.E, ebase = ss.ebase;
    const long long eoff = *cl.map_shared_rank(&ss.eoff, 0);
    const bool fits = eoff + E <= P.edge_cap;
    int64_t* ip = P.indptr_out + ub + b;
    for (long long c = c_lo + tid; c < c_hi; c += SH_THREADS) ip[c] = ebase + __ldcg(ucnt + c);
    if (rank == 0 && tid == 0) {
      ip[nU] = E;
      long long* m = (long long*)(P.meta + b * 8);
      m[0] = nU; m[1] = nU; m[2] = E; m[3] = ub; m[4] = ub;
      m[5] = ub + b; m[6] = fits ? eoff : 0; m[7] = 0;
      if (!fits) m[2] = 0;  // nothing was written: an overflowed block is empty (GS_ERR_CAPACITY)
      if (!fits) atomicOr(P.err, ERR_CAPACITY);
    }
    // ---- write kept edges in CSC order: a copy of the staged edges (the
    // claiming warp staged it, ustart is absolute); columns that did not fit re-stream ----
    if (fits) {
      for (long long c = c_lo + warp; c < c_hi; c += SH_WARPS) {
        const long long st = __ldcg(ustart + c);
        if (st >= 0) {
          const long long p0 = __ldcg(ucnt + c);
          const long long n = (c + 1 < c_hi ? (long long)__ldcg(ucnt + c + 1) : ss.etotal) - p0;
          const long long dst = eoff + ebase + p0;
          for (long long i0 = lane; i0 < n; i0 += 32 * SH_ILP) {  // SH_ILP loads in flight
            int32_t r[SH_ILP];
            int64_t e[SH_ILP];
#pragma unroll
            for (int q = 0; q < SH_ILP; ++q) {
              const long long i = i0 + 32 * q;
              if (i < n) {
                r[q] = __ldcs(P.stage_row + st + i);
                e[q] = __ldcs(P.stage_eid + st + i);
              }
            }
#pragma unroll
            for (int q = 0; q < SH_ILP; ++q) {
              const long long i = i0 + 32 * q;
              if (i < n) {
                sth(P.row_local + dst + i, r[q], pf);
                sth(P.eid + dst + i, e[q], pf);
              }
            }
          }
          continue;
        }
        const int32_t v = __ldcg(U + c);
        const int64_t o = __ldg(P.indptr + v), d = __ldg(P.indptr + v + 1) - o;
        long long pos = eoff + ebase + __ldcg(ucnt + c);
        for (int64_t i0 = 0; i0 < d; i0 += 32 * SH_ILP) {
          uint32_t u[SH_ILP];
          bool m[SH_ILP];
#pragma unroll
          for (int q = 0; q < SH_ILP; ++q) {
            const int64_t i = i0 + q * 32 + lane;
            u[q] = i < d ? (uint32_t)ldg_h(P.indices + o + i, pg) : 0xFFFFFFFFu;
          }
#pragma unroll
          for (int q = 0; q < SH_ILP; ++q) m[q] = u[q] != 0xFFFFFFFFu && sh_member(cl, bm, bpc32, inv, u[q]);
#pragma unroll
          for (int q = 0; q < SH_ILP; ++q) {
            const uint32_t bal = __ballot_sync(0xffffffffu, m[q]);
            if (m[q]) {
              const long long e = pos + __popc(bal & ((1u << lane) - 1u));
              sth(P.row_local + e, (int32_t)sh_rank(cl, bm, gp, off8, ss, bpc32, inv, u[q]), pf);
              sth(P.eid + e, (int64_t)(o + i0 + q * 32 + lane), pf);
            }
            pos += __popc(bal);
          }
        }
      }
    }
    cl.sync();  // the bitmap is reused by the next batch
  }
}

// Cluster size for an N-bit membership bitmap (+ 1/64 prefix + 1/32 offsets)
// split over at most 8 CTAs' shared memory.
static gs_status induce_envelope(int64_t N, int* CS_out, int64_t* bpc_out) {
  int CS = 1;
  int64_t bpc = 0;
  for (; CS <= SH_MAX_CS; CS *= 2) {
    bpc = ((N + CS - 1) / CS + 255) / 256 * 256;
    if (bpc / 8 + bpc / 64 + bpc / 32 <= SH_SMEM_CAP) break;
  }
  if (CS > SH_MAX_CS)
    return fail(GS_ERR_NOT_SUPPORTED, "induce: N = %lld exceeds the shared-memory bitmap envelope (%lld nodes)",
                (long long)N, (long long)(SH_MAX_CS * (SH_SMEM_CAP * 64 / 11)));
  if (const char* e = getenv("GS_SH_CS")) {  // tests: a larger cluster than the graph needs
    const int want = atoi(e);
    while (CS < want && CS < SH_MAX_CS) {
      CS *= 2;
      bpc = ((N + CS - 1) / CS + 255) / 256 * 256;
    }
  }
  *CS_out = CS;
  *bpc_out = bpc;
  return GS_OK;
}

// Induce on U (one block per batch) -- P carries the U sources (seeds + node-wise
// rows, or walk traces); stride = U capacity per batch; err_src = the device
// error word of the producing kernel, folded into the result's.
static gs_status launch_induce(const gs_graph* g, SHParams P, int CS, int64_t bpc, int64_t nbatch,
                               int64_t mult, const int* err_src, cudaStream_t stream,
                               gs_blocks* blk) {
  const Allocator& al = blk->al;
  const int64_t nodes = P.bptr ? P.num_seeds * mult : nbatch * P.batch_size * mult;
  blk->kind = gs_blocks::SHADOW;
  blk->num_batches = nbatch;
  blk->num_layers = 1;
  blk->stream = stream;
  blk->synced = false;
  auto need = [&](DevBuf& b, int64_t bytes) -> bool {
    return b.ensure(al, (size_t)std::max<int64_t>(bytes, 256), stream);
  };
  int64_t edges = std::max<int64_t>(std::max<int64_t>(int64_t(1) << 20, blk->sh_edge_hint), nodes * 4);
  bool ok = need(blk->b_col[1], nodes * 4) && need(blk->b_indptr[0], (nodes + nbatch) * 8) &&
            need(blk->b_rowl[0], edges * 4) && need(blk->b_eid[0], edges * 8) &&
            need(blk->b_row[0], nodes * 4) && need(blk->b_meta, std::max<int64_t>(nbatch, 1) * 64) &&
            need(blk->b_err, 16) && need(blk->b_ctr, 8 * (MAX_LAYERS + 2));
  if (!ok) return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (induce buffers)");
  edges = (int64_t)std::min(blk->b_rowl[0].bytes / 4, blk->b_eid[0].bytes / 8);
  gs_layer_buffers& lb = blk->layers[0];
  lb = gs_layer_buffers{};
  lb.col_map = lb.row_map = (int32_t*)blk->b_col[1].ptr;
  lb.col_capacity = lb.row_capacity = nodes;
  lb.indptr = (int64_t*)blk->b_indptr[0].ptr;
  lb.indptr_capacity = nodes + nbatch;
  lb.row_local = (int32_t*)blk->b_rowl[0].ptr;
  lb.eid = (int64_t*)blk->b_eid[0].ptr;
  lb.edge_capacity = edges;

  P.indptr = g->indptr;
  P.indices = g->indices;
  P.N = g->num_nodes;
  P.num_batches = nbatch;
  P.mult = mult;
  P.stride = P.batch_size * mult;
  P.U = lb.row_map;
  P.indptr_out = lb.indptr;
  P.row_local = lb.row_local;
  P.eid = lb.eid;
  P.edge_cap = edges;
  P.edge_ctr = (unsigned long long*)blk->b_ctr.ptr;
  P.ucnt = (int32_t*)blk->b_row[0].ptr;
  P.meta = (int64_t*)blk->b_meta.ptr;
  P.err = (int*)blk->b_err.ptr;
  P.claim = (unsigned int*)((char*)blk->b_ctr.ptr + 8 * (MAX_LAYERS + 1));
  P.bpc = bpc;
  P.inv = (uint32_t)((uint64_t(1) << 32) / (uint64_t)bpc);
  P.load_first = getenv("GS_SH_LOAD_FIRST") ? 1 : 0;
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_err.ptr, 0, 16, stream));
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_ctr.ptr, 0, 8 * (MAX_LAYERS + 2), stream));
  if (nbatch == 0) return GS_OK;
  if (err_src)
    GS_CUDA_TRY(cudaMemcpyAsync(blk->b_err.ptr, err_src, 4, cudaMemcpyDeviceToDevice, stream));

  const size_t smem = (size_t)(bpc / 8 + bpc / 64 + bpc / 32);
  GS_CUDA_TRY(cudaFuncSetAttribute(shadow_induce_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)smem));
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = (unsigned)CS;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.blockDim = dim3(SH_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = stream;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cfg.gridDim = dim3((unsigned)CS);
  int nclusters = 0;
  GS_CUDA_TRY(cudaOccupancyMaxActiveClusters(&nclusters, (void*)shadow_induce_kernel, &cfg));
  nclusters = (int)std::max<int64_t>(1, std::min<int64_t>(nclusters, nbatch));
  cfg.gridDim = dim3((unsigned)(nclusters * CS));
  // staging of kept edges: a fixed region per warp (columns that do not fit
  // fall back to a second stream), then the per-column staged starts
  P.wcap = int64_t(1) << 17;
  if (const char* e = getenv("GS_SH_WCAP")) P.wcap = std::max<int64_t>(1, atoll(e));  // tests: force re-streams
  {
    const int64_t nw = (int64_t)nclusters * CS * SH_WARPS;
    const int64_t o_e = ((nw * P.wcap * 4) + 255) & ~int64_t(255);
    const int64_t o_s = o_e + nw * P.wcap * 8;
    if (!blk->b_ws.ensure(al, (size_t)(o_s + std::max<int64_t>(nodes, 1) * 8), stream))
      return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (induce staging)");
    // the staging overwrites whatever layout another sampler left in b_ws
    // (node-wise / PinSAGE / layer-wise keep zeroed bitmaps there between
    // calls): invalidate it so their next launch on this object re-clears it
    blk->ws_kind_prev = 0;
    blk->ws_stride_prev = -1;
    P.stage_row = (int32_t*)blk->b_ws.ptr;
    P.stage_eid = (int64_t*)((char*)blk->b_ws.ptr + o_e);
    P.ustart = (int64_t*)((char*)blk->b_ws.ptr + o_s);
  }
  GS_CUDA_TRY(cudaLaunchKernelEx(&cfg, shadow_induce_kernel, P));
  count_launch();
  return GS_OK;
}

gs_status run_induce(const gs_graph* g, const gs_blocks* nw, cudaStream_t stream, gs_blocks* blk);

gs_status run_shadow(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                     int64_t batch_size, int64_t batch_base, const int32_t* fanouts, int L,
                     int bias, uint64_t key, cudaStream_t stream, gs_blocks* blk) {
  int CS = 1;
  int64_t bpc = 0;
  gs_status st = induce_envelope(g->num_nodes, &CS, &bpc);
  if (st) return st;
  // 1. node-wise sampling of every hop (internal result object)
  if (!blk->aux) {
    blk->aux = new (std::nothrow) gs_blocks();
    if (!blk->aux) return fail(GS_ERR_OUT_OF_MEMORY, "host allocation failed");
    blk->aux->al = blk->al;
  }
  blk->aux->stream = stream;
  st = run_nodewise(g, seeds, num_seeds, batch_size, batch_base, fanouts, L, 0, bias, key,
                         stream, blk->aux);
  if (st) return st;
  return run_induce(g, blk->aux, stream, blk);
}

// Induce (a7; R12) over a node-wise result: per batch U = its
// seeds + every hop's rows, ascending; the subgraph of A induced on U.
gs_status run_induce(const gs_graph* g, const gs_blocks* nw, cudaStream_t stream, gs_blocks* blk) {
  int CS = 1;
  int64_t bpc = 0;
  gs_status st = induce_envelope(g->num_nodes, &CS, &bpc);
  if (st) return st;
  if (nw->kind != gs_blocks::NODEWISE || (nw->num_seeds <= 0 && nw->num_batches > 0))
    return fail(GS_ERR_INVALID_ARGUMENT, "induce: the sampled blocks must be a node-wise result");
  const int L = nw->num_layers;
  const int64_t num_seeds = nw->num_seeds;
  int64_t sumK = 0;
  SHParams P = {};
  P.seeds = nw->layers[0].col_map;
  P.num_seeds = num_seeds;
  P.batch_size = nw->batch_size;
  P.bptr = nw->bptr_dev;
  P.L = L;
  for (int l = 0; l < L; ++l) {
    P.rows[l] = nw->layers[l].row_map;
    P.K[l] = num_seeds > 0 ? nw->layers[l].row_capacity / num_seeds : 0;
    sumK += P.K[l];
  }
  P.nmeta = (const int64_t*)nw->b_meta.ptr;
  return launch_induce(g, P, CS, bpc, nw->num_batches, 1 + sumK, (const int*)nw->b_err.ptr, stream, blk);
}

// GraphSAINT-RW (Table 2; R26): a DeepWalk walk from every root
// (walk.cu, global walker ids batch_base * batch_size + i), then per batch the
// subgraph induced on the nodes its walks visited.  The traces stay in HBM
// between the two launches (4 B per visited slot, written once, read once).
gs_status run_saint_rw(const gs_graph* g, const int32_t* roots, int64_t num_roots,
                       int64_t batch_size, int64_t batch_base, int walk_length, uint64_t key,
                       cudaStream_t stream, gs_blocks* blk) {
  int CS = 1;
  int64_t bpc = 0;
  gs_status st = induce_envelope(g->num_nodes, &CS, &bpc);
  if (st) return st;
  const int64_t L1 = (int64_t)walk_length + 1;
  const int64_t nbatch = (num_roots + batch_size - 1) / batch_size;
  const int64_t tr_bytes = (num_roots * L1 * 4 + 255) & ~int64_t(255);
  if (!blk->b_trace.ensure(blk->al, (size_t)(tr_bytes + 256), stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (GraphSAINT-RW traces)");
  int* werr = (int*)((char*)blk->b_trace.ptr + tr_bytes);  // the walk's own error word (not the graph's)
  GS_CUDA_TRY(cudaMemsetAsync(werr, 0, 4, stream));
  st = launch_walk(g, roots, num_roots, batch_base * batch_size, walk_length, 1.0f, 1.0f, key,
                   false, false, stream, (int32_t*)blk->b_trace.ptr, werr);
  if (st) return st;
  SHParams P = {};
  P.seeds = roots;
  P.num_seeds = num_roots;
  P.batch_size = batch_size;
  P.traces = (const int32_t*)blk->b_trace.ptr;
  P.L1 = L1;
  return launch_induce(g, P, CS, bpc, nbatch, L1, werr, stream, blk);
}

}  // namespace gsb
