// pinsage.cu -- PinSAGE-style sampling (Table 2: "random walks ...
// using restarts, select top-k visited neighbors as sampled nodes"; R27).
//
// One persistent kernel per call; a CTA owns one mini-batch at a time and runs
// all its layers.  Per (batch, layer) with frontier F:
//   W  walks: the frontier is cut into chunks of C columns whose visit-count
//      hash tables (HCAP >= 2 * num_walks * walk_length entries each, linear
//      probing, shared memory) fit the CTA's shared memory; every thread runs
//      the flat (column, walk) pairs of the chunk -- one Philox call, the
//      current node's indptr pair and one index gather per step -- and counts
//      each visit of x != v with a shared-memory atomicAdd;
//   S  select: a warp per column takes the k most visited entries (count
//      descending, id ascending) -- a warp bitonic sort of the (<= 32)
//      visited nodes, else k rounds of a warp arg-max -- writes them
//      (count, id) to the layer's eid region as scratch at column-major
//      positions j*k + r, and marks the ids in the CTA's N-bit row bitmap
//      (global memory, L2-resident, left cleared after every layer);
//   F  finalize: CSC indptr by a block scan of the per-column counts; a
//      popcount prefix per 4 bitmap words (global, per CTA); row_local =
//      rank of the id (prefix + popc of the words before it in its group +
//      popc below it in its word), val = fp32(count); row_map = the set bits
//      in ascending order (R3), clearing the bitmap as it goes; eid = -1.
//   The next layer's frontier is this row_map (R2).
// No host sync and no capacity overflow: every (batch, layer) has a fixed
// padded region (T_l * k_l edges, T_l = batch_size * prod k_m over m < l).
#include <algorithm>
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "gs_internal.h"

namespace gsb {

constexpr uint32_t TAG_PINSAGE = 7;
constexpr int PS_THREADS = 512;
constexpr int PS_WARPS = PS_THREADS / 32;
constexpr int PS_SMEM = 48 * 1024;   // hash tables of one chunk (4 CTAs per SM fit)
constexpr int PS_GROUP = 4;          // bitmap words per prefix entry (one uint4; the relabel relies on it)
constexpr int PS_ILP = 2;            // walks per thread in lockstep

struct PSParams {
  const int64_t* indptr;
  const int32_t* indices;
  int64_t N;
  const int32_t* seeds;
  int64_t num_seeds, batch_size, num_batches, batch_base;
  int L;
  int k[MAX_LAYERS];
  int num_walks, walk_length;
  float restart;
  uint64_t key;
  int hlog;                          // log2 HCAP
  int chunk;                         // columns per chunk
  // per layer: padded regions per batch
  int64_t colcap[MAX_LAYERS], edgecap[MAX_LAYERS];
  int32_t* col0;                     // layer-0 col_map (the seeds) [b * colcap0]
  int32_t* row[MAX_LAYERS];          // row_map [b * edgecap]
  int64_t* ip[MAX_LAYERS];           // indptr [b * (colcap + 1)]
  int32_t* rowl[MAX_LAYERS];         // row_local [b * edgecap]
  int64_t* eid[MAX_LAYERS];          // eid [b * edgecap] (scratch: (count << 32) | id)
  float* val[MAX_LAYERS];            // val [b * edgecap] = visit count
  int64_t* meta;                     // [b][L][8]
  uint32_t* bitmap;                  // [CTA][nwords]
  int32_t* gprefix;                  // [CTA][ngroups]
  int64_t nwords, ngroups;
  int* err;
  unsigned int* claim;
};

__device__ __forceinline__ uint32_t ps_hash(uint32_t x) {
  x ^= x >> 16;
  x *= 0x7feb352du;
  x ^= x >> 15;
  x *= 0x846ca68bu;
  x ^= x >> 16;
  return x;
}

__global__ void __launch_bounds__(PS_THREADS) pinsage_kernel(PSParams P) {
  extern __shared__ __align__(16) int32_t ps_smem[];
  __shared__ long long s_b;
  __shared__ int scr[40];
  __shared__ long long scr64[40];
  __shared__ unsigned long long wstage[PS_WARPS * 32];  // per-warp top-k staging
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  // L2 policies: the walks' random reads evict-first, the CTA's row bitmap
  // (148 x N/8 bytes) evict-last
  const uint64_t pfw = pol_first(), pkw = pol_last();
  const int HCAP = 1 << P.hlog;
  const int C = P.chunk;
  int32_t* hkey = ps_smem;             // [C][HCAP]
  int32_t* hcnt = ps_smem + C * HCAP;  // [C][HCAP]
  uint32_t* bm = P.bitmap + (int64_t)blockIdx.x * P.nwords;
  int32_t* gp = P.gprefix + (int64_t)blockIdx.x * P.ngroups;
  const int W = P.num_walks, T = P.walk_length;
  for (int i = tid; i < C * HCAP; i += PS_THREADS) {
    hkey[i] = -1;
    hcnt[i] = 0;
  }
  while (true) {
    if (tid == 0) s_b = (long long)atomicAdd(P.claim, 1u);
    __syncthreads();
    const long long b = s_b;
    __syncthreads();
    if (b >= P.num_batches) break;
    const uint32_t gb = (uint32_t)(P.batch_base + b);
    const int64_t bstart = b * P.batch_size;
    long long nF = min((long long)P.batch_size, (long long)(P.num_seeds - bstart));
    // layer-0 frontier: the batch's seeds (copied to col_map, range-checked)
    for (long long j = tid; j < nF; j += PS_THREADS) {
      const int32_t v = __ldg(P.seeds + bstart + j);
      P.col0[b * P.colcap[0] + j] = v;
      if (v < 0 || (int64_t)v >= P.N) atomicOr(P.err, ERR_SEED_RANGE);
    }
    __syncthreads();
    const int32_t* F = P.col0 + b * P.colcap[0];
    long long Foff = b * P.colcap[0];
    for (int l = 0; l < P.L; ++l) {
      const int k = P.k[l];
      const int64_t ebase = b * P.edgecap[l];
      int64_t* scratch = P.eid[l] + ebase;       // (count << 32) | id at j*k + r
      int64_t* ip = P.ip[l] + b * (P.colcap[l] + 1);
      // ---- W + S: walks and top-k, one chunk of columns at a time ----
      for (long long c0 = 0; c0 < nF; c0 += C) {
        const int nc = (int)min((long long)C, nF - c0);
        const int npairs = nc * W;
        // PS_ILP independent walks per thread advance in lockstep, so their
        // dependent loads (indptr pair, then the index) overlap
        for (int i = tid; i < npairs; i += PS_ILP * PS_THREADS) {
          int32_t wv[PS_ILP], wx[PS_ILP];
          int wcol[PS_ILP], ww[PS_ILP];
          bool alive[PS_ILP];
#pragma unroll
          for (int a = 0; a < PS_ILP; ++a) {
            const int ia = i + a * PS_THREADS;
            alive[a] = ia < npairs;
            wcol[a] = alive[a] ? ia / W : 0;
            ww[a] = ia - wcol[a] * W;
            wv[a] = alive[a] ? __ldcg(F + c0 + wcol[a]) : 0;
            if (wv[a] < 0 || (int64_t)wv[a] >= P.N) alive[a] = false;
            wx[a] = wv[a];
          }
          for (int t = 1; t <= T; ++t) {
            U4 r[PS_ILP];
            int64_t off[PS_ILP], d[PS_ILP];
#pragma unroll
            for (int a = 0; a < PS_ILP; ++a) {
              r[a] = philox((uint32_t)wv[a], (uint32_t)(ww[a] * T + t - 1), ctr2(l, TAG_PINSAGE), gb, P.key);
              if ((float)(r[a].z >> 8) * 0x1p-24f < P.restart) alive[a] = false;  // restart at v (R27)
              off[a] = alive[a] ? ldg_h64(P.indptr + wx[a], pfw) : 0;
              d[a] = alive[a] ? ldg_h64(P.indptr + wx[a] + 1, pfw) : 0;
            }
            bool any = false;
#pragma unroll
            for (int a = 0; a < PS_ILP; ++a) {
              d[a] -= off[a];
              if (d[a] == 0) alive[a] = false;            // dead end (R13)
              if (alive[a]) wx[a] = ldg_h(P.indices + off[a] + (int64_t)draw_below((uint64_t)d[a], r[a].x, r[a].y), pfw);
              any |= alive[a];
            }
            if (!any) break;
#pragma unroll
            for (int a = 0; a < PS_ILP; ++a) {
              if (!alive[a] || wx[a] == wv[a]) continue;
              int32_t* tk = hkey + wcol[a] * HCAP;
              int32_t* tc = hcnt + wcol[a] * HCAP;
              uint32_t h = ps_hash((uint32_t)wx[a]) & (uint32_t)(HCAP - 1);
              while (true) {
                const int32_t old = atomicCAS(tk + h, -1, wx[a]);
                if (old == -1 || old == wx[a]) {
                  atomicAdd(tc + h, 1);
                  break;
                }
                h = (h + 1) & (uint32_t)(HCAP - 1);
              }
            }
          }
        }
        __syncthreads();
        for (int cj = warp; cj < nc; cj += PS_WARPS) {
          int32_t* tk = hkey + cj * HCAP;
          int32_t* tc = hcnt + cj * HCAP;
          const long long j = c0 + cj;
          int taken = 0;
          // fast path: at most 32 visited nodes -> one key per lane, a warp
          // bitonic sort (15 compare-exchange steps) instead of k arg-max rounds
          unsigned long long* st = wstage + warp * 32;
          int nv = 0;
          for (int e0 = 0; e0 < HCAP; e0 += 32) {
            const int e = e0 + lane;
            const int cnt = tc[e];
            const unsigned bal = __ballot_sync(0xffffffffu, cnt > 0);
            if (cnt > 0) {
              const int pos = nv + __popc(bal & ((1u << lane) - 1u));
              if (pos < 32)
                st[pos] = ((unsigned long long)(uint32_t)cnt << 32) | (uint32_t)(0x7FFFFFFF - tk[e]);
            }
            nv += __popc(bal);
          }
          __syncwarp();
          if (nv <= 32) {
            // ascending sort of ~key == descending (count, -id)
            unsigned long long key = lane < nv ? ~st[lane] : ~0ull;
#pragma unroll
            for (int kk = 2; kk <= 32; kk <<= 1) {
#pragma unroll
              for (int jj = kk >> 1; jj > 0; jj >>= 1) {
                const unsigned long long o = __shfl_xor_sync(0xffffffffu, key, jj);
                const bool asc = (lane & kk) == 0, low = (lane & jj) == 0;
                key = (low == asc) ? (o < key ? o : key) : (o > key ? o : key);
              }
            }
            taken = min(k, nv);
            if (lane < taken) {
              const unsigned long long kv = ~key;
              const int32_t id = 0x7FFFFFFF - (int32_t)(uint32_t)kv;
              scratch[j * k + lane] = ((int64_t)(kv >> 32) << 32) | (uint32_t)id;
              asm volatile("red.global.or.L2::cache_hint.b32 [%0], %1, %2;" ::"l"(bm + (id >> 5)),
                           "r"(1u << (id & 31)), "l"(pkw) : "memory");
            }
          }
          __syncwarp();
          if (nv > 32)
          for (; taken < k; ++taken) {
            // best entry of this lane: count descending, id ascending
            unsigned long long best = 0;
            int bpos = -1;
            for (int e = lane; e < HCAP; e += 32) {
              const int cnt = tc[e];
              if (cnt > 0) {
                const unsigned long long kk =
                    ((unsigned long long)(uint32_t)cnt << 32) | (uint32_t)(0x7FFFFFFF - tk[e]);
                if (kk > best) {
                  best = kk;
                  bpos = e;
                }
              }
            }
            unsigned long long m = best;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
              const unsigned long long y = __shfl_xor_sync(0xffffffffu, m, o);
              m = y > m ? y : m;
            }
            if (m == 0) break;
            if (best == m && bpos >= 0) {  // unique owner: ids are distinct
              const int32_t id = tk[bpos];
              scratch[j * k + taken] = ((int64_t)(uint32_t)tc[bpos] << 32) | (uint32_t)id;
              tc[bpos] = 0;
              asm volatile("red.global.or.L2::cache_hint.b32 [%0], %1, %2;" ::"l"(bm + (id >> 5)),
                           "r"(1u << (id & 31)), "l"(pkw) : "memory");
            }
            __syncwarp();
          }
          if (lane == 0) ip[j + 1] = taken;  // count, scanned below
          for (int e = lane; e < HCAP; e += 32) {
            tk[e] = -1;
            tc[e] = 0;
          }
        }
        __syncthreads();
      }
      // ---- F: CSC indptr (block scan of the per-column counts) ----
      long long run = 0;
      for (long long j0 = 0; j0 < nF; j0 += PS_THREADS) {
        const long long j = j0 + tid;
        const long long x = j < nF ? ip[j + 1] : 0;
        long long tot;
        const long long ex = block_exclusive_scan<long long>(x, scr64, &tot);
        if (j < nF) ip[j + 1] = run + ex + x;
        run += tot;
      }
      if (tid == 0) ip[0] = 0;
      const long long E = run;
      // ---- popcount prefix per group of PS_GROUP bitmap words ----
      long long rrun = 0;
      for (long long g0 = 0; g0 < P.ngroups; g0 += PS_THREADS) {
        const long long g = g0 + tid;
        int c = 0;
        if (g < P.ngroups) {
          const uint4* w4 = reinterpret_cast<const uint4*>(bm + g * PS_GROUP);
#pragma unroll
          for (int q = 0; q < PS_GROUP / 4; ++q) {
            const uint4 u = __ldcg(w4 + q);
            c += __popc(u.x) + __popc(u.y) + __popc(u.z) + __popc(u.w);
          }
        }
        int tot;
        const int ex = block_exclusive_scan<int>(c, scr, &tot);
        if (g < P.ngroups) gp[g] = (int32_t)(rrun + ex);
        rrun += tot;
      }
      const long long R = rrun;
      __syncthreads();
      // ---- relabel: row_local = rank of the id, val = count ----
      int32_t* rowl = P.rowl[l] + ebase;
      float* val = P.val[l] + ebase;
      // flat over the (column, rank) slots so every lane works; the rank of
      // an id = its group prefix + popc of the group's words below it (one
      // 16-byte load of the group, issued beside the prefix load)
      for (long long t = tid; t < nF * k; t += PS_THREADS) {
        const long long j = t / k, r = t - j * k;
        const long long p0 = ip[j];
        if (r < ip[j + 1] - p0) {
          const int64_t sv = scratch[t];
          const int32_t id = (int32_t)(uint32_t)sv;
          const long long g = id >> 7;  // PS_GROUP (4) words x 32 bits
          const int base = __ldcg(gp + g);
          const uint4 w4 = __ldcg(reinterpret_cast<const uint4*>(bm) + g);
          const int q = (id >> 5) & 3;
          const uint32_t below = (1u << (id & 31)) - 1u;
          int rank = base;
          rank += q > 0 ? __popc(w4.x) : __popc(w4.x & below);
          if (q >= 1) rank += q > 1 ? __popc(w4.y) : __popc(w4.y & below);
          if (q >= 2) rank += q > 2 ? __popc(w4.z) : __popc(w4.z & below);
          if (q >= 3) rank += __popc(w4.w & below);
          rowl[p0 + r] = rank;
          val[p0 + r] = (float)(uint32_t)(sv >> 32);
        }
      }
      __syncthreads();
      // ---- row_map = set bits ascending; bitmap cleared; eid = -1 ----
      int32_t* rowm = P.row[l] + ebase;
      for (long long g = tid; g < P.ngroups; g += PS_THREADS) {
        long long r = __ldcg(gp + g);
        for (int q = 0; q < PS_GROUP; ++q) {
          uint32_t m = __ldcg(bm + g * PS_GROUP + q);
          if (!m) continue;
          bm[g * PS_GROUP + q] = 0u;
          while (m) {
            const int bit = __ffs(m) - 1;
            m &= m - 1u;
            rowm[r++] = (int32_t)((g * PS_GROUP + q) * 32 + bit);
          }
        }
      }
      for (long long e = tid; e < E; e += PS_THREADS) scratch[e] = -1;
      if (tid == 0) {
        long long* m = (long long*)(P.meta + (b * P.L + l) * 8);
        m[0] = nF; m[1] = R; m[2] = E; m[3] = Foff;
        m[4] = ebase; m[5] = b * (P.colcap[l] + 1); m[6] = ebase; m[7] = 0;
      }
      __syncthreads();
      F = rowm;
      Foff = ebase;
      nF = R;
    }
  }
}

gs_status run_pinsage(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                      int64_t batch_size, int64_t batch_base, const int32_t* topk, int L,
                      int num_walks, int walk_length, float restart, uint64_t key,
                      cudaStream_t stream, gs_blocks* blk) {
  const Allocator& al = blk->al;
  const int64_t nbatch = (num_seeds + batch_size - 1) / batch_size;
  blk->kind = gs_blocks::NODEWISE;
  blk->num_batches = nbatch;
  blk->num_layers = L;
  blk->stream = stream;
  blk->synced = false;
  PSParams P = {};
  P.indptr = g->indptr;
  P.indices = g->indices;
  P.N = g->num_nodes;
  P.seeds = seeds;
  P.num_seeds = num_seeds;
  P.batch_size = batch_size;
  P.num_batches = nbatch;
  P.batch_base = batch_base;
  P.L = L;
  P.num_walks = num_walks;
  P.walk_length = walk_length;
  P.restart = restart;
  P.key = key;
  int hlog = 5;
  while ((1 << hlog) < 2 * num_walks * walk_length) ++hlog;
  P.hlog = hlog;
  P.chunk = std::max(1, PS_SMEM / ((1 << hlog) * 8));
  auto need = [&](DevBuf& b, int64_t bytes) -> bool {
    return b.ensure(al, (size_t)std::max<int64_t>(bytes, 256), stream);
  };
  int64_t cols = batch_size;
  for (int l = 0; l < L; ++l) {
    P.k[l] = topk[l];
    P.colcap[l] = cols;
    P.edgecap[l] = cols * topk[l];
    const int64_t E = nbatch * P.edgecap[l];
    bool ok = need(blk->b_row[l], E * 4) && need(blk->b_indptr[l], nbatch * (cols + 1) * 8) &&
              need(blk->b_rowl[l], E * 4) && need(blk->b_eid[l], E * 8) && need(blk->b_val[l], E * 4);
    if (l == 0) ok = ok && need(blk->b_col[0], nbatch * cols * 4);
    if (!ok) return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (PinSAGE layer %d)", l);
    gs_layer_buffers& lb = blk->layers[l];
    lb = gs_layer_buffers{};
    lb.col_map = l == 0 ? (int32_t*)blk->b_col[0].ptr : blk->layers[l - 1].row_map;
    lb.col_capacity = l == 0 ? nbatch * cols : blk->layers[l - 1].row_capacity;
    lb.row_map = (int32_t*)blk->b_row[l].ptr;
    lb.row_capacity = E;
    lb.indptr = (int64_t*)blk->b_indptr[l].ptr;
    lb.indptr_capacity = nbatch * (cols + 1);
    lb.row_local = (int32_t*)blk->b_rowl[l].ptr;
    lb.eid = (int64_t*)blk->b_eid[l].ptr;
    lb.val = (float*)blk->b_val[l].ptr;
    lb.edge_capacity = E;
    P.row[l] = lb.row_map;
    P.ip[l] = lb.indptr;
    P.rowl[l] = lb.row_local;
    P.eid[l] = lb.eid;
    P.val[l] = lb.val;
    cols = P.edgecap[l];
  }
  P.col0 = blk->layers[0].col_map;
  if (!need(blk->b_meta, std::max<int64_t>(nbatch, 1) * L * 64) || !need(blk->b_err, 16) ||
      !need(blk->b_ctr, 8 * (MAX_LAYERS + 2)))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (PinSAGE meta)");
  P.meta = (int64_t*)blk->b_meta.ptr;
  P.err = (int*)blk->b_err.ptr;
  P.claim = (unsigned int*)blk->b_ctr.ptr;
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_err.ptr, 0, 16, stream));
  GS_CUDA_TRY(cudaMemsetAsync(blk->b_ctr.ptr, 0, 8 * (MAX_LAYERS + 2), stream));
  if (nbatch == 0) return GS_OK;

  const size_t smem = (size_t)P.chunk * (1 << hlog) * 8;
  GS_CUDA_TRY(cudaFuncSetAttribute(pinsage_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int dev = 0, sms = 148, per_sm = 1;
  GS_CUDA_TRY(cudaGetDevice(&dev));
  GS_CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  GS_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, pinsage_kernel, PS_THREADS, smem));
  // per-CTA row bitmap + group prefix (left cleared by every layer; zeroed
  // whenever the workspace is (re)allocated or last served another kernel)
  P.nwords = ((g->num_nodes + 31) / 32 + PS_GROUP - 1) / PS_GROUP * PS_GROUP;
  P.ngroups = P.nwords / PS_GROUP;
  const int64_t per_cta = P.nwords * 4 + P.ngroups * 4;
  int64_t grid = std::min<int64_t>((int64_t)sms * std::max(per_sm, 1), nbatch);
  const int64_t budget = int64_t(4) << 30;  // bitmap workspace cap
  grid = std::max<int64_t>(1, std::min<int64_t>(grid, budget / per_cta));
  const int64_t ws = grid * per_cta;
  const int64_t layout = P.nwords * 65536 + grid;  // the prefix region follows grid bitmaps
  const bool fresh = !blk->b_ws.ptr || blk->b_ws.bytes < (size_t)ws || blk->ws_kind_prev != 9 ||
                     blk->ws_stride_prev != layout;
  if (!blk->b_ws.ensure(al, (size_t)ws, stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (PinSAGE bitmaps)");
  if (fresh) GS_CUDA_TRY(cudaMemsetAsync(blk->b_ws.ptr, 0, blk->b_ws.bytes, stream));
  blk->ws_kind_prev = 9;
  blk->ws_stride_prev = layout;
  P.bitmap = (uint32_t*)blk->b_ws.ptr;
  P.gprefix = (int32_t*)((char*)blk->b_ws.ptr + grid * P.nwords * 4);
  pinsage_kernel<<<(unsigned)grid, PS_THREADS, smem, stream>>>(P); count_launch();
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

}  // namespace gsb
