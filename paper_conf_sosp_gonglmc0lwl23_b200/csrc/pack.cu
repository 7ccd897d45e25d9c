// pack.cu -- gs_blocks_pack: one layer of every mini-batch packed into dense,
// batch-ordered device arrays, so that a host copy moves exactly the sampled
// blocks (the sampling kernels write each batch into a fixed, padded region,
// DESIGN.md section 5).  Two kernels on the caller's stream, no host sync:
// an exclusive scan of the per-batch counts over batches (one CTA), then a
// grid-stride copy: CTA (x, y) copies slice y of every gridDim.x-th
// mini-batch (a few batches still spread over the whole GPU).
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "common.cuh"
#include "gs_internal.h"

namespace gsb {

constexpr int PK_THREADS = 512;

// off[b] = (edges, indptr entries, rows) before batch b; off[nb] = totals.
__global__ void __launch_bounds__(PK_THREADS) pack_scan_kernel(const int64_t* __restrict__ meta, int64_t nb,
                                                               int L, int layer, int64_t* __restrict__ off,
                                                               int64_t* __restrict__ totals) {
  __shared__ long long scr[33];
  long long run[3] = {0, 0, 0};
  for (int64_t b0 = 0; b0 < nb; b0 += PK_THREADS) {
    const int64_t b = b0 + threadIdx.x;
    long long v[3] = {0, 0, 0};
    if (b < nb) {
      const int64_t* m = meta + (b * L + layer) * GS_META_FIELDS;
      v[0] = m[2];
      v[1] = m[0] + 1;  // a block's indptr has n_cols + 1 entries
      v[2] = m[1];
    }
    for (int f = 0; f < 3; ++f) {
      long long tot;
      const long long ex = block_exclusive_scan<long long>(v[f], scr, &tot);
      if (b < nb) off[b * 3 + f] = run[f] + ex;
      run[f] += tot;
    }
  }
  if (threadIdx.x == 0) {
    for (int f = 0; f < 3; ++f) {
      off[nb * 3 + f] = run[f];
      totals[f] = run[f];
    }
  }
}

struct PackParams {
  const int64_t* meta;
  int64_t nb;
  int L, layer;
  const int64_t* off;
  const int32_t* row_local_in;
  const int64_t* eid_in;
  const int64_t* indptr_in;
  const int32_t* row_map_in;
  int32_t* row_local;
  void* eid;       // int64 (or int32: narrow)
  void* indptr;    // int64 (or int32: narrow)
  int32_t* row_map;
  int64_t edge_cap, indptr_cap, row_cap;  // the layer buffers' capacities (copies are clamped)
};

template <bool NARROW>
__global__ void __launch_bounds__(PK_THREADS) pack_copy_kernel(PackParams P) {
  const int64_t t0 = (int64_t)blockIdx.y * PK_THREADS + threadIdx.x, ts = (int64_t)gridDim.y * PK_THREADS;
  for (int64_t b = blockIdx.x; b < P.nb; b += gridDim.x) {
    const int64_t* m = P.meta + (b * P.L + P.layer) * GS_META_FIELDS;
    // clamped to the layer buffers: a block recorded past them is never read
    const int64_t E = min(m[2], max(P.edge_cap - m[6], (int64_t)0));
    const int64_t T = min(m[0], max(P.indptr_cap - m[5] - 1, (int64_t)-1));
    const int64_t R = min(m[1], max(P.row_cap - m[4], (int64_t)0));
    const int64_t* o = P.off + b * 3;
    const int64_t eo = o[0], io = o[1], ro = o[2];
    for (int64_t i = t0; i < E; i += ts) {
      P.row_local[eo + i] = __ldcs(P.row_local_in + m[6] + i);
      const int64_t e = __ldcs(P.eid_in + m[6] + i);
      if (NARROW) ((int32_t*)P.eid)[eo + i] = (int32_t)e;
      else ((int64_t*)P.eid)[eo + i] = e;
    }
    for (int64_t i = t0; i <= T; i += ts) {
      const int64_t x = __ldcs(P.indptr_in + m[5] + i);
      if (NARROW) ((int32_t*)P.indptr)[io + i] = (int32_t)x;  // block-relative (<= 2^25)
      else ((int64_t*)P.indptr)[io + i] = x;
    }
    for (int64_t i = t0; i < R; i += ts) P.row_map[ro + i] = __ldcs(P.row_map_in + m[4] + i);
  }
}

}  // namespace gsb

using namespace gsb;

static gs_status pack_impl(const gs_blocks* b, int layer, int32_t* row_local, void* eid, void* indptr,
                           int32_t* row_map, int64_t* totals, void* stream_, bool narrow) {
  cudaStream_t stream = (cudaStream_t)stream_;
  if (!b || !row_local || !eid || !indptr || !row_map || !totals)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_blocks_pack: null argument");
  if (layer < 0 || layer >= b->num_layers) return fail(GS_ERR_INVALID_ARGUMENT, "gs_blocks_pack: bad layer");
  gs_blocks* mb = const_cast<gs_blocks*>(b);
  const int64_t nb = b->num_batches;
  if (!mb->b_pack.ensure(mb->al, (size_t)std::max<int64_t>((nb + 1) * 3 * 8, 256), stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "gs_blocks_pack: device allocation failed");
  const gs_layer_buffers& lb = b->layers[layer];
  int64_t* off = (int64_t*)mb->b_pack.ptr;
  pack_scan_kernel<<<1, PK_THREADS, 0, stream>>>((const int64_t*)b->b_meta.ptr, nb, b->num_layers, layer,
                                                 off, totals); count_launch();
  GS_CUDA_TRY(cudaGetLastError());
  if (nb == 0) return GS_OK;
  PackParams P;
  P.meta = (const int64_t*)b->b_meta.ptr;
  P.nb = nb;
  P.L = b->num_layers;
  P.layer = layer;
  P.off = off;
  P.row_local_in = lb.row_local;
  P.eid_in = lb.eid;
  P.indptr_in = lb.indptr;
  P.row_map_in = lb.row_map;
  P.row_local = row_local;
  P.eid = eid;
  P.indptr = indptr;
  P.row_map = row_map;
  P.edge_cap = lb.edge_capacity;
  P.indptr_cap = lb.indptr_capacity;
  P.row_cap = lb.row_capacity;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int64_t gx = std::min<int64_t>(nb, (int64_t)sms * 4);
  const int64_t gy = std::max<int64_t>(1, std::min<int64_t>(64, ((int64_t)sms * 8 + gx - 1) / gx));
  const dim3 grid((unsigned)gx, (unsigned)gy);
  if (narrow) pack_copy_kernel<true><<<grid, PK_THREADS, 0, stream>>>(P);
  else pack_copy_kernel<false><<<grid, PK_THREADS, 0, stream>>>(P);
  count_launch();
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

extern "C" gs_status gs_blocks_pack(const gs_blocks* b, int layer, int32_t* row_local, int64_t* eid,
                                    int64_t* indptr, int32_t* row_map, int64_t* totals, void* stream) {
  return pack_impl(b, layer, row_local, eid, indptr, row_map, totals, stream, false);
}

extern "C" gs_status gs_blocks_pack_narrow(const gs_blocks* b, int layer, int32_t* row_local, int32_t* eid,
                                           int32_t* indptr, int32_t* row_map, int64_t* totals, void* stream) {
  if (b && b->graph_edges >= (int64_t(1) << 31))
    return fail(GS_ERR_NOT_SUPPORTED, "gs_blocks_pack_narrow: the graph has >= 2^31 edges (int32 edge ids)");
  return pack_impl(b, layer, row_local, eid, indptr, row_map, totals, stream, true);
}
