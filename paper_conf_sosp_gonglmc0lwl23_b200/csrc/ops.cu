// ops.cu -- the matrix-centric operators of Table 4 as standalone
// device operators on a materialised sub-matrix (gs_matrix): the general layer
// a new sampling algorithm composes when no fused sampler exists (SURVEY 8(f)
// f3).  The fused samplers (nodewise_wave.cu, layerwise*.cu, ...) never
// materialise these intermediates (Extract-Select / Edge-MapReduce fusion,
// P:289-294); this layer is the unfused reference path of the same algebra.
//
//   A[:, cols]      degree gather + CUB-free multi-block scan + a flat copy of
//                   each 32-column group's slices (indices, edge ids, weights)
//   A[rows, :]      N-bit row bitmap, warp ballot count + scan + compaction
//   A.sum(axis)     axis 0: warp shuffle fp64 reduction per column; axis 1:
//                   fp64 atomics into a dense per-node accumulator (R1, R19)
//   A.<op>(V, axis) in-place broadcast (axis 0: V per local column, 1: per row id)
//   A <op> v        in-place element-wise map (+ - * / **)
//   A.row()         row bitmap -> popcount scan over words -> ascending ids (R3)
// All HBM streaming kernels; grids are multiples of the SM count.
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <new>

#include "common.cuh"
#include "gs_internal.h"

struct gs_matrix {
  gsb::Allocator al;
  int64_t num_nodes = 0, n_cols = 0, nnz = 0;
  gsb::DevBuf b_cols, b_indptr, b_row, b_eid, b_val;
};

namespace gsb {

constexpr int OPS_THREADS = 512;
constexpr int SCAN_THREADS = 1024;
constexpr int SCAN_ITEMS = 4;
constexpr int64_t SCAN_TILE = SCAN_THREADS * SCAN_ITEMS;

static int sm_count() {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return sms;
}

static unsigned grid_for(int64_t work_items, int per_block) {
  const int64_t want = (work_items + per_block - 1) / per_block;
  const int64_t cap = (int64_t)sm_count() * 8;
  return (unsigned)std::max<int64_t>(1, std::min(want, cap));
}

// ---- inclusive scan of int64 a[0..n) in place (tile scan + tile offsets) ----
__global__ void __launch_bounds__(SCAN_THREADS) scan_tile_kernel(int64_t* a, int64_t n, int64_t* tsum) {
  __shared__ long long scr[40];
  const int64_t base = (int64_t)blockIdx.x * SCAN_TILE + (int64_t)threadIdx.x * SCAN_ITEMS;
  long long v[SCAN_ITEMS];
  long long loc = 0;
#pragma unroll
  for (int i = 0; i < SCAN_ITEMS; ++i) {
    v[i] = base + i < n ? a[base + i] : 0;
    loc += v[i];
    v[i] = loc;  // running inclusive sum of this thread's items
  }
  long long tot;
  const long long ex = block_exclusive_scan<long long>(loc, scr, &tot);
#pragma unroll
  for (int i = 0; i < SCAN_ITEMS; ++i)
    if (base + i < n) a[base + i] = v[i] + ex;
  if (threadIdx.x == 0 && tsum) tsum[blockIdx.x] = tot;
}

__global__ void scan_add_kernel(int64_t* a, int64_t n, const int64_t* tsum_incl) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t t = i / SCAN_TILE;
    if (t > 0) a[i] += tsum_incl[t - 1];
  }
}

static gs_status scan_inclusive(int64_t* a, int64_t n, const Allocator& al, cudaStream_t s) {
  if (n <= 0) return GS_OK;
  const int64_t tiles = (n + SCAN_TILE - 1) / SCAN_TILE;
  if (tiles == 1) {
    scan_tile_kernel<<<1, SCAN_THREADS, 0, s>>>(a, n, nullptr); count_launch();
    GS_CUDA_TRY(cudaGetLastError());
    return GS_OK;
  }
  DevBuf t;
  if (!t.ensure(al, (size_t)tiles * 8, s)) return fail(GS_ERR_OUT_OF_MEMORY, "scan workspace");
  scan_tile_kernel<<<(unsigned)tiles, SCAN_THREADS, 0, s>>>(a, n, (int64_t*)t.ptr); count_launch();
  gs_status st = scan_inclusive((int64_t*)t.ptr, tiles, al, s);
  if (st == GS_OK) {
    scan_add_kernel<<<grid_for(n, 256), 256, 0, s>>>(a, n, (const int64_t*)t.ptr); count_launch();
    if (cudaGetLastError() != cudaSuccess) st = fail(GS_ERR_CUDA, "scan_add_kernel launch");
  }
  t.reset(al, s);
  return st;
}

// ---- A[:, cols] ----
__global__ void col_degree_kernel(const int64_t* __restrict__ indptr, int64_t N, const int32_t* __restrict__ cols,
                                  int64_t n, int64_t* __restrict__ ip, int* err) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = cols[j];
    int64_t d = 0;
    if (v < 0 || (int64_t)v >= N) atomicOr(err, ERR_SEED_RANGE);
    else d = __ldg(indptr + v + 1) - __ldg(indptr + v);
    ip[j + 1] = d;
    if (j == 0) ip[0] = 0;
  }
}

// A warp takes 32 columns at a time: one round trip fetches their ids, indptr
// pairs and output offsets (a lane each); the group's entries are then copied
// as one flat range, 4 per lane in flight, each lane finding its column by a
// 5-step shuffle search over the inclusive degree prefix (no per-column
// dependent-load chain, every lane busy whatever the degrees).
__global__ void __launch_bounds__(OPS_THREADS) col_copy_kernel(const int64_t* __restrict__ indptr,
                                                              const int32_t* __restrict__ indices,
                                                              const float* __restrict__ w, int64_t N,
                                                              const int32_t* __restrict__ cols, int64_t n,
                                                              const int64_t* __restrict__ ip, int32_t* __restrict__ row,
                                                              int64_t* __restrict__ eid, float* __restrict__ val) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t g0 = warp * 32; g0 < n; g0 += nwarps * 32) {
    const int64_t j = g0 + lane;
    const int32_t v = j < n ? __ldg(cols + j) : -1;
    const bool valid = v >= 0 && (int64_t)v < N;
    const int64_t o = valid ? __ldg(indptr + v) : 0;
    const int64_t d = valid ? __ldg(indptr + v + 1) - o : 0;
    const int64_t p = j < n ? __ldg(ip + j) : 0;
    int64_t S = d;  // inclusive prefix of the group's degrees
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      const int64_t y = __shfl_up_sync(0xffffffffu, S, off);
      if (lane >= off) S += y;
    }
    const int64_t D = __shfl_sync(0xffffffffu, S, 31);
    for (int64_t f0 = 0; f0 < D; f0 += 32 * 4) {
      int64_t src[4], dst[4];
      int32_t rv[4];
      float wv[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const int64_t f = f0 + k * 32 + lane;
        int l = 0;  // smallest l with S_l > f
#pragma unroll
        for (int step = 16; step >= 1; step >>= 1) {
          const int64_t sc = __shfl_sync(0xffffffffu, S, l + step - 1);
          if (sc <= f) l += step;
        }
        const int64_t Sl = __shfl_sync(0xffffffffu, S, l & 31), dl = __shfl_sync(0xffffffffu, d, l & 31);
        const int64_t ol = __shfl_sync(0xffffffffu, o, l & 31), pl = __shfl_sync(0xffffffffu, p, l & 31);
        const int64_t r = f - (Sl - dl);
        src[k] = f < D ? ol + r : -1;
        dst[k] = pl + r;
        rv[k] = src[k] >= 0 ? __ldcs(indices + src[k]) : 0;
        wv[k] = (src[k] >= 0 && w) ? __ldcs(w + src[k]) : 1.0f;
      }
#pragma unroll
      for (int k = 0; k < 4; ++k)
        if (src[k] >= 0) {
          row[dst[k]] = rv[k];
          eid[dst[k]] = src[k];
          val[dst[k]] = wv[k];
        }
    }
  }
}

// ---- A[rows, :] ----
__global__ void mark_rows_kernel(const int32_t* __restrict__ rows, int64_t n, int64_t N, uint32_t* bm, int* err) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t u = rows[i];
    if (u < 0 || (int64_t)u >= N) {
      atomicOr(err, ERR_SEED_RANGE);
      continue;
    }
    atomicOr(bm + (u >> 5), 1u << (u & 31));
  }
}

__device__ __forceinline__ bool in_bm(const uint32_t* bm, int32_t u) {
  return (__ldg(bm + (u >> 5)) >> (u & 31)) & 1u;
}

__global__ void __launch_bounds__(OPS_THREADS) row_count_kernel(const int64_t* __restrict__ ip_in,
                                                               const int32_t* __restrict__ row, int64_t n,
                                                               const uint32_t* __restrict__ bm,
                                                               int64_t* __restrict__ ip_out) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t j = warp; j < n; j += nwarps) {
    int64_t cnt = 0;
    for (int64_t i = ip_in[j] + lane; i < ip_in[j + 1]; i += 32) cnt += in_bm(bm, __ldcs(row + i));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
    if (lane == 0) ip_out[j + 1] = cnt;
    if (j == 0 && lane == 0) ip_out[0] = 0;
  }
}

__global__ void __launch_bounds__(OPS_THREADS) row_copy_kernel(const int64_t* __restrict__ ip_in,
                                                              const int32_t* __restrict__ row_in,
                                                              const int64_t* __restrict__ eid_in,
                                                              const float* __restrict__ val_in, int64_t n,
                                                              const uint32_t* __restrict__ bm,
                                                              const int64_t* __restrict__ ip_out,
                                                              int32_t* __restrict__ row, int64_t* __restrict__ eid,
                                                              float* __restrict__ val) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t j = warp; j < n; j += nwarps) {
    int64_t p = ip_out[j];
    const int64_t hi = ip_in[j + 1];
    for (int64_t i0 = ip_in[j]; i0 < hi; i0 += 32) {
      const int64_t i = i0 + lane;
      const int32_t u = i < hi ? __ldcs(row_in + i) : -1;
      const bool keep = u >= 0 && in_bm(bm, u);
      const unsigned bal = __ballot_sync(0xffffffffu, keep);
      if (keep) {
        const int64_t q = p + __popc(bal & ((1u << lane) - 1u));
        row[q] = u;
        eid[q] = eid_in[i];
        val[q] = val_in[i];
      }
      p += __popc(bal);
    }
  }
}

// ---- sums ----
__global__ void __launch_bounds__(OPS_THREADS) col_sum_kernel(const int64_t* __restrict__ ip,
                                                             const float* __restrict__ val, int64_t n,
                                                             float* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t j = warp; j < n; j += nwarps) {
    double s = 0.0;
    for (int64_t i = ip[j] + lane; i < ip[j + 1]; i += 32) s += (double)__ldcs(val + i);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) out[j] = (float)s;
  }
}

__global__ void row_sum_kernel(const int32_t* __restrict__ row, const float* __restrict__ val, int64_t nnz,
                               double* __restrict__ acc) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(acc + __ldcs(row + i), (double)__ldcs(val + i));
}

__global__ void to_float_kernel(const double* __restrict__ acc, int64_t n, float* __restrict__ out) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = (float)acc[i];
}

// ---- maps ----
__device__ __forceinline__ float apply_op(int op, float a, float b) {
  switch (op) {
    case GS_OP_ADD: return __fadd_rn(a, b);
    case GS_OP_SUB: return __fsub_rn(a, b);
    case GS_OP_MUL: return __fmul_rn(a, b);
    case GS_OP_DIV: return __fdiv_rn(a, b);
    default: return (b == 2.0f) ? (float)((double)a * (double)a) : (float)pow((double)a, (double)b);
  }
}

__global__ void __launch_bounds__(OPS_THREADS) bcast_col_kernel(const int64_t* __restrict__ ip, float* val,
                                                               int64_t n, int op, const float* __restrict__ V) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t j = warp; j < n; j += nwarps) {
    const float x = __ldg(V + j);
    for (int64_t i = ip[j] + lane; i < ip[j + 1]; i += 32) val[i] = apply_op(op, val[i], x);
  }
}

__global__ void bcast_row_kernel(const int32_t* __restrict__ row, float* val, int64_t nnz, int op,
                                 const float* __restrict__ V) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x)
    val[i] = apply_op(op, val[i], __ldg(V + __ldcs(row + i)));
}

// 16-byte vectors (val is 256-byte aligned by the allocator), scalar tail
__global__ void map_kernel(float* val, int64_t nnz, int op, float x) {
  float4* v4 = reinterpret_cast<float4*>(val);
  const int64_t n4 = nnz >> 2;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
    float4 a = __ldcs(v4 + i);
    a.x = apply_op(op, a.x, x);
    a.y = apply_op(op, a.y, x);
    a.z = apply_op(op, a.z, x);
    a.w = apply_op(op, a.w, x);
    __stcs(v4 + i, a);
  }
  const int64_t t = (n4 << 2) + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t < nnz) val[t] = apply_op(op, val[t], x);
}

// ---- row() ----
__global__ void mark_all_rows_kernel(const int32_t* __restrict__ row, int64_t nnz, uint32_t* bm) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t u = __ldcs(row + i);
    atomicOr(bm + (u >> 5), 1u << (u & 31));
  }
}

__global__ void word_count_kernel(const uint32_t* __restrict__ bm, int64_t nw, int64_t* __restrict__ cnt) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nw; i += (int64_t)gridDim.x * blockDim.x)
    cnt[i] = __popc(bm[i]);
}

__global__ void emit_rows_kernel(const uint32_t* __restrict__ bm, int64_t nw, const int64_t* __restrict__ incl,
                                 int32_t* __restrict__ out) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nw; i += (int64_t)gridDim.x * blockDim.x) {
    uint32_t m = bm[i];
    int64_t r = incl[i] - __popc(m);
    while (m) {
      const int b = __ffs(m) - 1;
      m &= m - 1u;
      out[r++] = (int32_t)(i * 32 + b);
    }
  }
}

}  // namespace gsb

using namespace gsb;

static gs_status check_err(int* d_err, cudaStream_t s) {
  int h = 0;
  GS_CUDA_TRY(cudaMemcpyAsync(&h, d_err, 4, cudaMemcpyDeviceToHost, s));
  GS_CUDA_TRY(cudaStreamSynchronize(s));
  if (h & ERR_SEED_RANGE) return fail(GS_ERR_INDEX_OUT_OF_RANGE, "a node id is outside [0, N)");
  return GS_OK;
}

static gs_status new_matrix(gs_matrix** out, int64_t N) {
  if (!*out) {
    *out = new (std::nothrow) gs_matrix();
    if (!*out) return fail(GS_ERR_OUT_OF_MEMORY, "host allocation failed");
    (*out)->al = current_allocator();
  }
  (*out)->num_nodes = N;
  return GS_OK;
}

static gs_status alloc_entries(gs_matrix* m, int64_t n_cols, int64_t nnz, cudaStream_t s) {
  const Allocator& al = m->al;
  if (!m->b_cols.ensure(al, (size_t)std::max<int64_t>(n_cols, 1) * 4, s) ||
      !m->b_indptr.ensure(al, (size_t)(n_cols + 1) * 8, s) ||
      !m->b_row.ensure(al, (size_t)std::max<int64_t>(nnz, 1) * 4, s) ||
      !m->b_eid.ensure(al, (size_t)std::max<int64_t>(nnz, 1) * 8, s) ||
      !m->b_val.ensure(al, (size_t)std::max<int64_t>(nnz, 1) * 4, s))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (gs_matrix)");
  m->n_cols = n_cols;
  m->nnz = nnz;
  return GS_OK;
}

extern "C" {

gs_status gs_matrix_slice_columns(const gs_graph* g, const int32_t* cols, int64_t n_cols, void* stream_,
                                  gs_matrix** out) {
  if (!g || !out || (!cols && n_cols > 0) || n_cols < 0)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_matrix_slice_columns: null pointer or negative size");
  cudaStream_t s = (cudaStream_t)stream_;
  gs_status st = new_matrix(out, g->num_nodes);
  if (st) return st;
  gs_matrix* m = *out;
  DevBuf err;
  if (!m->b_indptr.ensure(m->al, (size_t)(n_cols + 1) * 8, s) || !err.ensure(m->al, 16, s))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (gs_matrix indptr)");
  GS_CUDA_TRY(cudaMemsetAsync(err.ptr, 0, 4, s));
  GS_CUDA_TRY(cudaMemsetAsync(m->b_indptr.ptr, 0, 8, s));
  int64_t* ip = (int64_t*)m->b_indptr.ptr;
  if (n_cols > 0) {
    col_degree_kernel<<<grid_for(n_cols, 256), 256, 0, s>>>(g->indptr, g->num_nodes, cols, n_cols, ip, (int*)err.ptr); count_launch();
    GS_CUDA_TRY(cudaGetLastError());
    if ((st = scan_inclusive(ip + 1, n_cols, m->al, s))) return st;
  }
  int64_t nnz = 0;
  GS_CUDA_TRY(cudaMemcpyAsync(&nnz, ip + n_cols, 8, cudaMemcpyDeviceToHost, s));
  if ((st = check_err((int*)err.ptr, s))) {
    err.reset(m->al, s);
    return st;
  }
  err.reset(m->al, s);
  if ((st = alloc_entries(m, n_cols, nnz, s))) return st;
  if (n_cols > 0) GS_CUDA_TRY(cudaMemcpyAsync(m->b_cols.ptr, cols, n_cols * 4, cudaMemcpyDeviceToDevice, s));
  if (n_cols > 0) {
    col_copy_kernel<<<grid_for(n_cols, OPS_THREADS), OPS_THREADS, 0, s>>>(
        g->indptr, g->indices, g->weights, g->num_nodes, cols, n_cols, ip, (int32_t*)m->b_row.ptr,
        (int64_t*)m->b_eid.ptr, (float*)m->b_val.ptr); count_launch();
    GS_CUDA_TRY(cudaGetLastError());
  }
  return GS_OK;
}

gs_status gs_matrix_slice_rows(const gs_matrix* in, const int32_t* rows, int64_t n_rows, void* stream_,
                               gs_matrix** out) {
  if (!in || !out || (!rows && n_rows > 0) || n_rows < 0 || *out == in)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_matrix_slice_rows: null pointer, negative size or in == out");
  cudaStream_t s = (cudaStream_t)stream_;
  gs_status st = new_matrix(out, in->num_nodes);
  if (st) return st;
  gs_matrix* m = *out;
  const int64_t nw = (in->num_nodes + 31) / 32, n = in->n_cols;
  DevBuf bm, err;
  if (!bm.ensure(m->al, (size_t)std::max<int64_t>(nw, 1) * 4, s) || !err.ensure(m->al, 16, s) ||
      !m->b_indptr.ensure(m->al, (size_t)(n + 1) * 8, s))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (row slice)");
  GS_CUDA_TRY(cudaMemsetAsync(bm.ptr, 0, (size_t)std::max<int64_t>(nw, 1) * 4, s));
  GS_CUDA_TRY(cudaMemsetAsync(err.ptr, 0, 4, s));
  GS_CUDA_TRY(cudaMemsetAsync(m->b_indptr.ptr, 0, 8, s));
  int64_t* ip = (int64_t*)m->b_indptr.ptr;
  if (n_rows > 0) {
    mark_rows_kernel<<<grid_for(n_rows, 256), 256, 0, s>>>(rows, n_rows, in->num_nodes, (uint32_t*)bm.ptr, (int*)err.ptr);
    count_launch();
  }
  if (n > 0) {
    row_count_kernel<<<grid_for(n * 32, OPS_THREADS), OPS_THREADS, 0, s>>>(
        (const int64_t*)in->b_indptr.ptr, (const int32_t*)in->b_row.ptr, n, (const uint32_t*)bm.ptr, ip); count_launch();
    GS_CUDA_TRY(cudaGetLastError());
    if ((st = scan_inclusive(ip + 1, n, m->al, s))) return st;
  }
  int64_t nnz = 0;
  GS_CUDA_TRY(cudaMemcpyAsync(&nnz, ip + n, 8, cudaMemcpyDeviceToHost, s));
  st = check_err((int*)err.ptr, s);
  if (st == GS_OK) st = alloc_entries(m, n, nnz, s);
  if (st == GS_OK && n > 0) {
    if (cudaMemcpyAsync(m->b_cols.ptr, in->b_cols.ptr, n * 4, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
      st = fail(GS_ERR_CUDA, "column copy");
    row_copy_kernel<<<grid_for(n * 32, OPS_THREADS), OPS_THREADS, 0, s>>>(
        (const int64_t*)in->b_indptr.ptr, (const int32_t*)in->b_row.ptr, (const int64_t*)in->b_eid.ptr,
        (const float*)in->b_val.ptr, n, (const uint32_t*)bm.ptr, ip, (int32_t*)m->b_row.ptr,
        (int64_t*)m->b_eid.ptr, (float*)m->b_val.ptr); count_launch();
    if (cudaGetLastError() != cudaSuccess) st = fail(GS_ERR_CUDA, "row_copy_kernel launch");
  }
  bm.reset(m->al, s);
  err.reset(m->al, s);
  return st;
}

gs_status gs_matrix_sum(const gs_matrix* m, int axis, float* out, void* stream_) {
  if (!m || (axis != 0 && axis != 1) || (!out && (axis == 0 ? m->n_cols : m->num_nodes) > 0))
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_matrix_sum: bad argument");
  cudaStream_t s = (cudaStream_t)stream_;
  if (axis == 0) {
    if (m->n_cols > 0) {
      col_sum_kernel<<<grid_for(m->n_cols * 32, OPS_THREADS), OPS_THREADS, 0, s>>>(
          (const int64_t*)m->b_indptr.ptr, (const float*)m->b_val.ptr, m->n_cols, out); count_launch();
      GS_CUDA_TRY(cudaGetLastError());
    }
    return GS_OK;
  }
  DevBuf acc;
  const int64_t N = m->num_nodes;
  if (!acc.ensure(m->al, (size_t)std::max<int64_t>(N, 1) * 8, s)) return fail(GS_ERR_OUT_OF_MEMORY, "row-sum accumulator");
  GS_CUDA_TRY(cudaMemsetAsync(acc.ptr, 0, (size_t)std::max<int64_t>(N, 1) * 8, s));
  if (m->nnz > 0) {
    row_sum_kernel<<<grid_for(m->nnz, 256), 256, 0, s>>>((const int32_t*)m->b_row.ptr, (const float*)m->b_val.ptr,
                                                        m->nnz, (double*)acc.ptr);
    count_launch();
  }
  if (N > 0) {
    to_float_kernel<<<grid_for(N, 256), 256, 0, s>>>((const double*)acc.ptr, N, out);
    count_launch();
  }
  cudaError_t e = cudaGetLastError();
  acc.reset(m->al, s);
  if (e != cudaSuccess) return cuda_fail(e, "gs_matrix_sum(axis=1)");
  return GS_OK;
}

gs_status gs_matrix_broadcast(gs_matrix* m, int op, const float* V, int axis, void* stream_) {
  if (!m || !V || op < GS_OP_ADD || op > GS_OP_POW || (axis != 0 && axis != 1))
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_matrix_broadcast: bad argument");
  cudaStream_t s = (cudaStream_t)stream_;
  if (m->nnz == 0) return GS_OK;
  if (axis == 0) {
    bcast_col_kernel<<<grid_for(m->n_cols * 32, OPS_THREADS), OPS_THREADS, 0, s>>>(
        (const int64_t*)m->b_indptr.ptr, (float*)m->b_val.ptr, m->n_cols, op, V);
    count_launch();
  }
  else
    bcast_row_kernel<<<grid_for(m->nnz, 256), 256, 0, s>>>((const int32_t*)m->b_row.ptr, (float*)m->b_val.ptr,
                                                          m->nnz, op, V); count_launch();
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

gs_status gs_matrix_elementwise(gs_matrix* m, int op, float x, void* stream_) {
  if (!m || op < GS_OP_ADD || op > GS_OP_POW) return fail(GS_ERR_INVALID_ARGUMENT, "gs_matrix_elementwise: bad argument");
  if (m->nnz == 0) return GS_OK;
  map_kernel<<<grid_for((m->nnz + 3) / 4, 256), 256, 0, (cudaStream_t)stream_>>>((float*)m->b_val.ptr, m->nnz, op, x); count_launch();
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

gs_status gs_matrix_row_ids(const gs_matrix* m, int32_t* out, int64_t* n_out, void* stream_) {
  if (!m || !out || !n_out) return fail(GS_ERR_INVALID_ARGUMENT, "gs_matrix_row_ids: null pointer");
  cudaStream_t s = (cudaStream_t)stream_;
  const int64_t nw = (m->num_nodes + 31) / 32;
  *n_out = 0;
  if (nw == 0) return GS_OK;
  DevBuf bm, cnt;
  if (!bm.ensure(m->al, (size_t)nw * 4, s) || !cnt.ensure(m->al, (size_t)nw * 8, s))
    return fail(GS_ERR_OUT_OF_MEMORY, "row() workspace");
  gs_status st = GS_OK;
  GS_CUDA_TRY(cudaMemsetAsync(bm.ptr, 0, (size_t)nw * 4, s));
  if (m->nnz > 0) {
    mark_all_rows_kernel<<<grid_for(m->nnz, 256), 256, 0, s>>>((const int32_t*)m->b_row.ptr, m->nnz, (uint32_t*)bm.ptr);
    count_launch();
  }
  word_count_kernel<<<grid_for(nw, 256), 256, 0, s>>>((const uint32_t*)bm.ptr, nw, (int64_t*)cnt.ptr); count_launch();
  st = scan_inclusive((int64_t*)cnt.ptr, nw, m->al, s);
  if (st == GS_OK) {
    emit_rows_kernel<<<grid_for(nw, 256), 256, 0, s>>>((const uint32_t*)bm.ptr, nw, (const int64_t*)cnt.ptr, out); count_launch();
    if (cudaGetLastError() != cudaSuccess) st = fail(GS_ERR_CUDA, "emit_rows_kernel launch");
    else if (cudaMemcpyAsync(n_out, (int64_t*)cnt.ptr + nw - 1, 8, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
             cudaStreamSynchronize(s) != cudaSuccess)
      st = fail(GS_ERR_CUDA, "row() count read-back");
  }
  bm.reset(m->al, s);
  cnt.reset(m->al, s);
  return st;
}

gs_status gs_matrix_get_view(const gs_matrix* m, gs_matrix_view* out) {
  if (!m || !out) return fail(GS_ERR_INVALID_ARGUMENT, "gs_matrix_get_view: null pointer");
  out->num_nodes = m->num_nodes;
  out->n_cols = m->n_cols;
  out->nnz = m->nnz;
  out->cols = (const int32_t*)m->b_cols.ptr;
  out->indptr = (const int64_t*)m->b_indptr.ptr;
  out->row = (const int32_t*)m->b_row.ptr;
  out->eid = (const int64_t*)m->b_eid.ptr;
  out->val = (float*)m->b_val.ptr;
  return GS_OK;
}

void gs_matrix_destroy(gs_matrix* m) {
  if (!m) return;
  cudaStream_t s = nullptr;
  m->b_cols.reset(m->al, s);
  m->b_indptr.reset(m->al, s);
  m->b_row.reset(m->al, s);
  m->b_eid.reset(m->al, s);
  m->b_val.reset(m->al, s);
  delete m;
}

}  // extern "C"
