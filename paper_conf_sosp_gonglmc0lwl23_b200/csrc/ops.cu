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
#include <vector>

#include "common.cuh"
#include "gs_internal.h"
#include "nodewise_common.cuh"
#include <cuda_bf16.h>

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


// ---- Select operators (Table 4; oracle/ops.py individual_sample,
// collective_sample) ----
// A.individual_sample, count pass: kept entries per column (R5 / R6 / R10).
__global__ void isamp_count_kernel(const int64_t* __restrict__ ip, const float* __restrict__ val, int64_t n,
                                   int K, int use_values, int replace, int64_t* __restrict__ out_ip) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t j = warp; j < n; j += nwarps) {
    const int64_t lo = ip[j], hi = ip[j + 1], d = hi - lo;
    int64_t c;
    if (replace) {
      c = d > 0 ? K : 0;
    } else if (use_values) {
      int64_t pos = 0;
      for (int64_t i = lo + lane; i < hi; i += 32) pos += val[i] > 0.0f ? 1 : 0;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) pos += __shfl_xor_sync(0xffffffffu, pos, o);
      c = pos < K ? pos : K;
    } else {
      c = d < K ? d : K;
    }
    if (lane == 0) out_ip[j + 1] = c;
    if (j == 0 && lane == 0) out_ip[0] = 0;
  }
}

// A.individual_sample, select + copy: a thread per column (the general,
// unfused operator; the fused samplers are the fast path).
__global__ void isamp_select_kernel(const int32_t* __restrict__ cols, const int64_t* __restrict__ ip,
                                    const int32_t* __restrict__ row, const int64_t* __restrict__ eid,
                                    const float* __restrict__ val, int64_t n, int K, int use_values, int replace,
                                    uint64_t key, int layer, uint32_t batch, const int64_t* __restrict__ out_ip,
                                    int32_t* __restrict__ orow, int64_t* __restrict__ oeid, float* __restrict__ oval) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t v = (uint32_t)cols[j];
    const int64_t lo = ip[j], d = ip[j + 1] - lo;
    int64_t o = out_ip[j];
    const int64_t cnt = out_ip[j + 1] - o;
    uint32_t pos[MAX_FANOUT];
    double kk[MAX_FANOUT];
    int n_sel = 0;
    if (replace) {
      for (int s = 0; s < (int)cnt; ++s) {
        const U4 r = philox(v, (uint32_t)s, ctr2(layer, TAG_REPLACE), batch, key);
        pos[n_sel++] = (uint32_t)draw_below((uint64_t)d, r.x, r.y);
      }
    } else if (!use_values) {
      if (d <= K) {
        for (int i = 0; i < (int)d; ++i) pos[n_sel++] = (uint32_t)i;
      } else {  // Floyd (R5), the list kept sorted
        for (int s = 0; s < K; ++s) {
          const U4 r = philox(v, (uint32_t)s, ctr2(layer, TAG_FLOYD), batch, key);
          const uint32_t m = (uint32_t)(d - K + s);
          const uint32_t t = (uint32_t)draw_below((uint64_t)m + 1, r.x, r.y);
          bool dup = false;
          for (int q = 0; q < n_sel; ++q) dup |= pos[q] == t;
          const uint32_t x = dup ? m : t;
          int q = n_sel;
          while (q > 0 && pos[q - 1] > x) {
            pos[q] = pos[q - 1];
            --q;
          }
          pos[q] = x;
          ++n_sel;
        }
      }
    } else {  // A-Res (R6): the cnt smallest (key, position) among the positive values
      for (int64_t i = 0; i < d && cnt > 0; ++i) {
        const float w = val[lo + i];
        if (!(w > 0.0f)) continue;
        const U4 r = philox(v, (uint32_t)(i >> 2), ctr2(layer, TAG_ARES_NODE), batch, key);
        const double k2 = ares_key(sel_word(r, (int)(i & 3)), (double)w);
        if (n_sel == cnt && !(k2 < kk[n_sel - 1])) continue;
        int q = n_sel < cnt ? n_sel : (int)cnt - 1;
        while (q > 0 && kk[q - 1] > k2) {
          kk[q] = kk[q - 1];
          pos[q] = pos[q - 1];
          --q;
        }
        kk[q] = k2;
        pos[q] = (uint32_t)i;
        if (n_sel < cnt) ++n_sel;
      }
      for (int a = 1; a < n_sel; ++a) {  // positions ascending
        const uint32_t x = pos[a];
        int q = a;
        while (q > 0 && pos[q - 1] > x) {
          pos[q] = pos[q - 1];
          --q;
        }
        pos[q] = x;
      }
    }
    for (int q = 0; q < n_sel; ++q) {
      const int64_t i = lo + pos[q];
      orow[o] = row[i];
      oeid[o] = eid[i];
      oval[o] = val[i];
      ++o;
    }
  }
}

// A.collective_sample helpers: per-row entry counts (node_probs omitted)
__global__ void row_count_dense_kernel(const int32_t* __restrict__ row, int64_t nnz, float* __restrict__ cnt) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(cnt + __ldcs(row + i), 1.0f);  // exact: integer counts < 2^24
}

// keys of the candidates C (ascending ids): eligible (b > 0) -> (key, u); B;
// count of keys below tau and the ones below tau collected (<= cap)
__global__ void csamp_keys_kernel(const int32_t* __restrict__ C, int64_t nc, const float* __restrict__ b,
                                  uint64_t key, int layer, uint32_t batch, double* __restrict__ ckey,
                                  double* __restrict__ bsum, unsigned long long* __restrict__ nelig) {
  double s = 0.0;
  unsigned long long e = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nc; i += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t u = (uint32_t)C[i];
    const float bias = b[u];
    double k2 = INFINITY;
    if (bias > 0.0f) {
      const U4 r = philox(u, 0u, ctr2(layer, TAG_ARES_LAYER), batch, key);
      k2 = ares_key(r.x, (double)bias);
      ++e;
    }
    s += (double)bias;
    ckey[i] = k2;
  }
  for (int o = 16; o > 0; o >>= 1) {
    s += __shfl_xor_sync(0xffffffffu, s, o);
    e += __shfl_xor_sync(0xffffffffu, e, o);
  }
  if ((threadIdx.x & 31) == 0) {
    atomicAdd(bsum, s);
    atomicAdd(nelig, e);
  }
}

__global__ void csamp_collect_kernel(const int32_t* __restrict__ C, const double* __restrict__ ckey, int64_t nc,
                                     double tau, int cap, double* __restrict__ bk, int32_t* __restrict__ bu,
                                     unsigned int* __restrict__ nb) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nc; i += (int64_t)gridDim.x * blockDim.x) {
    const double k2 = ckey[i];
    if (!(k2 < tau)) continue;
    const unsigned int slot = atomicAdd(nb, 1u);
    if ((int)slot < cap) {
      bk[slot] = k2;
      bu[slot] = C[i];
    }
  }
}

// one CTA: the K smallest (key, u) of n buffered candidates -> their rows'
// bits in the bitmap (the sub-matrix is then A restricted to them)
constexpr int CS_CAP = 4096;
__global__ void __launch_bounds__(1024) csamp_select_kernel(const double* __restrict__ bk, const int32_t* __restrict__ bu,
                                                          int n, int K, uint32_t* __restrict__ bm) {
  __shared__ double sk[CS_CAP];
  __shared__ int32_t su[CS_CAP];
  int n2 = 1;
  while (n2 < n) n2 <<= 1;
  for (int i = threadIdx.x; i < n2; i += blockDim.x) {
    sk[i] = i < n ? bk[i] : INFINITY;
    su[i] = i < n ? bu[i] : 0x7FFFFFFF;
  }
  __syncthreads();
  for (int k = 2; k <= n2; k <<= 1)
    for (int j = k >> 1; j > 0; j >>= 1) {
      for (int i = threadIdx.x; i < n2; i += blockDim.x) {
        const int o = i ^ j;
        if (o > i) {
          const bool gt = sk[i] > sk[o] || (sk[i] == sk[o] && su[i] > su[o]);
          if (gt == ((i & k) == 0)) {
            const double t = sk[i]; sk[i] = sk[o]; sk[o] = t;
            const int32_t tu = su[i]; su[i] = su[o]; su[o] = tu;
          }
        }
      }
      __syncthreads();
    }
  for (int i = threadIdx.x; i < K && i < n; i += blockDim.x) atomicOr(bm + (su[i] >> 5), 1u << (su[i] & 31));
}

// eligible rows (b > 0) of C into the bitmap (at most K of them: all are taken, R24)
__global__ void csamp_all_kernel(const int32_t* __restrict__ C, int64_t nc, const float* __restrict__ b,
                                 uint32_t* __restrict__ bm) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nc; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t u = C[i];
    if (b[u] > 0.0f) atomicOr(bm + (u >> 5), 1u << (u & 31));
  }
}

// ---- fused Edge-Map chain (+ Edge-Reduce), P:291-294 ----
constexpr int MR_MAX_OPS = 8;
struct MapChain {
  int n;
  int op[MR_MAX_OPS];
  float x[MR_MAX_OPS];
};
__device__ __forceinline__ float chain_apply(const MapChain& c, float v) {
  for (int i = 0; i < c.n; ++i) v = apply_op(c.op[i], v, c.x[i]);
  return v;
}
__global__ void map_chain_kernel(float* val, int64_t nnz, MapChain c) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x)
    val[i] = chain_apply(c, val[i]);
}
__global__ void __launch_bounds__(OPS_THREADS) map_col_sum_kernel(const int64_t* __restrict__ ip,
                                                                 const float* __restrict__ val, int64_t n,
                                                                 MapChain c, float* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t j = warp; j < n; j += nwarps) {
    double s = 0.0;
    for (int64_t i = ip[j] + lane; i < ip[j + 1]; i += 32) s += (double)chain_apply(c, __ldcs(val + i));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) out[j] = (float)s;
  }
}
__global__ void map_row_sum_kernel(const int32_t* __restrict__ row, const float* __restrict__ val, int64_t nnz,
                                   MapChain c, double* __restrict__ acc) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(acc + __ldcs(row + i), (double)chain_apply(c, __ldcs(val + i)));
}

// ---- AS-GCN-style bias (R30): b(u) = fp32(s(u) * relu(fp32(sum_fp64 X[u] wg))) ----
__global__ void asgcn_bias_kernel(const double* __restrict__ s, const __nv_bfloat16* __restrict__ X, int F,
                                  const float* __restrict__ wg, int64_t N, float* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = warp; u < N; u += nwarps) {
    const float su = (float)s[u];
    if (su == 0.0f) {  // not a row of the matrix (or a zero sum): b = 0
      if (lane == 0) out[u] = 0.0f;
      continue;
    }
    double dot = 0.0;
    for (int f = lane; f < F; f += 32) dot += (double)__bfloat162float(X[u * F + f]) * (double)wg[f];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) dot += __shfl_xor_sync(0xffffffffu, dot, o);
    if (lane == 0) {
      const float g = (float)dot;
      out[u] = __fmul_rn(su, g > 0.0f ? g : 0.0f);
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


gs_status gs_matrix_individual_sample(const gs_matrix* in, int K, int use_values, int replace, uint64_t rng_key,
                                      int layer, int64_t batch_index, void* stream_, gs_matrix** out) {
  if (!in || !out || *out == in || K < 1 || K > MAX_FANOUT || (replace && use_values) || layer < 0 ||
      layer >= (1 << 24) || batch_index < 0)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_matrix_individual_sample: bad argument (1 <= K <= %d, no weighted "
                "replacement, out != in)", MAX_FANOUT);
  cudaStream_t s = (cudaStream_t)stream_;
  gs_status st = new_matrix(out, in->num_nodes);
  if (st) return st;
  gs_matrix* m = *out;
  const int64_t n = in->n_cols;
  if (!m->b_indptr.ensure(m->al, (size_t)(n + 1) * 8, s))
    return fail(GS_ERR_OUT_OF_MEMORY, "device allocation failed (individual_sample)");
  int64_t* ip = (int64_t*)m->b_indptr.ptr;
  GS_CUDA_TRY(cudaMemsetAsync(ip, 0, 8, s));
  if (n > 0) {
    isamp_count_kernel<<<grid_for(n * 32, 256), 256, 0, s>>>((const int64_t*)in->b_indptr.ptr,
                                                           (const float*)in->b_val.ptr, n, K, use_values, replace, ip);
    count_launch();
    GS_CUDA_TRY(cudaGetLastError());
    if ((st = scan_inclusive(ip + 1, n, m->al, s))) return st;
  }
  int64_t nnz = 0;
  GS_CUDA_TRY(cudaMemcpyAsync(&nnz, ip + n, 8, cudaMemcpyDeviceToHost, s));
  GS_CUDA_TRY(cudaStreamSynchronize(s));
  if ((st = alloc_entries(m, n, nnz, s))) return st;
  if (n > 0) {
    GS_CUDA_TRY(cudaMemcpyAsync(m->b_cols.ptr, in->b_cols.ptr, n * 4, cudaMemcpyDeviceToDevice, s));
    isamp_select_kernel<<<grid_for(n, 128), 128, 0, s>>>(
        (const int32_t*)in->b_cols.ptr, (const int64_t*)in->b_indptr.ptr, (const int32_t*)in->b_row.ptr,
        (const int64_t*)in->b_eid.ptr, (const float*)in->b_val.ptr, n, K, use_values, replace, rng_key, layer,
        (uint32_t)batch_index, ip, (int32_t*)m->b_row.ptr, (int64_t*)m->b_eid.ptr, (float*)m->b_val.ptr);
    count_launch();
    GS_CUDA_TRY(cudaGetLastError());
  }
  return GS_OK;
}

gs_status gs_matrix_collective_sample(const gs_matrix* in, int K, const float* node_probs, uint64_t rng_key,
                                      int layer, int64_t batch_index, void* stream_, gs_matrix** out) {
  if (!in || !out || *out == in || K < 1 || layer < 0 || layer >= (1 << 24) || batch_index < 0)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_matrix_collective_sample: bad argument (K >= 1, out != in)");
  cudaStream_t s = (cudaStream_t)stream_;
  const int64_t N = in->num_nodes, nw = (N + 31) / 32;
  const Allocator al = in->al;
  // C = row(): the distinct rows ascending
  DevBuf cbuf, bias, keys, sel, bbuf, misc;
  if (!cbuf.ensure(al, (size_t)std::max<int64_t>(std::min(in->nnz, N), 1) * 4, s) ||
      !misc.ensure(al, 64, s) || !sel.ensure(al, (size_t)std::max<int64_t>(nw, 1) * 4, s))
    return fail(GS_ERR_OUT_OF_MEMORY, "collective_sample workspace");
  auto cleanup = [&](gs_status st) {
    cbuf.reset(al, s); bias.reset(al, s); keys.reset(al, s); sel.reset(al, s); bbuf.reset(al, s); misc.reset(al, s);
    return st;
  };
  int64_t nc = 0;
  gs_status st = gs_matrix_row_ids(in, (int32_t*)cbuf.ptr, &nc, stream_);
  if (st) return cleanup(st);
  const float* b = node_probs;
  if (!b) {  // "the sampling bias on each edge is 1 and automatically aggregates"
    if (!bias.ensure(al, (size_t)std::max<int64_t>(N, 1) * 4, s)) return cleanup(fail(GS_ERR_OUT_OF_MEMORY, "bias"));
    GS_CUDA_TRY(cudaMemsetAsync(bias.ptr, 0, (size_t)std::max<int64_t>(N, 1) * 4, s));
    if (in->nnz > 0) {
      row_count_dense_kernel<<<grid_for(in->nnz, 256), 256, 0, s>>>((const int32_t*)in->b_row.ptr, in->nnz,
                                                                    (float*)bias.ptr);
      count_launch();
    }
    b = (const float*)bias.ptr;
  }
  GS_CUDA_TRY(cudaMemsetAsync(sel.ptr, 0, (size_t)std::max<int64_t>(nw, 1) * 4, s));
  GS_CUDA_TRY(cudaMemsetAsync(misc.ptr, 0, 64, s));
  double* bsum = (double*)misc.ptr;
  unsigned long long* nelig = (unsigned long long*)((char*)misc.ptr + 8);
  unsigned int* nbuf = (unsigned int*)((char*)misc.ptr + 16);
  if (nc > 0) {
    if (!keys.ensure(al, (size_t)nc * 8, s)) return cleanup(fail(GS_ERR_OUT_OF_MEMORY, "keys"));
    csamp_keys_kernel<<<grid_for(nc, 256), 256, 0, s>>>((const int32_t*)cbuf.ptr, nc, b, rng_key, layer,
                                                        (uint32_t)batch_index, (double*)keys.ptr, bsum, nelig);
    count_launch();
    double hb = 0.0;
    unsigned long long he = 0;
    GS_CUDA_TRY(cudaMemcpyAsync(&hb, bsum, 8, cudaMemcpyDeviceToHost, s));
    GS_CUDA_TRY(cudaMemcpyAsync(&he, nelig, 8, cudaMemcpyDeviceToHost, s));
    GS_CUDA_TRY(cudaStreamSynchronize(s));
    if ((int64_t)he <= K) {  // every eligible row (R24)
      csamp_all_kernel<<<grid_for(nc, 256), 256, 0, s>>>((const int32_t*)cbuf.ptr, nc, b, (uint32_t*)sel.ptr);
      count_launch();
    } else {
      // threshold: keys below tau (expected ~2K of them), widened / narrowed
      // until K <= count <= CS_CAP, then the K smallest in one CTA
      if (K > CS_CAP / 2) return cleanup(fail(GS_ERR_NOT_SUPPORTED, "collective_sample: K <= %d", CS_CAP / 2));
      if (!bbuf.ensure(al, (size_t)CS_CAP * 12, s)) return cleanup(fail(GS_ERR_OUT_OF_MEMORY, "buffer"));
      double tau = hb > 0.0 ? 2.0 * K / hb : 1.0, lo = 0.0, hi = 0.0;
      unsigned int cnt = 0;
      for (int att = 0; att < 200; ++att) {
        GS_CUDA_TRY(cudaMemsetAsync(nbuf, 0, 4, s));
        csamp_collect_kernel<<<grid_for(nc, 256), 256, 0, s>>>((const int32_t*)cbuf.ptr, (const double*)keys.ptr,
                                                               nc, tau, CS_CAP, (double*)bbuf.ptr,
                                                               (int32_t*)((char*)bbuf.ptr + CS_CAP * 8), nbuf);
        count_launch();
        GS_CUDA_TRY(cudaMemcpyAsync(&cnt, nbuf, 4, cudaMemcpyDeviceToHost, s));
        GS_CUDA_TRY(cudaStreamSynchronize(s));
        if ((int)cnt >= K && (int)cnt <= CS_CAP) break;
        if ((int)cnt < K) lo = tau;
        else hi = tau;
        tau = (lo > 0.0 && hi > 0.0) ? 0.5 * (lo + hi) : (lo > 0.0 ? lo * 4.0 : hi * 0.5);
      }
      if ((int)cnt < K || (int)cnt > CS_CAP) return cleanup(fail(GS_ERR_CUDA, "collective_sample: threshold search failed"));
      csamp_select_kernel<<<1, 1024, 0, s>>>((const double*)bbuf.ptr, (const int32_t*)((char*)bbuf.ptr + CS_CAP * 8),
                                             (int)cnt, K, (uint32_t*)sel.ptr);
      count_launch();
    }
    GS_CUDA_TRY(cudaGetLastError());
  }
  // the sub-matrix: the entries whose row was selected (CSC order), as A[rows, :]
  st = new_matrix(out, N);
  if (st) return cleanup(st);
  gs_matrix* m = *out;
  const int64_t n = in->n_cols;
  if (!m->b_indptr.ensure(m->al, (size_t)(n + 1) * 8, s)) return cleanup(fail(GS_ERR_OUT_OF_MEMORY, "indptr"));
  int64_t* ip = (int64_t*)m->b_indptr.ptr;
  GS_CUDA_TRY(cudaMemsetAsync(ip, 0, 8, s));
  if (n > 0) {
    row_count_kernel<<<grid_for(n * 32, OPS_THREADS), OPS_THREADS, 0, s>>>(
        (const int64_t*)in->b_indptr.ptr, (const int32_t*)in->b_row.ptr, n, (const uint32_t*)sel.ptr, ip);
    count_launch();
    if ((st = scan_inclusive(ip + 1, n, m->al, s))) return cleanup(st);
  }
  int64_t nnz = 0;
  GS_CUDA_TRY(cudaMemcpyAsync(&nnz, ip + n, 8, cudaMemcpyDeviceToHost, s));
  GS_CUDA_TRY(cudaStreamSynchronize(s));
  if ((st = alloc_entries(m, n, nnz, s))) return cleanup(st);
  if (n > 0) {
    GS_CUDA_TRY(cudaMemcpyAsync(m->b_cols.ptr, in->b_cols.ptr, n * 4, cudaMemcpyDeviceToDevice, s));
    row_copy_kernel<<<grid_for(n * 32, OPS_THREADS), OPS_THREADS, 0, s>>>(
        (const int64_t*)in->b_indptr.ptr, (const int32_t*)in->b_row.ptr, (const int64_t*)in->b_eid.ptr,
        (const float*)in->b_val.ptr, n, (const uint32_t*)sel.ptr, ip, (int32_t*)m->b_row.ptr, (int64_t*)m->b_eid.ptr,
        (float*)m->b_val.ptr);
    count_launch();
    GS_CUDA_TRY(cudaGetLastError());
  }
  return cleanup(GS_OK);
}

gs_status gs_matrix_map_reduce(gs_matrix* m, const int* ops, const float* scalars, int n_ops, int axis, float* out,
                               void* stream_) {
  if (!m || (n_ops > 0 && (!ops || !scalars)) || n_ops < 0 || n_ops > MR_MAX_OPS || axis < -1 || axis > 1 ||
      (axis >= 0 && !out))
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_matrix_map_reduce: bad argument (<= %d ops, axis -1/0/1)", MR_MAX_OPS);
  MapChain c = {};
  c.n = n_ops;
  for (int i = 0; i < n_ops; ++i) {
    if (ops[i] < GS_OP_ADD || ops[i] > GS_OP_POW) return fail(GS_ERR_INVALID_ARGUMENT, "gs_matrix_map_reduce: op");
    c.op[i] = ops[i];
    c.x[i] = scalars[i];
  }
  cudaStream_t s = (cudaStream_t)stream_;
  if (axis < 0) {  // Edge-Map fusion: the chain applied in place in one pass
    if (m->nnz > 0) {
      map_chain_kernel<<<grid_for(m->nnz, 256), 256, 0, s>>>((float*)m->b_val.ptr, m->nnz, c);
      count_launch();
    }
  } else if (axis == 0) {
    if (m->n_cols > 0) {
      map_col_sum_kernel<<<grid_for(m->n_cols * 32, OPS_THREADS), OPS_THREADS, 0, s>>>(
          (const int64_t*)m->b_indptr.ptr, (const float*)m->b_val.ptr, m->n_cols, c, out);
      count_launch();
    }
  } else {
    const int64_t N = m->num_nodes;
    DevBuf acc;
    if (!acc.ensure(m->al, (size_t)std::max<int64_t>(N, 1) * 8, s)) return fail(GS_ERR_OUT_OF_MEMORY, "map_reduce acc");
    GS_CUDA_TRY(cudaMemsetAsync(acc.ptr, 0, (size_t)std::max<int64_t>(N, 1) * 8, s));
    if (m->nnz > 0) {
      map_row_sum_kernel<<<grid_for(m->nnz, 256), 256, 0, s>>>((const int32_t*)m->b_row.ptr, (const float*)m->b_val.ptr,
                                                               m->nnz, c, (double*)acc.ptr);
      count_launch();
    }
    if (N > 0) {
      to_float_kernel<<<grid_for(N, 256), 256, 0, s>>>((const double*)acc.ptr, N, out);
      count_launch();
    }
    acc.reset(m->al, s);
  }
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

gs_status gs_matrix_asgcn_bias(const gs_matrix* m, const void* X, int F, const float* wg, float* out, void* stream_) {
  if (!m || !X || !wg || !out || F <= 0) return fail(GS_ERR_INVALID_ARGUMENT, "gs_matrix_asgcn_bias: bad argument");
  cudaStream_t s = (cudaStream_t)stream_;
  const int64_t N = m->num_nodes;
  DevBuf acc;
  if (!acc.ensure(m->al, (size_t)std::max<int64_t>(N, 1) * 8, s)) return fail(GS_ERR_OUT_OF_MEMORY, "asgcn acc");
  GS_CUDA_TRY(cudaMemsetAsync(acc.ptr, 0, (size_t)std::max<int64_t>(N, 1) * 8, s));
  if (m->nnz > 0) {
    row_sum_kernel<<<grid_for(m->nnz, 256), 256, 0, s>>>((const int32_t*)m->b_row.ptr, (const float*)m->b_val.ptr,
                                                         m->nnz, (double*)acc.ptr);
    count_launch();
  }
  if (N > 0) {
    asgcn_bias_kernel<<<grid_for(N * 32, 256), 256, 0, s>>>((const double*)acc.ptr, (const __nv_bfloat16*)X, F, wg,
                                                             N, out);
    count_launch();
  }
  GS_CUDA_TRY(cudaGetLastError());
  acc.reset(m->al, s);
  return GS_OK;
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

// ---------------------------------------------------------------------------
// Heterogeneous node-wise sampling (each edge type is a sparse matrix
// sampled by the same workflow; oracle/ops.py
// hetero_sample_neighbors).  Per layer and relation r: A_r[:, F_dst(r)]
// (gs_matrix_slice_columns) .individual_sample(k) (Floyd, R5) under the
// relation's key (R33); the next frontier of every node type is the union of
// the rows of the relations out of that type, ascending (A.row() of each,
// merged in one bitmap: mark -> popcount scan -> emit).
// ---------------------------------------------------------------------------
struct gs_hetero {
  gsb::Allocator al;
  int L = 0, R = 0, T = 0;
  std::vector<gs_matrix*> blocks;    // [L][R], NULL where skipped
  std::vector<gsb::DevBuf> fr;       // [L + 1][T] frontier ids
  std::vector<int64_t> nfr;          // [L + 1][T]
};

namespace gsb {
static uint64_t relation_key(uint64_t key, int r) {  // R33
  return key ^ (0x9E3779B97F4A7C15ull * (uint64_t)(r + 1));
}
}  // namespace gsb

void gs_hetero_destroy(gs_hetero* h) {
  if (!h) return;
  for (gs_matrix* m : h->blocks) gs_matrix_destroy(m);
  for (auto& b : h->fr) b.reset(h->al, nullptr);
  delete h;
}

gs_status gs_sample_neighbors_hetero(const gs_graph* const* graphs, const int32_t* src_type, const int32_t* dst_type,
                                     int num_relations, int num_node_types, const int64_t* num_nodes,
                                     const int32_t* const* seeds, const int64_t* num_seeds, const int32_t* fanouts,
                                     int num_layers, uint64_t rng_key, void* stream_, gs_hetero** out) {
  if (!graphs || !src_type || !dst_type || !num_nodes || !seeds || !num_seeds || !fanouts || !out ||
      num_relations < 1 || num_node_types < 1 || num_layers < 1 || num_layers > MAX_LAYERS)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_sample_neighbors_hetero: null pointer or bad count");
  for (int r = 0; r < num_relations; ++r) {
    if (!graphs[r] || src_type[r] < 0 || src_type[r] >= num_node_types || dst_type[r] < 0 ||
        dst_type[r] >= num_node_types)
      return fail(GS_ERR_INVALID_ARGUMENT, "gs_sample_neighbors_hetero: relation %d: bad graph or node type", r);
    if (graphs[r]->num_nodes < num_nodes[dst_type[r]] || graphs[r]->num_nodes < num_nodes[src_type[r]])
      return fail(GS_ERR_INVALID_ARGUMENT,
                  "gs_sample_neighbors_hetero: relation %d: its graph needs max(|src|, |dst|) columns", r);
  }
  for (int l = 0; l < num_layers; ++l)
    for (int r = 0; r < num_relations; ++r)
      if (fanouts[l * num_relations + r] < 0 || fanouts[l * num_relations + r] > MAX_FANOUT)
        return fail(GS_ERR_INVALID_ARGUMENT, "gs_sample_neighbors_hetero: fanouts in [0, %d]", MAX_FANOUT);
  for (int t = 0; t < num_node_types; ++t)
    if (num_seeds[t] < 0 || (num_seeds[t] > 0 && !seeds[t]) || num_nodes[t] < 0)
      return fail(GS_ERR_INVALID_ARGUMENT, "gs_sample_neighbors_hetero: node type %d: bad seeds", t);
  cudaStream_t s = (cudaStream_t)stream_;
  gs_hetero* h = new (std::nothrow) gs_hetero();
  if (!h) return fail(GS_ERR_OUT_OF_MEMORY, "gs_sample_neighbors_hetero: host allocation failed");
  h->al = current_allocator();
  h->L = num_layers;
  h->R = num_relations;
  h->T = num_node_types;
  h->blocks.assign((size_t)num_layers * num_relations, nullptr);
  h->fr.resize((size_t)(num_layers + 1) * num_node_types);
  h->nfr.assign((size_t)(num_layers + 1) * num_node_types, 0);
  auto bail = [&](gs_status st) {
    gs_hetero_destroy(h);
    return st;
  };
  for (int t = 0; t < num_node_types; ++t) {
    DevBuf& b = h->fr[(size_t)t];
    if (!b.ensure(h->al, (size_t)std::max<int64_t>(num_seeds[t], 1) * 4, s))
      return bail(fail(GS_ERR_OUT_OF_MEMORY, "hetero frontier"));
    if (num_seeds[t] > 0)
      if (cudaMemcpyAsync(b.ptr, seeds[t], (size_t)num_seeds[t] * 4, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
        return bail(fail(GS_ERR_CUDA, "hetero seed copy"));
    h->nfr[(size_t)t] = num_seeds[t];
  }
  DevBuf bm, cnt, err;
  int64_t maxn = 1;
  for (int t = 0; t < num_node_types; ++t) maxn = std::max<int64_t>(maxn, num_nodes[t]);
  const int64_t maxw = (maxn + 31) / 32;
  if (!bm.ensure(h->al, (size_t)maxw * 4, s) || !cnt.ensure(h->al, (size_t)maxw * 8, s) ||
      !err.ensure(h->al, 16, s, true))
    return bail(fail(GS_ERR_OUT_OF_MEMORY, "hetero union workspace"));
  gs_status st = GS_OK;
  for (int l = 0; l < num_layers && st == GS_OK; ++l) {
    for (int r = 0; r < num_relations && st == GS_OK; ++r) {
      const int k = fanouts[l * num_relations + r];
      const int dt = dst_type[r];
      const int64_t nf = h->nfr[(size_t)l * num_node_types + dt];
      if (k == 0 || nf == 0) continue;
      gs_matrix* M = nullptr;
      st = gs_matrix_slice_columns(graphs[r], (const int32_t*)h->fr[(size_t)l * num_node_types + dt].ptr, nf, s, &M);
      if (st == GS_OK)
        st = gs_matrix_individual_sample(M, k, 0, 0, relation_key(rng_key, r), l, 0, s,
                                         &h->blocks[(size_t)l * num_relations + r]);
      gs_matrix_destroy(M);
    }
    for (int t = 0; t < num_node_types && st == GS_OK; ++t) {
      const int64_t nw = (num_nodes[t] + 31) / 32;
      DevBuf& o = h->fr[(size_t)(l + 1) * num_node_types + t];
      if (!o.ensure(h->al, (size_t)std::max<int64_t>(num_nodes[t], 1) * 4, s)) {
        st = fail(GS_ERR_OUT_OF_MEMORY, "hetero frontier");
        break;
      }
      if (nw == 0) continue;
      if (cudaMemsetAsync(bm.ptr, 0, (size_t)nw * 4, s) != cudaSuccess) {
        st = fail(GS_ERR_CUDA, "hetero union memset");
        break;
      }
      for (int r = 0; r < num_relations; ++r) {
        const gs_matrix* B = h->blocks[(size_t)l * num_relations + r];
        if (src_type[r] != t || !B || B->nnz == 0) continue;
        mark_rows_kernel<<<grid_for(B->nnz, 256), 256, 0, s>>>((const int32_t*)B->b_row.ptr, B->nnz, num_nodes[t],
                                                               (uint32_t*)bm.ptr, (int*)err.ptr);
        count_launch();
      }
      word_count_kernel<<<grid_for(nw, 256), 256, 0, s>>>((const uint32_t*)bm.ptr, nw, (int64_t*)cnt.ptr);
      count_launch();
      if ((st = scan_inclusive((int64_t*)cnt.ptr, nw, h->al, s))) break;
      emit_rows_kernel<<<grid_for(nw, 256), 256, 0, s>>>((const uint32_t*)bm.ptr, nw, (const int64_t*)cnt.ptr,
                                                         (int32_t*)o.ptr);
      count_launch();
      int64_t n = 0;
      if (cudaMemcpyAsync(&n, (int64_t*)cnt.ptr + nw - 1, 8, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
          cudaStreamSynchronize(s) != cudaSuccess) {
        st = fail(GS_ERR_CUDA, "hetero frontier count read-back");
        break;
      }
      h->nfr[(size_t)(l + 1) * num_node_types + t] = n;
    }
  }
  if (st == GS_OK) st = check_err((int*)err.ptr, s);
  bm.reset(h->al, s);
  cnt.reset(h->al, s);
  err.reset(h->al, s);
  if (st) return bail(st);
  *out = h;
  return GS_OK;
}

gs_status gs_hetero_block(const gs_hetero* h, int layer, int relation, const gs_matrix** out) {
  if (!h || !out || layer < 0 || layer >= h->L || relation < 0 || relation >= h->R)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_hetero_block: bad layer / relation");
  *out = h->blocks[(size_t)layer * h->R + relation];
  return GS_OK;
}

gs_status gs_hetero_frontier(const gs_hetero* h, int layer, int node_type, const int32_t** ids, int64_t* n) {
  if (!h || !ids || !n || layer < 0 || layer > h->L || node_type < 0 || node_type >= h->T)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_hetero_frontier: bad layer / node type");
  *ids = (const int32_t*)h->fr[(size_t)layer * h->T + node_type].ptr;
  *n = h->nfr[(size_t)layer * h->T + node_type];
  return GS_OK;
}
