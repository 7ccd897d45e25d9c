// pass_att.cu -- PASS's learned sampling bias in full (Fig. 3(c) lines 3-9,
// P:185-226; R29).  For every edge e = (u -> v) with weight w_e:
//   A1 = w_e <X_u W1, X_v W1>,  A2 = w_e <X_u W2, X_v W2>,  A3 = fp32(w_e / colsum_v),
//   att = relu((s0 A1 + s1 A2) + s2 A3),  s = softmax(W3).
// Every term depends on the edge alone, so att is computed once per set of
// projection weights for the whole graph (the paper's pre-processing rule (2),
// P:300) and line 10's individual_sample(k, att) is the weighted A-Res sampler
// over att (gs_graph_set_weights + gs_sample_neighbors(GS_W_EDGE)).
//
//   1. projections P = X [W1 | W2] : [N, F] x [F, 2H] bf16 -> fp32, one dense
//      GEMM on the 5th-generation tensor cores: the hand-written TMA +
//      tcgen05.mma + TMEM kernel of proj_gemm.cuh (F % 16 == 0; cuBLAS for
//      other F, or with GS_PASS_GEMM=cublas); fp32 accumulation, so general
//      inputs agree with the fp64 oracle within the magnitude-scaled bound of
//      DESIGN.md R29 and the grid-valued inputs bit for bit.
//   2. SDDMM + mix: a warp per column v keeps P_v (2H floats) in shared memory;
//      8 lanes per in-edge gather P_u as 16-byte vectors (one random 2H*4-byte
//      row per edge), form both dot products in fp64 (exact, any order), A3
//      from the a0 column sum, mix in fp64 and write fp32 att.
#include <cublas_v2.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include <algorithm>
#include <mutex>

#include "common.cuh"
#include "gs_internal.h"
#include "proj_gemm.cuh"
#include <cudaTypedefs.h>
#include <cstdlib>

namespace gsb {

constexpr int PA_THREADS = 256;
constexpr int PA_WARPS = PA_THREADS / 32;
constexpr int PA_MAX_H = 64;
constexpr int PA_EILP = 4;  // edge steps (4 edges each) per warp in flight

template <int H2>  // 2H floats per projected row
__global__ void __launch_bounds__(PA_THREADS) pass_att_kernel(const int64_t* __restrict__ indptr,
                                                              const int32_t* __restrict__ indices,
                                                              const float* __restrict__ w,
                                                              const float* __restrict__ colsum,
                                                              const float* __restrict__ P, int64_t N,
                                                              double s0, double s1, double s2,
                                                              float* __restrict__ att) {
  __shared__ __align__(16) float pv[PA_WARPS][H2];
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  constexpr int H = H2 / 2;
  constexpr int QL = (H2 / 4 + 7) / 8;  // 16-byte vectors per lane per edge
  for (int64_t v = warp; v < N; v += nwarps) {
    const int64_t o = __ldg(indptr + v), d = __ldg(indptr + v + 1) - o;
    if (d == 0) continue;
    __syncwarp();
    for (int i = lane; i < H2; i += 32) pv[wl][i] = __ldg(P + v * H2 + i);
    __syncwarp();
    const float cs = w ? __ldg(colsum + v) : (float)d;
    // 8 lanes per edge, 4 edges per warp step: a load instruction covers 4
    // projected rows as whole 128-byte lines (lane-per-edge gathers touch 32
    // lines per instruction); the 8 partial sums of each dot are combined by
    // xor-shuffles (exact in fp64, so the combination order is immaterial)
    const int slot = lane >> 3, sub = lane & 7;
    const float4* pv4 = reinterpret_cast<const float4*>(pv[wl]);
    for (int64_t i0 = 0; i0 < d; i0 += 4 * PA_EILP) {  // PA_EILP edge steps in flight
      int64_t e[PA_EILP];
      int32_t u[PA_EILP];
#pragma unroll
      for (int r = 0; r < PA_EILP; ++r) {
        const int64_t i = i0 + r * 4 + slot;
        e[r] = i < d ? o + i : -1;
        u[r] = e[r] >= 0 ? __ldg(indices + e[r]) : 0;
      }
      float4 a[PA_EILP][QL];
#pragma unroll
      for (int r = 0; r < PA_EILP; ++r) {
        const float4* pu = reinterpret_cast<const float4*>(P + (int64_t)u[r] * H2);
#pragma unroll
        for (int j = 0; j < QL; ++j) {
          const int q = sub + 8 * j;
          a[r][j] = (e[r] >= 0 && q < H2 / 4) ? __ldg(pu + q) : make_float4(0.f, 0.f, 0.f, 0.f);
        }
      }
#pragma unroll
      for (int r = 0; r < PA_EILP; ++r) {
        double d1 = 0.0, d2 = 0.0;
#pragma unroll
        for (int j = 0; j < QL; ++j) {
          const int q = sub + 8 * j;
          if (q < H2 / 4) {
            const float4 b = pv4[q];
            const double t = (double)a[r][j].x * b.x + (double)a[r][j].y * b.y +
                             (double)a[r][j].z * b.z + (double)a[r][j].w * b.w;
            if (q < H / 4) d1 += t;
            else d2 += t;
          }
        }
#pragma unroll
        for (int off = 4; off > 0; off >>= 1) {
          d1 += __shfl_xor_sync(0xffffffffu, d1, off);
          d2 += __shfl_xor_sync(0xffffffffu, d2, off);
        }
        if (e[r] >= 0 && sub == 0) {
          const float we = w ? __ldg(w + e[r]) : 1.0f;
          const double a1 = (double)we * d1, a2 = (double)we * d2;
          const double a3 = (double)__fdiv_rn(we, cs);
          const double mix = (s0 * a1 + s1 * a2) + s2 * a3;
          att[e[r]] = mix > 0.0 ? (float)mix : 0.0f;  // relu (NaN -> 0)
        }
      }
    }
  }
}

static cublasHandle_t pa_handle() {
  static cublasHandle_t h = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    if (cublasCreate(&h) != CUBLAS_STATUS_SUCCESS) h = nullptr;
  });
  return h;
}

static std::mutex pa_mutex;  // the shared handle's stream binding

// WT[n][f] = [W1 | W2][f][n]: the B operand K-major (f contiguous)
__global__ void pg_pack_wt_kernel(const __nv_bfloat16* __restrict__ W1, const __nv_bfloat16* __restrict__ W2,
                                  int F, int H, __nv_bfloat16* __restrict__ WT) {
  const int n2 = 2 * H;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n2 * F; i += gridDim.x * blockDim.x) {
    const int n = i / F, f = i - n * F;
    WT[i] = n < H ? W1[(size_t)f * H + n] : W2[(size_t)f * H + (n - H)];
  }
}

static PFN_cuTensorMapEncodeTiled_v12000 pg_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (PFN_cuTensorMapEncodeTiled_v12000)p;
  });
  return fn;
}

// P[N][2H] = X[N][F] [W1 | W2] on the tensor cores (proj_gemm.cuh).
static gs_status pg_project(const void* X, int64_t N, int F, const void* W1, const void* W2, int H, float* P,
                            const Allocator& al, cudaStream_t s) {
  const int N2 = 2 * H;
  PFN_cuTensorMapEncodeTiled_v12000 enc = pg_encode();
  if (!enc) return fail(GS_ERR_CUDA, "gs_pass_attention: cuTensorMapEncodeTiled unavailable");
  DevBuf wt;
  if (!wt.ensure(al, (size_t)N2 * F * 2, s)) return fail(GS_ERR_OUT_OF_MEMORY, "gs_pass_attention: WT");
  pg_pack_wt_kernel<<<(N2 * F + 255) / 256, 256, 0, s>>>((const __nv_bfloat16*)W1, (const __nv_bfloat16*)W2, F, H,
                                                         (__nv_bfloat16*)wt.ptr);
  count_launch();
  CUtensorMap map;
  const cuuint64_t gdim[2] = {(cuuint64_t)F, (cuuint64_t)N};
  const cuuint64_t gstride[1] = {(cuuint64_t)F * 2};
  const cuuint32_t box[2] = {8, (cuuint32_t)PG_BM};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(X), gdim, gstride, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    wt.reset(al, s);
    return fail(GS_ERR_CUDA, "gs_pass_attention: cuTensorMapEncodeTiled failed (%d)", (int)r);
  }
  const size_t a_bytes = (size_t)PG_BM * F * 2, b_bytes = (size_t)N2 * F * 2;
  const size_t cap = 200 * 1024;
  int stages = (int)std::min<size_t>(6, (cap - b_bytes) / a_bytes);
  stages = std::max(stages, 2);
  const size_t smem = stages * a_bytes + b_bytes + (size_t)(2 * stages + 4) * 8 + 16;
  gs_status st = GS_OK;
  cudaError_t e = cudaFuncSetAttribute(proj_gemm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t tiles = (N + PG_BM - 1) / PG_BM;
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(tiles, sms));
    proj_gemm_kernel<<<grid, PG_THREADS, smem, s>>>(map, (const __nv_bfloat16*)wt.ptr, P, N, F, N2, stages);
    count_launch();
    e = cudaGetLastError();
  }
  if (e != cudaSuccess) st = cuda_fail(e, "proj_gemm_kernel launch");
  wt.reset(al, s);
  return st;
}

}  // namespace gsb

using namespace gsb;

extern "C" gs_status gs_pass_attention(const gs_graph* g, const void* X, int F, const void* W1,
                                       const void* W2, int H, const float* W3, void* stream_,
                                       float* att) {
  if (!g || !X || !W1 || !W2 || !W3 || (!att && g && g->num_edges > 0))
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_pass_attention: null pointer");
  if (F <= 0 || (H != 8 && H != 16 && H != 32 && H != PA_MAX_H))
    return fail(GS_ERR_NOT_SUPPORTED, "gs_pass_attention: F > 0 and H in {8, 16, 32, 64} required");
  cudaStream_t s = (cudaStream_t)stream_;
  const int64_t N = g->num_nodes, H2 = 2 * (int64_t)H;
  // softmax(W3) in fp64, libm exp, sum order (e0 + e1) + e2 (R29)
  const double m = std::max((double)W3[0], std::max((double)W3[1], (double)W3[2]));
  const double e0 = exp((double)W3[0] - m), e1 = exp((double)W3[1] - m), e2 = exp((double)W3[2] - m);
  const double tot = (e0 + e1) + e2;
  const double s0 = e0 / tot, s1 = e1 / tot, s2 = e2 / tot;
  if (N == 0 || g->num_edges == 0) return GS_OK;
  const Allocator al = g->al;
  DevBuf wc, P;
  if (!wc.ensure(al, (size_t)F * H2 * 2, s) || !P.ensure(al, (size_t)N * H2 * 4 + 16, s))
    return fail(GS_ERR_OUT_OF_MEMORY, "gs_pass_attention: device allocation failed");
  gs_status st = GS_OK;
  // [W1 | W2] as one row-major [F, 2H] bf16 operand
  cudaError_t ce = cudaMemcpy2DAsync(wc.ptr, H2 * 2, W1, (size_t)H * 2, (size_t)H * 2, F,
                                     cudaMemcpyDeviceToDevice, s);
  if (ce == cudaSuccess)
    ce = cudaMemcpy2DAsync((char*)wc.ptr + H * 2, H2 * 2, W2, (size_t)H * 2, (size_t)H * 2, F,
                           cudaMemcpyDeviceToDevice, s);
  if (ce != cudaSuccess) st = cuda_fail(ce, "gs_pass_attention: weight copy");
  const char* ge = getenv("GS_PASS_GEMM");
  const bool tc = F % 16 == 0 && F <= 256 && !(ge && ge[0] == 'c');
  if (st == GS_OK && tc) st = pg_project(X, N, F, W1, W2, H, (float*)P.ptr, al, s);
  if (st == GS_OK && !tc) {
    // row-major P[N, 2H] = X[N, F] Wc[F, 2H]  <=>  column-major P^T = Wc^T X^T
    cublasHandle_t h = pa_handle();
    if (!h) {
      st = fail(GS_ERR_CUDA, "gs_pass_attention: cublasCreate failed");
    } else {
      std::lock_guard<std::mutex> lk(pa_mutex);
      const float one = 1.0f, zero = 0.0f;
      cublasStatus_t cs = cublasSetStream(h, s);
      if (cs == CUBLAS_STATUS_SUCCESS)
        cs = cublasGemmEx(h, CUBLAS_OP_N, CUBLAS_OP_N, (int)H2, (int)N, F, &one, wc.ptr, CUDA_R_16BF,
                          (int)H2, X, CUDA_R_16BF, F, &zero, P.ptr, CUDA_R_32F, (int)H2,
                          CUBLAS_COMPUTE_32F, CUBLAS_GEMM_DEFAULT);
      if (cs != CUBLAS_STATUS_SUCCESS) st = fail(GS_ERR_CUDA, "gs_pass_attention: cublasGemmEx failed (%d)", (int)cs);
    }
  }
  if (st == GS_OK) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((N + PA_WARPS - 1) / PA_WARPS, (int64_t)sms * 8));
    const float* Pp = (const float*)P.ptr;
    switch (H) {
      case 8: pass_att_kernel<16><<<grid, PA_THREADS, 0, s>>>(g->indptr, g->indices, g->weights, g->colsum, Pp, N, s0, s1, s2, att); count_launch(); break;
      case 16: pass_att_kernel<32><<<grid, PA_THREADS, 0, s>>>(g->indptr, g->indices, g->weights, g->colsum, Pp, N, s0, s1, s2, att); count_launch(); break;
      case 32: pass_att_kernel<64><<<grid, PA_THREADS, 0, s>>>(g->indptr, g->indices, g->weights, g->colsum, Pp, N, s0, s1, s2, att); count_launch(); break;
      default: pass_att_kernel<128><<<grid, PA_THREADS, 0, s>>>(g->indptr, g->indices, g->weights, g->colsum, Pp, N, s0, s1, s2, att); count_launch(); break;
    }
    ce = cudaGetLastError();
    if (ce != cudaSuccess) st = cuda_fail(ce, "pass_att_kernel launch");
  }
  wc.reset(al, s);
  P.reset(al, s);
  return st;
}
