// proj_gemm.cuh -- the one dense contraction on the path (PASS's feature
// projection, Fig. 3(c) lines 3-4; R29): P[M, N2] = X[M, F] * Wc[F, N2],
// bf16 inputs, fp32 accumulation, on the 5th-generation tensor cores.
//
// A persistent, warp-specialised sm_100a kernel, one CTA per SM:
//   warp 0      TMA producer: per 128-row tile of X, F/8 tensor-map loads of a
//               {8 elements, 128 rows} box into a multi-stage shared-memory
//               ring (mbarrier complete_tx);
//   warp 1      allocates TMEM (2 accumulators of N2 fp32 columns) and one lane
//               issues tcgen05.mma (M=128, N=N2, K=16, kind::f16) from shared
//               memory descriptors; tcgen05.commit frees the smem stage and
//               hands the accumulator to the epilogue;
//   warps 2..5  epilogue: tcgen05.ld (32 lanes x 32 columns per load) and fp32
//               row stores; then release the accumulator.
// Operands are K-major in the canonical no-swizzle layout: core matrices of
// 8 rows x 16 bytes, K-chunk stride LBO, 8-row-group stride SBO = 128 B.  Wc is
// passed transposed (WT[N2][F], K contiguous) and staged once per CTA.
// X is memory-bound here (K = F is small): the tensor cores only have to keep
// up with HBM; the ring keeps STAGES tiles of X in flight per SM.
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace gsb {

constexpr int PG_THREADS = 192;  // 6 warps: TMA, MMA, 4 x epilogue
constexpr int PG_BM = 128;       // rows per tile (UMMA M)

__device__ __forceinline__ uint32_t pg_smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void pg_mbar_init(uint64_t* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(pg_smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void pg_mbar_expect_tx(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(pg_smem_u32(b)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void pg_mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(pg_smem_u32(b)) : "memory");
}
__device__ __forceinline__ void pg_mbar_wait(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "PG_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra PG_WAIT_%=;\n\t}" ::"r"(pg_smem_u32(b)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void pg_tma_load_2d(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
      ::"r"(pg_smem_u32(dst)), "l"((uint64_t)map), "r"(c0), "r"(c1), "r"(pg_smem_u32(bar))
      : "memory");
}
// UMMA shared-memory descriptor: K-major, no swizzle (canonical
// ((8,n),2):((1,SBO),LBO) in 16-byte units), version 1 (sm_100).
__device__ __forceinline__ uint64_t pg_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1 << 46;  // version
  return d;                // base offset 0, layout type 0 (SWIZZLE_NONE)
}
// Instruction descriptor, kind::f16: bf16 A/B, fp32 D, K-major A and B.
__host__ __device__ constexpr uint32_t pg_idesc(int M, int N) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

// P[M][N2] = X[M][F] * WT[N2][F]^T.  F % 16 == 0, N2 in {16, 32, ..., 128}.
__global__ void __launch_bounds__(PG_THREADS, 1) proj_gemm_kernel(const __grid_constant__ CUtensorMap tmX,
                                                                   const __nv_bfloat16* __restrict__ WT,
                                                                   float* __restrict__ P, int64_t M, int F,
                                                                   int N2, int stages) {
  extern __shared__ __align__(1024) unsigned char pg_smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t a_bytes = (uint32_t)PG_BM * F * 2;  // one X tile
  unsigned char* sA = pg_smem;                        // stages x a_bytes (1024-aligned)
  unsigned char* sB = sA + (size_t)stages * a_bytes;  // N2 x F bf16
  uint64_t* bars = (uint64_t*)(sB + (size_t)N2 * F * 2);
  uint64_t* full = bars;                 // [stages]
  uint64_t* empty = bars + stages;       // [stages]
  uint64_t* tfull = bars + 2 * stages;   // [2]
  uint64_t* tempty = tfull + 2;          // [2]
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);
  const int kchunks = F / 8;
  const int ngroups = N2 / 8;
  const int64_t ntiles = (M + PG_BM - 1) / PG_BM;

  // B operand: WT[n][f] -> core matrix (kc, ng) at (kc * ngroups + ng) * 128 + (n % 8) * 16
  for (int i = threadIdx.x; i < N2 * kchunks; i += PG_THREADS) {
    const int n = i / kchunks, kc = i - n * kchunks;
    const uint4 v = *reinterpret_cast<const uint4*>(WT + (size_t)n * F + kc * 8);
    *reinterpret_cast<uint4*>(sB + ((size_t)kc * ngroups + (n >> 3)) * 128 + (n & 7) * 16) = v;
  }
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      pg_mbar_init(full + s, 1);
      pg_mbar_init(empty + s, 1);
    }
    for (int a = 0; a < 2; ++a) {
      pg_mbar_init(tfull + a, 1);
      pg_mbar_init(tempty + a, 4);  // one arrive per epilogue warp
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {  // TMEM: two accumulators of N2 columns (power of two >= 32)
    const uint32_t cols = N2 * 2 <= 32 ? 32u : (N2 * 2 <= 64 ? 64u : (N2 * 2 <= 128 ? 128u : 256u));
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(pg_smem_u32(tmem_slot)),
                 "r"(cols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // B staged by generic stores
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {  // ---- TMA producer ----
      int it = 0;
      for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x, ++it) {
        const int s = it % stages;
        const uint32_t ph = (uint32_t)((it / stages) & 1);
        pg_mbar_wait(empty + s, ph ^ 1u);
        pg_mbar_expect_tx(full + s, a_bytes);
        unsigned char* dst = sA + (size_t)s * a_bytes;
        for (int kc = 0; kc < kchunks; ++kc)
          pg_tma_load_2d(dst + (size_t)kc * (PG_BM * 16), &tmX, full + s, kc * 8, (int)(t * PG_BM));
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // ---- MMA issuer ----
      const uint32_t idesc = pg_idesc(PG_BM, N2);
      const uint32_t lbo_a = PG_BM * 16, lbo_b = (uint32_t)ngroups * 128;
      int it = 0;
      for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x, ++it) {
        const int s = it % stages;
        const uint32_t ph = (uint32_t)((it / stages) & 1);
        const int acc = it & 1;
        const uint32_t aph = (uint32_t)((it >> 1) & 1);
        pg_mbar_wait(tempty + acc, aph ^ 1u);
        pg_mbar_wait(full + s, ph);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t a0 = pg_smem_u32(sA + (size_t)s * a_bytes), b0 = pg_smem_u32(sB);
        const uint32_t d_tmem = tmem + (uint32_t)(acc * N2);
        for (int ks = 0; ks < F / 16; ++ks) {
          const uint64_t da = pg_desc(a0 + ks * 2 * lbo_a, lbo_a, 128);
          const uint64_t db = pg_desc(b0 + ks * 2 * lbo_b, lbo_b, 128);
          const uint32_t accum = ks > 0 ? 1u : 0u;
          asm volatile(
              "{\n\t.reg .pred p;\n\t"
              "setp.ne.b32 p, %4, 0;\n\t"
              "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
              "l"(da), "l"(db), "r"(idesc), "r"(accum)
              : "memory");
        }
        // frees the smem stage once these MMAs have read it; then hands the
        // accumulator to the epilogue (commit implies before_thread_sync)
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                         pg_smem_u32(empty + s))
                     : "memory");
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                         pg_smem_u32(tfull + acc))
                     : "memory");
      }
    }
  } else {  // ---- epilogue: warps 2..5, TMEM lane quarter = warp % 4 ----
    const int q = warp & 3;
    int it = 0;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x, ++it) {
      const int acc = it & 1;
      const uint32_t aph = (uint32_t)((it >> 1) & 1);
      pg_mbar_wait(tfull + acc, aph);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const int64_t row = t * PG_BM + q * 32 + lane;
      float* prow = P + row * N2;
      for (int c0 = 0; c0 < N2; c0 += 16) {
        uint32_t r[16];
        const uint32_t taddr = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * N2 + c0);
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, "
            "%14, %15}, [%16];"
            : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
              "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]),
              "=r"(r[15])
            : "r"(taddr));
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        if (row < M) {
          float4* dst = reinterpret_cast<float4*>(prow + c0);
#pragma unroll
          for (int j = 0; j < 4; ++j)
            dst[j] = make_float4(__uint_as_float(r[4 * j]), __uint_as_float(r[4 * j + 1]),
                                 __uint_as_float(r[4 * j + 2]), __uint_as_float(r[4 * j + 3]));
        }
      }
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      __syncwarp();
      if (lane == 0) pg_mbar_arrive(tempty + acc);
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  if (warp == 1) {
    const uint32_t cols = N2 * 2 <= 32 ? 32u : (N2 * 2 <= 64 ? 64u : (N2 * 2 <= 128 ? 128u : 256u));
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(cols) : "memory");
  }
}

}  // namespace gsb
