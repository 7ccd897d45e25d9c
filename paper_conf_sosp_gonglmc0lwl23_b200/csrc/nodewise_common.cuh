// nodewise_common.cuh -- device building blocks of the node-wise select
// (Extract + Select fused): per-warp chunks of 32 frontier columns and
// the weighted without-replacement select (A-Res, R6) by candidate filtering.
#pragma once
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include "common.cuh"
#include "gs_internal.h"

namespace gsb {

// Read-only graph + sampling parameters shared by the node-wise kernels.
struct NWCore {
  const int64_t* indptr;
  const int32_t* indices;
  const float* weights;
  const float* colsum;  // weighted graphs: fp32(sum_fp64 w) per column (a0)
  int64_t N;
  int* err;
  int replace, bias;
  uint64_t key;
  // host-mapped graphs: HBM copies of the hot pages (gs_graph_cache_hot), or NULL
  const int32_t* ptab;  // page -> slot in cidx / cw, -1 if not cached
  const int32_t* cidx;
  const float* cw;
  int cpsh;             // log2 entries per page
};

// Address of CSC entry pos of the index / weight array: its HBM copy when the
// page is cached (host-mapped graphs), else the array itself.
__device__ __forceinline__ const int32_t* nw_idx(const NWCore& P, int64_t pos) {
  if (P.ptab) {
    const int s = __ldg(P.ptab + (pos >> P.cpsh));
    if (s >= 0) return P.cidx + (((int64_t)s << P.cpsh) | (pos & ((int64_t(1) << P.cpsh) - 1)));
  }
  return P.indices + pos;
}
__device__ __forceinline__ const float* nw_w(const NWCore& P, int64_t pos) {
  if (P.ptab && P.cw) {
    const int s = __ldg(P.ptab + (pos >> P.cpsh));
    if (s >= 0) return P.cw + (((int64_t)s << P.cpsh) | (pos & ((int64_t(1) << P.cpsh) - 1)));
  }
  return P.weights + pos;
}

// Shared memory of one warp's chunk of 32 columns.
struct WarpChunk {
  uint32_t list[MAX_FANOUT][32];  // positions, [rank][column lane]
  int64_t coff[32];               // indptr[v]
  int64_t dcol[32];               // in-degree (0 for an invalid column)
  int32_t vcol[32];               // frontier node
  int32_t pre[32];                // exclusive prefix of the chunk's counts
  float csum[32];                 // PASS column sums
  int32_t cnt_all[32];            // count; bit 30: positions are 0..cnt-1
  uint32_t smask[MAX_FANOUT];     // slot -> column map: bit f set iff slot f starts a column
  uint8_t ne[32];                 // the chunk's non-empty columns, in order
};

// Builds the chunk's slot -> column map (warp-collective): slot f of the
// chunk's flat slot space belongs to column ne[r], r = (number of column
// starts <= f) - 1.  cnt / pre: this lane's column count and exclusive prefix.
__device__ __forceinline__ void chunk_map_build(WarpChunk& C, int cnt, int pre) {
  const int lane = threadIdx.x & 31;
  C.smask[lane] = 0u;
  __syncwarp();
  const unsigned nem = __ballot_sync(0xffffffffu, cnt > 0);
  if (cnt > 0) {
    atomicOr(&C.smask[pre >> 5], 1u << (pre & 31));
    C.ne[__popc(nem & ((1u << lane) - 1u))] = (uint8_t)lane;
  }
  __syncwarp();
}

// Column of slot f0 + lane in the round of slots [f0, f0 + 32) (f0 a multiple
// of 32, rounds visited in order); `starts` = column starts before f0, advanced.
__device__ __forceinline__ int chunk_map_col(const WarpChunk& C, int f0, int& starts) {
  const int lane = threadIdx.x & 31;
  const uint32_t w = C.smask[f0 >> 5];
  const int r = starts + __popc(w & ((2u << lane) - 1u)) - 1;
  starts += __popc(w);
  return C.ne[r < 0 ? 0 : r];
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

__device__ __forceinline__ long long warp_excl_ll(long long v, long long* total) {
  const int lane = threadIdx.x & 31;
  long long inc = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const long long n = __shfl_up_sync(0xffffffffu, inc, o);
    if (lane >= o) inc += n;
  }
  *total = __shfl_sync(0xffffffffu, inc, 31);
  return inc - v;
}

// ---------------------------------------------------------------------------
// A-Res by candidate filtering (R6).  The k smallest exact keys
// key_i = -ln((r_i + 0.5) 2^-32) / w_i (fp64, as the oracle) are found among
// the candidates {i : E_lb(r_i) <= tau w_i (1 + 1%)}, a superset of
// {i : key_i < tau}; whenever at least k exact keys fall below tau those
// candidates hold the answer.  tau = 2k / W (W = column weight sum) expects
// ~2k candidates, so only a handful of exact fp64 logarithms are taken per
// column: the stream costs one Philox per 4 edges, one weight load and one
// fp32 log per edge.  A tau that yields too few (or too many) is widened (or
// narrowed) and the column re-streamed -- rare.
// ---------------------------------------------------------------------------
// Candidate test E(r) <= t (conservatively: never rejects a true candidate)
// for E(r) = -ln((r + 0.5) 2^-32).  For r >= 2^31, E = -ln(1 - x) >= x + x^2/2
// with x = (2^32 - r - 0.5) 2^-32; for r < 2^31, E >= ln 2, so with
// t < 0.69 (the usual case: tau w is small) no logarithm is taken at all.
__device__ __forceinline__ bool ares_maybe_below(uint32_t r, float t) {
  if (r >= 0x80000000u) {
    const float x = __fmul_rn(__uint2float_rn(0xFFFFFFFFu - r) + 0.5f, 2.3283064365386963e-10f);
    return __fmaf_rn(0.5f * x, x, x) <= t;
  }
  if (t < 0.69f) return false;
  const float u = __fmul_rn(__uint2float_rn(r) + 0.5f, 2.3283064365386963e-10f);
  return -__logf(u) * 0.999f <= t;
}

// A-Res threshold search state: tau is widened / narrowed geometrically, or
// bisected once both a too-small and a too-large value are known.
struct TauSearch {
  float tau, lo, hi;
  __device__ bool next(int verdict, float tau0) {  // false: give up
    if (verdict == -3) { tau = -1.0f; return true; }
    if (verdict == -1) lo = tau;                     // too few below tau
    else hi = tau < 0.0f ? tau0 * 4.0f : tau;        // too many candidates
    if (lo > 0.0f && hi > 0.0f) {
      if (hi <= lo * 1.0001f) return false;
      tau = sqrtf(lo * hi);
    } else {
      tau = lo > 0.0f ? lo * 4.0f : hi * 0.25f;
    }
    return true;
  }
};

struct AresState {   // per filtering group (warp or CTA), in shared memory
  int m;             // candidates appended (may exceed the capacity)
  int elig;          // eligible (w > 0) edges seen
};

// Filter pass over column [off, off + d) by a group of NT threads (gtid in
// [0, NT)); candidate positions are appended to pos[0 .. cap).  tau < 0 means
// "every eligible edge".  The caller synchronises the group before and after.
template <int NT>
__device__ __forceinline__ void ares_filter(const NWCore& P, int32_t v, int64_t off, int64_t d, int l,
                                            uint32_t gb, float tau, int gtid, uint32_t* pos, int cap,
                                            AresState* st) {
  const int lane = threadIdx.x & 31;
  const uint64_t pf = pol_first();
  int elig = 0;
  for (int64_t base = 0; base < d; base += 4 * NT) {
    const int64_t i0 = base + 4 * (int64_t)gtid;
    float w[4] = {0.f, 0.f, 0.f, 0.f};
    uint32_t r[4] = {0u, 0u, 0u, 0u};
    if (i0 < d) {
      const U4 R = philox_nl((uint32_t)v, (uint32_t)(i0 >> 2), ctr2(l, TAG_ARES_NODE), gb, P.key);
      r[0] = R.x; r[1] = R.y; r[2] = R.z; r[3] = R.w;
#pragma unroll
      for (int q = 0; q < 4; ++q)
        w[q] = i0 + q < d ? (P.weights ? ldg_h(nw_w(P, off + i0 + q), pf) : 1.0f) : 0.0f;
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const bool e = w[q] > 0.0f;
      elig += e ? 1 : 0;
      const bool cand = e && (tau < 0.0f || ares_maybe_below(r[q], __fmul_rn(__fmul_rn(tau, w[q]), 1.01f)));
      const uint32_t bal = __ballot_sync(0xffffffffu, cand);
      if (bal) {
        int slot0 = 0;
        if (lane == 0) slot0 = atomicAdd(&st->m, __popc(bal));
        slot0 = __shfl_sync(0xffffffffu, slot0, 0);
        const int slot = slot0 + __popc(bal & ((1u << lane) - 1u));
        if (cand && slot < cap) pos[slot] = (uint32_t)(i0 + q);
      }
    }
  }
  for (int o = 16; o > 0; o >>= 1) elig += __shfl_xor_sync(0xffffffffu, elig, o);
  if (lane == 0 && elig) atomicAdd(&st->elig, elig);
}

// Exact step (one warp): fp64 keys of the candidates, then either the k
// smallest (ascending positions into out[.][c], returns the count) or a
// verdict: -1 widen tau, -2 narrow tau, -3 collect every eligible edge.
__device__ __forceinline__ int ares_exact(const NWCore& P, int32_t v, int64_t off, int l, uint32_t gb,
                                          int k, float tau, const uint32_t* pos, double* key, int* rk, int cap,
                                          const AresState& st, uint32_t (*out)[32], int c) {
  const int lane = threadIdx.x & 31;
  const int m = min(st.m, cap);
  if (st.elig <= k) {  // at most k eligible: all of them (R6)
    if (tau >= 0.0f) return -3;
  } else if (st.m > cap) {
    return -2;
  }
  int below = 0;
  for (int j = lane; j < m; j += 32) {
    const uint32_t p = pos[j];
    const U4 R = philox_nl((uint32_t)v, p >> 2, ctr2(l, TAG_ARES_NODE), gb, P.key);
    const float w = P.weights ? __ldg(nw_w(P, off + p)) : 1.0f;
    const double kk = ares_key_nl(sel_word(R, (int)(p & 3)), (double)w);
    key[j] = kk;
    below += (tau < 0.0f || kk < (double)tau) ? 1 : 0;
  }
  for (int o = 16; o > 0; o >>= 1) below += __shfl_xor_sync(0xffffffffu, below, o);
  __syncwarp();
  const int want = min(k, st.elig);
  if (below < want) return -1;
  // rank by (key, position); the selected ones are then ordered by position
  for (int j = lane; j < m; j += 32) {
    const double kj = key[j];
    const uint32_t pj = pos[j];
    int r = 0;
    for (int i = 0; i < m; ++i) r += key_less(key[i], pos[i], kj, pj) ? 1 : 0;
    rk[j] = r;
  }
  __syncwarp();
  for (int j = lane; j < m; j += 32) {
    if (rk[j] >= want) continue;
    const uint32_t pj = pos[j];
    int o = 0;
    for (int i = 0; i < m; ++i) o += (rk[i] < want && pos[i] < pj) ? 1 : 0;
    out[o][c] = pj;
  }
  __syncwarp();
  return want;
}

}  // namespace gsb
