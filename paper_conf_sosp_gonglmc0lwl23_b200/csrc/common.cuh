// common.cuh -- device primitives of the B200 ECSF path: counter-based RNG,
// integer draws, A-Res keys, per-(batch, layer) hash tables and warp/block scans.
// Independent of the CPU oracle (oracle/ shares no code with this directory).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace gsb {

// ---------------------------------------------------------------------------
// Philox4x32-10 (Salmon et al., SC'11).  Counter layout (R4):
//   c0 = subject (frontier node / candidate node / walker), c1 = slot,
//   c2 = layer_or_step | tag << 24, c3 = global batch index; key = rng_key.
// ---------------------------------------------------------------------------
struct U4 { uint32_t x, y, z, w; };

__device__ __forceinline__ U4 philox(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3,
                                     uint64_t key) {
  uint32_t k0 = (uint32_t)key, k1 = (uint32_t)(key >> 32);
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    uint32_t hi0 = __umulhi(0xD2511F53u, c0), lo0 = 0xD2511F53u * c0;
    uint32_t hi1 = __umulhi(0xCD9E8D57u, c2), lo1 = 0xCD9E8D57u * c2;
    uint32_t n0 = hi1 ^ c1 ^ k0, n2 = hi0 ^ c3 ^ k1;
    c0 = n0; c1 = lo1; c2 = n2; c3 = lo0;
    k0 += 0x9E3779B9u; k1 += 0xBB67AE85u;  // the 10th bump is never used
  }
  return U4{c0, c1, c2, c3};
}

// The same generator with the ten round keys precomputed (philox_keys, on the
// host): kept in kernel-parameter space they are constant-bank operands of the
// round's XOR, so a round is two wide multiplies and two LOP3s.
struct PhiloxKeys { uint32_t k[20]; };
inline PhiloxKeys philox_keys(uint64_t key) {
  PhiloxKeys r;
  uint32_t k0 = (uint32_t)key, k1 = (uint32_t)(key >> 32);
  for (int i = 0; i < 10; ++i) {
    r.k[2 * i] = k0;
    r.k[2 * i + 1] = k1;
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
  return r;
}
__device__ __forceinline__ U4 philox_k(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3, const PhiloxKeys& K) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    const uint64_t p0 = (uint64_t)0xD2511F53u * c0, p1 = (uint64_t)0xCD9E8D57u * c2;
    const uint32_t n0 = (uint32_t)(p1 >> 32) ^ c1 ^ K.k[2 * r], n2 = (uint32_t)(p0 >> 32) ^ c3 ^ K.k[2 * r + 1];
    c1 = (uint32_t)p1;
    c3 = (uint32_t)p0;
    c0 = n0;
    c2 = n2;
  }
  return U4{c0, c1, c2, c3};
}

// Out-of-line copies for the weighted select kernels: inlined at every call
// site they made the kernel ~9k instructions and its warps stalled on
// instruction fetch (ncu: no_instructions the top stall reason).
static __device__ __noinline__ U4 philox_nl(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3, uint64_t key) {
  return philox(c0, c1, c2, c3, key);
}

enum : uint32_t { TAG_FLOYD = 1, TAG_REPLACE = 2, TAG_ARES_NODE = 3, TAG_ARES_LAYER = 4,
                  TAG_DEEPWALK = 5, TAG_NODE2VEC = 6 };

__device__ __forceinline__ uint32_t ctr2(int layer, uint32_t tag) {
  return (uint32_t)layer | (tag << 24);
}

// floor(r * n / 2^64), r = hi:lo (R23).  Exact 64x64 -> high 64 product.
__device__ __forceinline__ uint64_t draw_below(uint64_t n, uint32_t lo, uint32_t hi) {
  uint64_t r = ((uint64_t)hi << 32) | lo;
  return __umul64hi(r, n);
}

// -ln((r + 0.5) 2^-32) / bias in fp64 (R6).
__device__ __forceinline__ double ares_key(uint32_t r, double bias) {
  double u = ((double)r + 0.5) * 0x1p-32;
  return -log(u) / bias;
}
static __device__ __noinline__ double ares_key_nl(uint32_t r, double bias) { return ares_key(r, bias); }

// (key, pos) lexicographic order: smaller key wins, ties -> smaller position.
__device__ __forceinline__ bool key_less(double ka, int64_t pa, double kb, int64_t pb) {
  return ka < kb || (ka == kb && pa < pb);
}

// ---------------------------------------------------------------------------
// Generation-tagged open-addressing table, one per cluster workspace.
// Entry = gen(8) | key(31) | val(25).  Entries whose gen differs from the
// current one are empty, so a table is reused without clearing for 255 uses.
// For a fixed (gen, key) the entry value is the atomicMin of all inserted
// vals: the first position at which the key occurs (R3, first occurrence).
// ---------------------------------------------------------------------------
constexpr int TAB_VAL_BITS = 25;
constexpr uint64_t TAB_VAL_MASK = (1ull << TAB_VAL_BITS) - 1;

__device__ __forceinline__ uint32_t tab_hash(uint32_t key, int log_cap) {
  return (key * 0x9E3779B1u) >> (32 - log_cap);
}
__device__ __forceinline__ uint64_t tab_entry(uint32_t gen, uint32_t key, uint32_t val) {
  return ((uint64_t)gen << 56) | ((uint64_t)key << TAB_VAL_BITS) | (uint64_t)val;
}
__device__ __forceinline__ uint32_t tab_gen(uint64_t e) { return (uint32_t)(e >> 56); }
__device__ __forceinline__ uint32_t tab_key(uint64_t e) {
  return (uint32_t)((e >> TAB_VAL_BITS) & 0x7FFFFFFFu);
}
__device__ __forceinline__ uint32_t tab_val(uint64_t e) { return (uint32_t)(e & TAB_VAL_MASK); }

// Insert key with val; keeps the minimum val per key.  Returns the slot.
__device__ __forceinline__ uint32_t tab_insert_min(unsigned long long* tab, int log_cap,
                                                   uint32_t gen, uint32_t key, uint32_t val) {
  const uint32_t mask = (1u << log_cap) - 1;
  const unsigned long long mine = tab_entry(gen, key, val);
  uint32_t h = tab_hash(key, log_cap);
  while (true) {
    unsigned long long old = __ldcg(&tab[h]);
    if (tab_gen(old) != gen) {
      unsigned long long prev = atomicCAS(&tab[h], old, mine);
      if (prev == old) return h;
      old = prev;
      if (tab_gen(old) != gen) continue;  // raced with a stale-entry writer: retry slot
    }
    if (tab_key(old) == key) {
      if ((uint32_t)tab_val(old) > val) atomicMin(&tab[h], mine);
      return h;
    }
    h = (h + 1) & mask;
  }
}

// Insert key if absent (value = val); returns slot and whether it was new.
__device__ __forceinline__ uint32_t tab_insert_once(unsigned long long* tab, int log_cap,
                                                    uint32_t gen, uint32_t key, uint32_t val,
                                                    bool* inserted) {
  const uint32_t mask = (1u << log_cap) - 1;
  const unsigned long long mine = tab_entry(gen, key, val);
  uint32_t h = tab_hash(key, log_cap);
  while (true) {
    unsigned long long old = __ldcg(&tab[h]);
    if (tab_gen(old) != gen) {
      unsigned long long prev = atomicCAS(&tab[h], old, mine);
      if (prev == old) { *inserted = true; return h; }
      old = prev;
      if (tab_gen(old) != gen) continue;
    }
    if (tab_key(old) == key) { *inserted = false; return h; }
    h = (h + 1) & mask;
  }
}

// Lookup: slot of key, or -1.  Call only after the inserting phase is fenced.
// Loads bypass L1 (ld.global.cg): L1 is not coherent with other SMs' atomics.
__device__ __forceinline__ int64_t tab_find(const unsigned long long* tab, int log_cap,
                                            uint32_t gen, uint32_t key) {
  const uint32_t mask = (1u << log_cap) - 1;
  uint32_t h = tab_hash(key, log_cap);
  while (true) {
    unsigned long long e = __ldcg(&tab[h]);
    if (tab_gen(e) != gen) return -1;
    if (tab_key(e) == key) return (int64_t)h;
    h = (h + 1) & mask;
  }
}

// ---------------------------------------------------------------------------
// Ordered open-addressing table (node-wise kernel).  Entry =
// tag(8) | key(31) | val(25) with tag = 255 - gen: entries of older
// generations (and the cleared value ~0) compare LARGER than every entry of
// the current generation, so one atomicMin both claims a stale slot and, for
// an equal key, keeps the minimum val (the first occurrence, R3).  When the
// atomicMin displaces a larger entry of another key, the displaced entry is
// carried on and re-inserted further along the probe sequence (ordered linear
// probing): no load-then-CAS round trip, one atomic per probe step.  Lookups
// scan from the hash until the key or a stale slot.  Between clears the
// generation must increase; a table is cleared to ~0 every 255 uses.
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t otag(uint32_t gen) { return 255u - gen; }

// Continues an insertion whose first atomicMin at slot h returned `old`.
__device__ __forceinline__ void otab_finish(unsigned long long* tab, uint32_t mask, uint32_t tag,
                                            uint32_t h, unsigned long long carry,
                                            unsigned long long old) {
  while (true) {
    if (tab_gen(old) != tag) return;               // stale slot: carry placed
    if (tab_key(old) == tab_key(carry)) return;    // same key: min kept
    if (old > carry) carry = old;                  // displaced: carry it on
    h = (h + 1) & mask;
    old = atomicMin(&tab[h], carry);
  }
}

__device__ __forceinline__ void otab_insert_min(unsigned long long* tab, int log_cap, uint32_t tag,
                                                uint32_t key, uint32_t val) {
  const unsigned long long e = tab_entry(tag, key, val);
  const uint32_t h = tab_hash(key, log_cap);
  otab_finish(tab, (1u << log_cap) - 1u, tag, h, e, atomicMin(&tab[h], e));
}

// Slot of key (current generation) or -1.
__device__ __forceinline__ int64_t otab_find(const unsigned long long* tab, int log_cap,
                                             uint32_t tag, uint32_t key) {
  const uint32_t mask = (1u << log_cap) - 1u;
  uint32_t h = tab_hash(key, log_cap);
  while (true) {
    const unsigned long long e = __ldcg(&tab[h]);
    if (tab_gen(e) != tag) return -1;
    if (tab_key(e) == key) return (int64_t)h;
    h = (h + 1) & mask;
  }
}

// ---------------------------------------------------------------------------
// L2 eviction-priority hints (createpolicy + .L2::cache_hint).  The graph
// gathers and the block outputs are streams (evict_first); the per-batch
// workspace (tables, staging) is reused within microseconds (evict_last), so
// it stays resident in the 126 MB L2 instead of being written back to HBM.
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint64_t pol_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t pol_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t pol_normal() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ int32_t ldh(const int32_t* a, uint64_t p) {
  int32_t v;
  asm volatile("ld.global.cg.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(a), "l"(p));
  return v;
}
__device__ __forceinline__ uint32_t ldh(const uint32_t* a, uint64_t p) {
  uint32_t v;
  asm volatile("ld.global.cg.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(a), "l"(p));
  return v;
}
__device__ __forceinline__ int64_t ldh(const int64_t* a, uint64_t p) {
  int64_t v;
  asm volatile("ld.global.cg.L2::cache_hint.b64 %0, [%1], %2;" : "=l"(v) : "l"(a), "l"(p));
  return v;
}
__device__ __forceinline__ unsigned long long ldh(const unsigned long long* a, uint64_t p) {
  unsigned long long v;
  asm volatile("ld.global.cg.L2::cache_hint.b64 %0, [%1], %2;" : "=l"(v) : "l"(a), "l"(p));
  return v;
}
__device__ __forceinline__ float ldh(const float* a, uint64_t p) {
  float v;
  asm volatile("ld.global.cg.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(a), "l"(p));
  return v;
}
// read-only graph data through the non-coherent path with a hint
__device__ __forceinline__ int32_t ldg_h(const int32_t* a, uint64_t p) {
  int32_t v;
  asm volatile("ld.global.nc.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(a), "l"(p));
  return v;
}
// predicated form (v unchanged when !on): no branch around the load, so a
// run of them stays in flight together -- a load inside an if() becomes a
// branch + reconvergence, and the compiler then waits on the loads' shared
// scoreboard before the next one is issued
__device__ __forceinline__ uint32_t ldg_h_if(bool on, const int32_t* a, uint64_t p, uint32_t v) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.global.nc.L2::cache_hint.b32 %0, [%1], %3; }"
               : "+r"(v) : "l"(a), "r"((int)on), "l"(p));
  return v;
}
__device__ __forceinline__ float ldg_h_if(bool on, const float* a, uint64_t p, float v) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.global.nc.L2::cache_hint.f32 %0, [%1], %3; }"
               : "+f"(v) : "l"(a), "r"((int)on), "l"(p));
  return v;
}
__device__ __forceinline__ int32_t ldcg_if(bool on, const int32_t* a, int32_t v) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.global.cg.b32 %0, [%1]; }"
               : "+r"(v) : "l"(a), "r"((int)on));
  return v;
}
__device__ __forceinline__ int64_t ldg_if(bool on, const int64_t* a, int64_t v) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.global.nc.b64 %0, [%1]; }"
               : "+l"(v) : "l"(a), "r"((int)on));
  return v;
}
__device__ __forceinline__ float ldg_if(bool on, const float* a, float v) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.global.nc.f32 %0, [%1]; }"
               : "+f"(v) : "l"(a), "r"((int)on));
  return v;
}
__device__ __forceinline__ int32_t ldg_if(bool on, const int32_t* a, int32_t v) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.global.nc.b32 %0, [%1]; }"
               : "+r"(v) : "l"(a), "r"((int)on));
  return v;
}
__device__ __forceinline__ int64_t ldg_h64(const int64_t* a, uint64_t p) {
  int64_t v;
  asm volatile("ld.global.nc.L2::cache_hint.b64 %0, [%1], %2;" : "=l"(v) : "l"(a), "l"(p));
  return v;
}
__device__ __forceinline__ float ldg_h(const float* a, uint64_t p) {
  float v;
  asm volatile("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(a), "l"(p));
  return v;
}
__device__ __forceinline__ void sth(int32_t* a, int32_t v, uint64_t p) {
  asm volatile("st.global.L2::cache_hint.b32 [%0], %1, %2;" ::"l"(a), "r"(v), "l"(p) : "memory");
}
__device__ __forceinline__ void sth(uint32_t* a, uint32_t v, uint64_t p) {
  asm volatile("st.global.L2::cache_hint.b32 [%0], %1, %2;" ::"l"(a), "r"(v), "l"(p) : "memory");
}
__device__ __forceinline__ void sth(int64_t* a, int64_t v, uint64_t p) {
  asm volatile("st.global.L2::cache_hint.b64 [%0], %1, %2;" ::"l"(a), "l"(v), "l"(p) : "memory");
}
__device__ __forceinline__ void sth(unsigned long long* a, unsigned long long v, uint64_t p) {
  asm volatile("st.global.L2::cache_hint.b64 [%0], %1, %2;" ::"l"(a), "l"(v), "l"(p) : "memory");
}
__device__ __forceinline__ void sth(float* a, float v, uint64_t p) {
  asm volatile("st.global.L2::cache_hint.f32 [%0], %1, %2;" ::"l"(a), "f"(v), "l"(p) : "memory");
}
__device__ __forceinline__ unsigned long long atom_cas_h(unsigned long long* a, unsigned long long cmp,
                                                         unsigned long long v, uint64_t) {
  // atom.cas takes no .L2::cache_hint; the table lines get their evict_last
  // priority from the hinted clears / loads
  return atomicCAS(a, cmp, v);
}

// ---------------------------------------------------------------------------
// Fixed-position table for concurrent insert + lookup (stream kernel).
// Entry = key(31) << 25 | val(25); EMPTY = ~0 (the table is reset to EMPTY
// after every use).  A key, once placed, never moves; its val only decreases
// (atomicMin), so lookups may run while later slots are still inserting.
// ---------------------------------------------------------------------------
constexpr unsigned long long CT_EMPTY = ~0ull;
__device__ __forceinline__ unsigned long long ct_entry(uint32_t key, uint32_t val) {
  return ((unsigned long long)key << TAB_VAL_BITS) | (unsigned long long)val;
}
// Continues an insertion whose first CAS(EMPTY -> mine) at slot h returned old.
__device__ __forceinline__ void ct_finish(unsigned long long* tab, uint32_t mask, uint32_t h,
                                          unsigned long long mine, unsigned long long old,
                                          uint64_t pol) {
  while (true) {
    if (old == CT_EMPTY) return;                                   // placed
    if ((old >> TAB_VAL_BITS) == (mine >> TAB_VAL_BITS)) {          // same key
      if (old > mine) atomicMin(&tab[h], mine);
      return;
    }
    h = (h + 1) & mask;
    old = atom_cas_h(&tab[h], CT_EMPTY, mine, pol);
  }
}
// Entry of key (its val = first slot) or CT_EMPTY when absent.
__device__ __forceinline__ unsigned long long ct_get(const unsigned long long* tab, int log_cap,
                                                     uint32_t key, uint64_t pol) {
  const uint32_t mask = (1u << log_cap) - 1u;
  uint32_t h = tab_hash(key, log_cap);
  while (true) {
    const unsigned long long e = ldh(&tab[h], pol);
    if (e == CT_EMPTY || (uint32_t)(e >> TAB_VAL_BITS) == key) return e;
    h = (h + 1) & mask;
  }
}

// ---------------------------------------------------------------------------
// Scans
// ---------------------------------------------------------------------------
template <typename T>
__device__ __forceinline__ T warp_inclusive_scan(T v) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T n = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += n;
  }
  return v;
}

// Block-wide exclusive scan; `total` gets the block sum.  scratch: >= 33 T.
template <typename T>
__device__ __forceinline__ T block_exclusive_scan(T v, T* scratch, T* total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  T inc = warp_inclusive_scan(v);
  if (lane == 31) scratch[wid] = inc;
  __syncthreads();
  if (wid == 0) {
    T s = lane < nw ? scratch[lane] : T(0);
    T si = warp_inclusive_scan(s);
    if (lane < nw) scratch[lane] = si - s;
    if (lane == nw - 1) scratch[32] = si;
  }
  __syncthreads();
  T ex = inc - v + scratch[wid];
  *total = scratch[32];
  __syncthreads();
  return ex;
}

template <typename T>
__device__ __forceinline__ T block_reduce_sum(T v, T* scratch) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  if (lane == 0) scratch[wid] = v;
  __syncthreads();
  if (wid == 0) {
    T s = lane < nw ? scratch[lane] : T(0);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) scratch[32] = s;
  }
  __syncthreads();
  T r = scratch[32];
  __syncthreads();
  return r;
}

}  // namespace gsb
