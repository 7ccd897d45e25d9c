// capi.cu -- the C ABI of libgsb200 (include/gs.h): argument validation, error
// reporting, the allocator hook, graph ingest (a0) and result objects.  Every
// sampling step runs in the kernels of nodewise_wave.cu / shadow.cu / layerwise.cu / walk.cu.
#include <cuda_runtime.h>
#include <stdarg.h>
#include <stdint.h>
#include <stdio.h>
#include <string.h>
#include <stdlib.h>

#include <algorithm>
#include <vector>
#include <new>

#include "gs_internal.h"

namespace gsb {

// ---------------------------------------------------------------------------
// errors
// ---------------------------------------------------------------------------
static thread_local char g_err[512] = "";
thread_local int64_t g_launches = 0;
bool g_profiling = false;

void set_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
}

gs_status fail(gs_status st, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
  return st;
}

gs_status cuda_fail(cudaError_t e, const char* what) {
  set_error("CUDA error %d (%s) in %s", (int)e, cudaGetErrorString(e), what);
  return GS_ERR_CUDA;
}

// ---------------------------------------------------------------------------
// allocator
// ---------------------------------------------------------------------------
static Allocator g_alloc;

Allocator current_allocator() { return g_alloc; }

void* Allocator::allocate(size_t bytes, cudaStream_t s) const {
  if (bytes == 0) bytes = 256;
  if (alloc) return alloc(bytes, (void*)s, ctx);
  void* p = nullptr;
  if (cudaMalloc(&p, bytes) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return p;
}

void Allocator::release(void* p, size_t bytes, cudaStream_t s) const {
  if (!p) return;
  if (free_fn) free_fn(p, bytes, (void*)s, ctx);
  else cudaFree(p);
}

bool DevBuf::ensure(const Allocator& al, size_t need, cudaStream_t s, bool zero) {
  if (ptr && bytes >= need) return true;
  reset(al, s);
  size_t want = need + need / 8;  // headroom: epoch-to-epoch size jitter
  ptr = al.allocate(want, s);
  if (!ptr) return false;
  bytes = want;
  if (zero && cudaMemsetAsync(ptr, 0, bytes, s) != cudaSuccess) return false;
  return true;
}

void DevBuf::reset(const Allocator& al, cudaStream_t s) {
  if (ptr) al.release(ptr, bytes, s);
  ptr = nullptr;
  bytes = 0;
}

gs_status run_shadow(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                     int64_t batch_size, int64_t batch_base, const int32_t* fanouts, int L,
                     int bias, uint64_t key, cudaStream_t stream, gs_blocks* blk);
gs_status run_nodewise_wave(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                            int64_t batch_size, int64_t batch_base, const int32_t* fanouts, int L,
                            int replace, int bias, uint64_t key, cudaStream_t stream,
                            gs_blocks* blk);
gs_status run_nodewise_hop(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                           const int64_t* bptr_host, int64_t batch_size, int64_t nbatch,
                           int64_t batch_base, const int32_t* fanouts, int L, int replace, int bias,
                           uint64_t key, cudaStream_t stream, gs_blocks* blk);
// node-wise engine: the hop-synchronous kernels (default) or the round-1
// single-launch wave kernel (GS_NODEWISE=wave; host-mapped graphs)
gs_status run_nodewise(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                       int64_t batch_size, int64_t batch_base, const int32_t* fanouts, int L,
                       int replace, int bias, uint64_t key, cudaStream_t stream, gs_blocks* blk) {
  // host-mapped (UVA) graphs: the wave kernel (PD, index array in host
  // memory: 31.5 ms vs 81.6 for the hop engine's per-lane register gathers)
  const char* e = getenv("GS_NODEWISE");
  if ((e && e[0] == 'w') || (g->host_mapped && !(e && e[0] == 'h')))
    return run_nodewise_wave(g, seeds, num_seeds, batch_size, batch_base, fanouts, L, replace, bias, key,
                             stream, blk);
  return run_nodewise_hop(g, seeds, num_seeds, nullptr, batch_size, (num_seeds + batch_size - 1) / batch_size,
                          batch_base, fanouts, L, replace, bias, key, stream, blk);
}
gs_status run_induce(const gs_graph* g, const gs_blocks* nw, cudaStream_t stream, gs_blocks* blk);
gs_status run_layerwise(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                        int64_t batch_size, int64_t batch_base, const int32_t* n_per_layer,
                        int L, int prob_mode, uint64_t key, cudaStream_t stream, gs_blocks* blk);
gs_status launch_walk(const gs_graph* g, const int32_t* starts, int64_t num_walkers,
                      int64_t walker_base, int length, float p, float q, uint64_t key,
                      bool node2vec, bool plain, cudaStream_t stream, int32_t* traces,
                      int* err = nullptr);
gs_status run_pinsage(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                      int64_t batch_size, int64_t batch_base, const int32_t* topk, int L,
                      int num_walks, int walk_length, float restart, uint64_t key,
                      cudaStream_t stream, gs_blocks* blk);
gs_status run_saint_rw(const gs_graph* g, const int32_t* roots, int64_t num_roots,
                       int64_t batch_size, int64_t batch_base, int walk_length, uint64_t key,
                       cudaStream_t stream, gs_blocks* blk);

// ---------------------------------------------------------------------------
// a0: CSC validation (indptr monotone and in range, indices in [0, N),
// column sortedness, max in-degree).  flags: 1 bad indptr, 2 bad index, 4 unsorted.
// ---------------------------------------------------------------------------
__global__ void validate_csc_kernel(const int64_t* __restrict__ indptr,
                                    const int32_t* __restrict__ indices, int64_t N, int64_t nnz,
                                    int* flags, unsigned long long* max_deg) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  int local = 0;
  unsigned long long mdeg = 0;
  for (int64_t v = warp; v < N; v += nwarps) {
    const int64_t a = indptr[v], b = indptr[v + 1];
    if (lane == 0 && (a < 0 || b < a || b > nnz)) local |= 1;
    if (a < 0 || b < a || b > nnz) continue;
    mdeg = max(mdeg, (unsigned long long)(b - a));
    for (int64_t i = a + lane; i < b; i += 32) {
      const int32_t x = indices[i];
      if (x < 0 || (int64_t)x >= N) local |= 2;
      if (i + 1 < b && indices[i + 1] < x) local |= 4;
    }
  }
  if (warp == 0 && lane == 0 && (indptr[0] != 0 || indptr[N] != nnz)) local |= 1;
  local = __reduce_or_sync(0xffffffffu, local);
  if (lane == 0) {
    if (local) atomicOr(flags, local);
    atomicMax(max_deg, mdeg);
  }
}

// a0 pre-processing of weighted graphs: colsum[v] = fp32(sum_fp64 of
// the column's weights) -- the PASS A3 denominator (R11) and the scale of the
// A-Res candidate threshold (nodewise_wave.cu).
// Also poscnt[v] = #{w > 0} in the column: the number of eligible edges, so
// the weighted node-wise sampler knows each column's sample count min(k,
// poscnt) (R6) before it samples.
__global__ void colsum_kernel(const int64_t* __restrict__ indptr, const float* __restrict__ w,
                              int64_t N, float* __restrict__ colsum, int32_t* __restrict__ poscnt) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t v = warp; v < N; v += nwarps) {
    const int64_t a = indptr[v], b = indptr[v + 1];
    double sum = 0.0;
    int pos = 0;
    for (int64_t i = a + lane; i < b; i += 32) {
      const float x = w[i];
      sum += (double)x;
      pos += x > 0.0f ? 1 : 0;
    }
    for (int o = 16; o > 0; o >>= 1) {
      sum += __shfl_xor_sync(0xffffffffu, sum, o);
      pos += __shfl_xor_sync(0xffffffffu, pos, o);
    }
    if (lane == 0) {
      colsum[v] = (float)sum;
      poscnt[v] = pos;
    }
  }
}

static int num_sms() {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return sms;
}

}  // namespace gsb

using namespace gsb;

extern "C" {

const char* gs_last_error(void) { return g_err; }

const char* gs_status_string(gs_status s) {
  switch (s) {
    case GS_OK: return "GS_OK";
    case GS_ERR_INVALID_ARGUMENT: return "GS_ERR_INVALID_ARGUMENT";
    case GS_ERR_OUT_OF_MEMORY: return "GS_ERR_OUT_OF_MEMORY";
    case GS_ERR_CUDA: return "GS_ERR_CUDA";
    case GS_ERR_UNSORTED_GRAPH: return "GS_ERR_UNSORTED_GRAPH";
    case GS_ERR_INDEX_OUT_OF_RANGE: return "GS_ERR_INDEX_OUT_OF_RANGE";
    case GS_ERR_NOT_SUPPORTED: return "GS_ERR_NOT_SUPPORTED";
    case GS_ERR_CAPACITY: return "GS_ERR_CAPACITY";
    case GS_ERR_INVALID_GRAPH: return "GS_ERR_INVALID_GRAPH";
  }
  return "GS_ERR_UNKNOWN";
}

int gs_version(void) { return 200; }

int64_t gs_kernel_launches(void) { return g_launches; }

gs_status gs_set_profiling(int on) {
  g_profiling = on != 0;
  return GS_OK;
}

gs_status gs_blocks_profile(const gs_blocks* b, int i, const char** name, double* ms) {
  if (!b || !name || !ms) return fail(GS_ERR_INVALID_ARGUMENT, "gs_blocks_profile: null argument");
  if (i < 0 || i >= (int)b->prof.size()) return fail(GS_ERR_INVALID_ARGUMENT, "gs_blocks_profile: no entry %d", i);
  *name = b->prof[i].first.c_str();
  *ms = b->prof[i].second;
  return GS_OK;
}

gs_status gs_set_allocator(gs_alloc_fn alloc, gs_free_fn free_fn, void* ctx) {
  if ((alloc == nullptr) != (free_fn == nullptr))
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_set_allocator: alloc and free must both be set or both NULL");
  g_alloc.alloc = alloc;
  g_alloc.free_fn = free_fn;
  g_alloc.ctx = ctx;
  return GS_OK;
}

gs_status gs_graph_create(const int64_t* indptr, const int32_t* indices, const float* weights,
                          int64_t num_nodes, int64_t num_edges, uint32_t flags, void* stream_,
                          gs_graph** out) {
  if (!out || !indptr || (!indices && num_edges > 0) || num_nodes < 0 || num_edges < 0)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_graph_create: null pointer or negative size");
  if (num_nodes >= (int64_t(1) << 31))
    return fail(GS_ERR_NOT_SUPPORTED, "gs_graph_create: num_nodes must be < 2^31 (int32 ids)");
  if ((flags & GS_GRAPH_HOST_PTRS) && (flags & GS_GRAPH_BORROW))
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_graph_create: BORROW needs device pointers");
  cudaStream_t stream = (cudaStream_t)stream_;
  gs_graph* g = new (std::nothrow) gs_graph();
  if (!g) return fail(GS_ERR_OUT_OF_MEMORY, "gs_graph_create: host allocation failed");
  g->al = current_allocator();
  g->num_nodes = num_nodes;
  g->num_edges = num_edges;
  auto cleanup = [&](gs_status st) {
    gs_graph_destroy(g);
    return st;
  };
  if (flags & GS_GRAPH_HOST_MAPPED) {
    // beyond-HBM graphs (P:415 UVA): indptr copied to HBM, the
    // index / weight arrays stay in pinned host memory and every kernel reads
    // them through their mapped device aliases over the host link
    if (!(flags & GS_GRAPH_HOST_PTRS))
      return cleanup(fail(GS_ERR_INVALID_ARGUMENT, "gs_graph_create: HOST_MAPPED needs host pointers"));
    if (!g->b_indptr.ensure(g->al, (num_nodes + 1) * 8, stream))
      return cleanup(fail(GS_ERR_OUT_OF_MEMORY, "gs_graph_create: device allocation failed"));
    g->indptr = (int64_t*)g->b_indptr.ptr;
    cudaError_t e = cudaMemcpyAsync(g->indptr, indptr, (num_nodes + 1) * 8, cudaMemcpyHostToDevice, stream);
    if (e != cudaSuccess) return cleanup(cuda_fail(e, "gs_graph_create copy"));
    const void* arrs[2] = {indices, weights};
    for (int k = 0; k < 2; ++k) {
      if (!arrs[k] || num_edges == 0) continue;
      void* hp = const_cast<void*>(arrs[k]);
      e = cudaHostRegister(hp, (size_t)num_edges * 4, cudaHostRegisterMapped | cudaHostRegisterReadOnly);
      if (e == cudaErrorHostMemoryAlreadyRegistered) {
        cudaGetLastError();  // already pinned by the caller: use its mapping, do not unregister
      } else if (e != cudaSuccess) {
        return cleanup(cuda_fail(e, "gs_graph_create: cudaHostRegister"));
      } else {
        g->host_reg[g->n_reg++] = hp;
      }
      void* dp = nullptr;
      e = cudaHostGetDevicePointer(&dp, hp, 0);
      if (e != cudaSuccess) return cleanup(cuda_fail(e, "gs_graph_create: cudaHostGetDevicePointer"));
      if (k == 0) g->indices = (int32_t*)dp;
      else g->weights = (float*)dp;
    }
    g->host_mapped = true;
  } else if (flags & GS_GRAPH_BORROW) {
    g->indptr = const_cast<int64_t*>(indptr);
    g->indices = const_cast<int32_t*>(indices);
    g->weights = const_cast<float*>(weights);
  } else {
    const cudaMemcpyKind kind =
        (flags & GS_GRAPH_HOST_PTRS) ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
    if (!g->b_indptr.ensure(g->al, (num_nodes + 1) * 8, stream) ||
        !g->b_indices.ensure(g->al, std::max<int64_t>(num_edges, 1) * 4, stream) ||
        (weights && !g->b_weights.ensure(g->al, std::max<int64_t>(num_edges, 1) * 4, stream)))
      return cleanup(fail(GS_ERR_OUT_OF_MEMORY, "gs_graph_create: device allocation failed"));
    g->owns = true;
    g->indptr = (int64_t*)g->b_indptr.ptr;
    g->indices = (int32_t*)g->b_indices.ptr;
    g->weights = weights ? (float*)g->b_weights.ptr : nullptr;
    cudaError_t e = cudaMemcpyAsync(g->indptr, indptr, (num_nodes + 1) * 8, kind, stream);
    if (e == cudaSuccess && num_edges)
      e = cudaMemcpyAsync(g->indices, indices, num_edges * 4, kind, stream);
    if (e == cudaSuccess && weights && num_edges)
      e = cudaMemcpyAsync(g->weights, weights, num_edges * 4, kind, stream);
    if (e != cudaSuccess) return cleanup(cuda_fail(e, "gs_graph_create copy"));
  }
  if (!g->b_err.ensure(g->al, 64, stream, true))
    return cleanup(fail(GS_ERR_OUT_OF_MEMORY, "gs_graph_create: device allocation failed"));
  g->d_err = (int*)g->b_err.ptr;
  int* d_flags = g->d_err + 4;
  unsigned long long* d_maxdeg = (unsigned long long*)(g->d_err + 8);
  const int sms = num_sms();
  int64_t blocks = std::max<int64_t>(1, std::min<int64_t>((num_nodes + 7) / 8, (int64_t)sms * 16));
  validate_csc_kernel<<<(unsigned)blocks, 256, 0, stream>>>(g->indptr, g->indices, num_nodes,
                                                             num_edges, d_flags, d_maxdeg); count_launch();
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cleanup(cuda_fail(e, "validate_csc_kernel launch"));
  int h[16] = {0};
  e = cudaMemcpyAsync(h, g->d_err, sizeof(h), cudaMemcpyDeviceToHost, stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
  if (e != cudaSuccess) return cleanup(cuda_fail(e, "gs_graph_create validation"));
  const int vflags = h[4];
  unsigned long long mdeg = 0;
  memcpy(&mdeg, &h[8], sizeof(mdeg));
  if (vflags & 1) return cleanup(fail(GS_ERR_INVALID_GRAPH, "gs_graph_create: indptr is not a valid CSC offset array"));
  if (vflags & 2) return cleanup(fail(GS_ERR_INVALID_GRAPH, "gs_graph_create: an index is outside [0, num_nodes)"));
  g->sorted = (vflags & 4) ? 0 : 1;
  g->max_in_degree = (int64_t)mdeg;
  if (g->weights) {
    if (!g->b_colsum.ensure(g->al, std::max<int64_t>(num_nodes, 1) * 4, stream) ||
        !g->b_poscnt.ensure(g->al, std::max<int64_t>(num_nodes, 1) * 4, stream))
      return cleanup(fail(GS_ERR_OUT_OF_MEMORY, "gs_graph_create: device allocation failed"));
    g->colsum = (float*)g->b_colsum.ptr;
    g->poscnt = (int32_t*)g->b_poscnt.ptr;
    colsum_kernel<<<(unsigned)blocks, 256, 0, stream>>>(g->indptr, g->weights, num_nodes, g->colsum,
                                                         g->poscnt); count_launch();
    e = cudaGetLastError();
    if (e != cudaSuccess) return cleanup(cuda_fail(e, "colsum_kernel launch"));
  }
  cudaMemsetAsync(g->d_err, 0, 64, stream);
  *out = g;
  return GS_OK;
}

gs_status gs_graph_set_weights(gs_graph* g, const float* weights, uint32_t flags, void* stream_) {
  if (!g || (!weights && g->num_edges > 0))
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_graph_set_weights: null pointer");
  cudaStream_t stream = (cudaStream_t)stream_;
  if (flags & GS_GRAPH_BORROW) {
    g->weights = const_cast<float*>(weights);
  } else {
    if (!g->b_weights.ensure(g->al, (size_t)std::max<int64_t>(g->num_edges, 1) * 4, stream))
      return fail(GS_ERR_OUT_OF_MEMORY, "gs_graph_set_weights: device allocation failed");
    g->weights = (float*)g->b_weights.ptr;
    if (g->num_edges)
      GS_CUDA_TRY(cudaMemcpyAsync(g->weights, weights, g->num_edges * 4, cudaMemcpyDeviceToDevice, stream));
  }
  if (!g->b_colsum.ensure(g->al, (size_t)std::max<int64_t>(g->num_nodes, 1) * 4, stream) ||
      !g->b_poscnt.ensure(g->al, (size_t)std::max<int64_t>(g->num_nodes, 1) * 4, stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "gs_graph_set_weights: device allocation failed");
  g->colsum = (float*)g->b_colsum.ptr;
  g->poscnt = (int32_t*)g->b_poscnt.ptr;
  const int64_t blocks = std::max<int64_t>(1, std::min<int64_t>((g->num_nodes + 7) / 8, (int64_t)num_sms() * 16));
  if (g->num_nodes > 0) {
    colsum_kernel<<<(unsigned)blocks, 256, 0, stream>>>(g->indptr, g->weights, g->num_nodes, g->colsum, g->poscnt);
    count_launch();
  }
  GS_CUDA_TRY(cudaGetLastError());
  return GS_OK;
}

gs_status gs_graph_get_info(const gs_graph* g, gs_graph_info* out) {
  if (!g || !out) return fail(GS_ERR_INVALID_ARGUMENT, "gs_graph_get_info: null pointer");
  out->num_nodes = g->num_nodes;
  out->num_edges = g->num_edges;
  out->weighted = g->weights != nullptr;
  out->sorted = g->sorted;
  out->max_in_degree = g->max_in_degree;
  out->indptr = g->indptr;
  out->indices = g->indices;
  out->weights = g->weights;
  out->host_mapped = g->host_mapped ? 1 : 0;
  out->cached_pages = g->ptab ? g->cached_pages : 0;
  out->cache_page_entries = int64_t(1) << g->cpsh;
  return GS_OK;
}

// Hot-page cache (gs_graph_cache_hot): score[p] = sum over the CSC entries of
// page p of min(32, in-degree of the entry's column) -- the expected
// node-wise accesses of an entry when frontier nodes come in proportion to
// degree and a column access reads min(k, d) of its d entries.
__global__ void page_score_kernel(const int64_t* __restrict__ indptr, int64_t N, int psh,
                                  unsigned long long* __restrict__ score) {
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < N; v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t a = indptr[v], b = indptr[v + 1];
    if (b <= a) continue;
    const unsigned long long wgt = (unsigned long long)(b - a < 32 ? b - a : 32);
    for (int64_t p = a >> psh; p <= (b - 1) >> psh; ++p) {
      const int64_t lo = max(a, p << psh), hi = min(b, (p + 1) << psh);
      atomicAdd(score + p, (unsigned long long)(hi - lo) * wgt);
    }
  }
}

// Copies page slot_page[s] of the (host-mapped) index / weight arrays into slot s.
__global__ void page_copy_kernel(const int32_t* __restrict__ idx, const float* __restrict__ w, int64_t nnz, int psh,
                                 const int32_t* __restrict__ slot_page, int32_t* __restrict__ cidx,
                                 float* __restrict__ cw) {
  const int64_t s = blockIdx.x;
  const int64_t p = slot_page[s];
  const int64_t a = p << psh, b = min(nnz, (p + 1) << psh);
  for (int64_t i = a + threadIdx.x; i < b; i += blockDim.x) {
    cidx[(s << psh) + (i - a)] = idx[i];
    if (w) cw[(s << psh) + (i - a)] = w[i];
  }
}

gs_status gs_graph_cache_hot(gs_graph* g, int64_t budget_bytes, void* stream_) {
  if (!g || !g->host_mapped || budget_bytes < 0)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_graph_cache_hot: needs a host-mapped graph and budget >= 0");
  cudaStream_t stream = (cudaStream_t)stream_;
  g->ptab = nullptr;
  g->cidx = nullptr;
  g->cw = nullptr;
  g->cached_pages = 0;
  const int psh = g->cpsh;
  const int64_t npages = (g->num_edges + (int64_t(1) << psh) - 1) >> psh;
  const int64_t page_bytes = (int64_t(1) << psh) * (g->weights ? 8 : 4);
  const int64_t nsel = std::min<int64_t>(npages, budget_bytes / page_bytes);
  if (nsel <= 0) return GS_OK;
  // page scores on the device, ranked on the host
  gsb::DevBuf sc;
  if (!sc.ensure(g->al, (size_t)npages * 8, stream, true))
    return fail(GS_ERR_OUT_OF_MEMORY, "gs_graph_cache_hot: device allocation failed");
  const int64_t blocks = std::max<int64_t>(1, std::min<int64_t>((g->num_nodes + 255) / 256, (int64_t)num_sms() * 16));
  page_score_kernel<<<(unsigned)blocks, 256, 0, stream>>>(g->indptr, g->num_nodes, psh,
                                                           (unsigned long long*)sc.ptr);
  count_launch();
  std::vector<unsigned long long> score((size_t)npages);
  GS_CUDA_TRY(cudaMemcpyAsync(score.data(), sc.ptr, (size_t)npages * 8, cudaMemcpyDeviceToHost, stream));
  GS_CUDA_TRY(cudaStreamSynchronize(stream));
  sc.reset(g->al, stream);
  std::vector<int32_t> order((size_t)npages);
  for (int64_t p = 0; p < npages; ++p) order[(size_t)p] = (int32_t)p;
  std::partial_sort(order.begin(), order.begin() + nsel, order.end(), [&](int32_t a, int32_t b) {
    return score[(size_t)a] > score[(size_t)b] || (score[(size_t)a] == score[(size_t)b] && a < b);
  });
  order.resize((size_t)nsel);
  std::sort(order.begin(), order.end());  // slots in page order
  std::vector<int32_t> ptab((size_t)npages, -1);
  for (int64_t s = 0; s < nsel; ++s) ptab[(size_t)order[(size_t)s]] = (int32_t)s;
  gsb::DevBuf sp;
  if (!g->b_ptab.ensure(g->al, (size_t)npages * 4, stream) ||
      !g->b_cidx.ensure(g->al, (size_t)nsel << psh << 2, stream) ||
      (g->weights && !g->b_cw.ensure(g->al, (size_t)nsel << psh << 2, stream)) ||
      !sp.ensure(g->al, (size_t)nsel * 4, stream))
    return fail(GS_ERR_OUT_OF_MEMORY, "gs_graph_cache_hot: device allocation failed (cache)");
  GS_CUDA_TRY(cudaMemcpyAsync(g->b_ptab.ptr, ptab.data(), (size_t)npages * 4, cudaMemcpyHostToDevice, stream));
  GS_CUDA_TRY(cudaMemcpyAsync(sp.ptr, order.data(), (size_t)nsel * 4, cudaMemcpyHostToDevice, stream));
  page_copy_kernel<<<(unsigned)nsel, 512, 0, stream>>>(g->indices, g->weights, g->num_edges, psh,
                                                       (const int32_t*)sp.ptr, (int32_t*)g->b_cidx.ptr,
                                                       g->weights ? (float*)g->b_cw.ptr : nullptr);
  count_launch();
  GS_CUDA_TRY(cudaGetLastError());
  GS_CUDA_TRY(cudaStreamSynchronize(stream));  // the host vectors above die with this call
  sp.reset(g->al, stream);
  g->ptab = (int32_t*)g->b_ptab.ptr;
  g->cidx = (int32_t*)g->b_cidx.ptr;
  g->cw = g->weights ? (float*)g->b_cw.ptr : nullptr;
  g->cached_pages = nsel;
  return GS_OK;
}

void gs_graph_destroy(gs_graph* g) {
  if (!g) return;
  cudaStream_t s = nullptr;
  g->b_indptr.reset(g->al, s);
  g->b_indices.reset(g->al, s);
  g->b_weights.reset(g->al, s);
  g->b_colsum.reset(g->al, s);
  g->b_poscnt.reset(g->al, s);
  g->b_deg.reset(g->al, s);
  g->b_degsrc.reset(g->al, s);
  g->b_walk.reset(g->al, s);
  g->b_err.reset(g->al, s);
  g->b_ptab.reset(g->al, s);
  g->b_cidx.reset(g->al, s);
  g->b_cw.reset(g->al, s);
  for (int k = 0; k < g->n_reg; ++k) cudaHostUnregister(g->host_reg[k]);
  delete g;
}

static gs_status check_batches(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                               int64_t batch_size, int64_t batch_base, const int32_t* per_layer,
                               int num_layers, gs_blocks** out) {
  if (!g || !out || (!seeds && num_seeds > 0) || !per_layer)
    return fail(GS_ERR_INVALID_ARGUMENT, "null pointer argument");
  if (num_seeds < 0 || batch_size <= 0 || batch_base < 0)
    return fail(GS_ERR_INVALID_ARGUMENT, "num_seeds >= 0, batch_size > 0, batch_index_base >= 0 required");
  if (num_layers < 1 || num_layers > MAX_LAYERS)
    return fail(GS_ERR_INVALID_ARGUMENT, "num_layers must be in [1, %d]", MAX_LAYERS);
  if (num_seeds >= (int64_t(1) << 31))
    return fail(GS_ERR_NOT_SUPPORTED, "num_seeds must be < 2^31");
  for (int l = 0; l < num_layers; ++l)
    if (per_layer[l] <= 0) return fail(GS_ERR_INVALID_ARGUMENT, "fanout / layer size must be > 0");
  return GS_OK;
}

static gs_status prepare_blocks(gs_blocks** out, cudaStream_t stream, const gs_graph* g) {
  if (!*out) {
    gs_blocks* b = new (std::nothrow) gs_blocks();
    if (!b) return fail(GS_ERR_OUT_OF_MEMORY, "host allocation failed");
    b->al = current_allocator();
    *out = b;
  }
  (*out)->stream = stream;
  (*out)->synced = false;
  (*out)->graph_edges = g ? g->num_edges : 0;
  return GS_OK;
}

gs_status gs_sample_neighbors(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                              int64_t batch_size, int64_t batch_index_base,
                              const int32_t* fanouts, int num_layers, int replace, int bias_mode,
                              uint64_t rng_key, void* stream_, gs_blocks** out) {
  gs_status st = check_batches(g, seeds, num_seeds, batch_size, batch_index_base, fanouts,
                               num_layers, out);
  if (st) return st;
  if (bias_mode < 0 || bias_mode > 2) return fail(GS_ERR_INVALID_ARGUMENT, "unknown bias_mode %d", bias_mode);
  if (replace && bias_mode != GS_W_UNIFORM)
    return fail(GS_ERR_NOT_SUPPORTED, "weighted sampling with replacement is not implemented");
  int64_t prod = batch_size;
  for (int l = 0; l < num_layers; ++l) {
    if (fanouts[l] > MAX_FANOUT) return fail(GS_ERR_NOT_SUPPORTED, "fanout must be <= %d", MAX_FANOUT);
    prod *= fanouts[l];
    if (prod > MAX_SLOTS_PER_BATCH)
      return fail(GS_ERR_NOT_SUPPORTED, "batch_size * prod(fanouts) must be <= 2^25");
  }
  cudaStream_t stream = (cudaStream_t)stream_;
  if ((st = prepare_blocks(out, stream, g))) return st;
  return run_nodewise(g, seeds, num_seeds, batch_size, batch_index_base, fanouts,
                      num_layers, replace, bias_mode, rng_key, stream, *out);
}

gs_status gs_sample_neighbors_ragged(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                                     const int64_t* batch_ptr, int64_t num_batches, int64_t batch_index_base,
                                     const int32_t* fanouts, int num_layers, int replace, int bias_mode,
                                     uint64_t rng_key, void* stream_, gs_blocks** out) {
  if (!batch_ptr || num_batches < 0) return fail(GS_ERR_INVALID_ARGUMENT, "batch_ptr: null or negative num_batches");
  int64_t maxbs = 1;
  if (batch_ptr[0] != 0 || batch_ptr[num_batches] != num_seeds)
    return fail(GS_ERR_INVALID_ARGUMENT, "batch_ptr must start at 0 and end at num_seeds");
  for (int64_t b = 0; b < num_batches; ++b) {
    if (batch_ptr[b + 1] < batch_ptr[b]) return fail(GS_ERR_INVALID_ARGUMENT, "batch_ptr must be non-decreasing");
    maxbs = std::max<int64_t>(maxbs, batch_ptr[b + 1] - batch_ptr[b]);
  }
  gs_status st = check_batches(g, seeds, num_seeds, maxbs, batch_index_base, fanouts, num_layers, out);
  if (st) return st;
  if (bias_mode < 0 || bias_mode > 2) return fail(GS_ERR_INVALID_ARGUMENT, "unknown bias_mode %d", bias_mode);
  if (replace && bias_mode != GS_W_UNIFORM)
    return fail(GS_ERR_NOT_SUPPORTED, "weighted sampling with replacement is not implemented");
  int64_t prod = maxbs;
  for (int l = 0; l < num_layers; ++l) {
    if (fanouts[l] > MAX_FANOUT) return fail(GS_ERR_NOT_SUPPORTED, "fanout must be <= %d", MAX_FANOUT);
    prod *= fanouts[l];
    if (prod > MAX_SLOTS_PER_BATCH)
      return fail(GS_ERR_NOT_SUPPORTED, "max batch size * prod(fanouts) must be <= 2^25");
  }
  cudaStream_t stream = (cudaStream_t)stream_;
  if ((st = prepare_blocks(out, stream, g))) return st;
  return run_nodewise_hop(g, seeds, num_seeds, batch_ptr, 0, num_batches, batch_index_base, fanouts, num_layers,
                          replace, bias_mode, rng_key, stream, *out);
}

gs_status gs_induce_subgraph(const gs_graph* g, const gs_blocks* sampled, void* stream_, gs_blocks** out) {
  if (!g || !sampled || !out) return fail(GS_ERR_INVALID_ARGUMENT, "gs_induce_subgraph: null argument");
  if (*out == sampled) return fail(GS_ERR_INVALID_ARGUMENT, "gs_induce_subgraph: out must differ from sampled");
  if (sampled->kind != gs_blocks::NODEWISE)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_induce_subgraph: sampled must come from gs_sample_neighbors");
  cudaStream_t stream = (cudaStream_t)stream_;
  gs_status st = prepare_blocks(out, stream, g);
  if (st) return st;
  return run_induce(g, sampled, stream, *out);
}

gs_status gs_sample_shadow(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                           int64_t batch_size, int64_t batch_index_base, const int32_t* fanouts,
                           int num_layers, int bias_mode, uint64_t rng_key, void* stream_,
                           gs_blocks** out) {
  gs_status st = check_batches(g, seeds, num_seeds, batch_size, batch_index_base, fanouts,
                               num_layers, out);
  if (st) return st;
  if (bias_mode < 0 || bias_mode > 1) return fail(GS_ERR_INVALID_ARGUMENT, "ShaDow bias_mode must be UNIFORM or EDGE");
  int64_t prod = batch_size, sum = batch_size;
  for (int l = 0; l < num_layers; ++l) {
    if (fanouts[l] > MAX_FANOUT) return fail(GS_ERR_NOT_SUPPORTED, "fanout must be <= %d", MAX_FANOUT);
    prod *= fanouts[l];
    sum += prod;
    if (sum > MAX_SLOTS_PER_BATCH)
      return fail(GS_ERR_NOT_SUPPORTED, "batch_size * (1 + sum of fanout products) must be <= 2^25");
  }
  cudaStream_t stream = (cudaStream_t)stream_;
  if ((st = prepare_blocks(out, stream, g))) return st;
  return run_shadow(g, seeds, num_seeds, batch_size, batch_index_base, fanouts, num_layers,
                    bias_mode, rng_key, stream, *out);
}

gs_status gs_sample_saint_rw(const gs_graph* g, const int32_t* roots, int64_t num_roots,
                             int64_t batch_size, int64_t batch_index_base, int walk_length,
                             uint64_t rng_key, void* stream_, gs_blocks** out) {
  if (!g || !out || (!roots && num_roots > 0))
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_sample_saint_rw: null pointer argument");
  if (num_roots < 0 || batch_size <= 0 || batch_index_base < 0 || walk_length < 0 ||
      walk_length >= (1 << 24))
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_sample_saint_rw: bad num_roots/batch_size/base/walk_length");
  if (num_roots >= (int64_t(1) << 31) || batch_size * ((int64_t)walk_length + 1) > MAX_SLOTS_PER_BATCH)
    return fail(GS_ERR_NOT_SUPPORTED, "gs_sample_saint_rw: batch_size * (walk_length + 1) must be <= 2^25");
  if ((batch_index_base + (num_roots + batch_size - 1) / batch_size) * batch_size > (int64_t(1) << 32))
    return fail(GS_ERR_NOT_SUPPORTED, "gs_sample_saint_rw: global walker ids must fit 32 bits");
  cudaStream_t stream = (cudaStream_t)stream_;
  gs_status st = prepare_blocks(out, stream, g);
  if (st) return st;
  return run_saint_rw(g, roots, num_roots, batch_size, batch_index_base, walk_length, rng_key,
                      stream, *out);
}

gs_status gs_sample_pinsage(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                            int64_t batch_size, int64_t batch_index_base, const int32_t* topk,
                            int num_layers, int num_walks, int walk_length, float restart_prob,
                            uint64_t rng_key, void* stream_, gs_blocks** out) {
  gs_status st = check_batches(g, seeds, num_seeds, batch_size, batch_index_base, topk,
                               num_layers, out);
  if (st) return st;
  if (num_walks < 1 || walk_length < 1 || !(restart_prob >= 0.0f) || !(restart_prob <= 1.0f))
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_sample_pinsage: num_walks, walk_length >= 1 and restart_prob in [0, 1] required");
  if ((int64_t)num_walks * walk_length > 2048)
    return fail(GS_ERR_NOT_SUPPORTED, "gs_sample_pinsage: num_walks * walk_length must be <= 2048");
  int64_t prod = batch_size;
  for (int l = 0; l < num_layers; ++l) {
    if (topk[l] > MAX_FANOUT) return fail(GS_ERR_NOT_SUPPORTED, "top-k must be <= %d", MAX_FANOUT);
    prod *= topk[l];
    if (prod > MAX_SLOTS_PER_BATCH)
      return fail(GS_ERR_NOT_SUPPORTED, "batch_size * prod(topk) must be <= 2^25");
  }
  cudaStream_t stream = (cudaStream_t)stream_;
  if ((st = prepare_blocks(out, stream, g))) return st;
  return run_pinsage(g, seeds, num_seeds, batch_size, batch_index_base, topk, num_layers, num_walks,
                     walk_length, restart_prob, rng_key, stream, *out);
}

gs_status gs_sample_layerwise(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                              int64_t batch_size, int64_t batch_index_base,
                              const int32_t* n_per_layer, int num_layers, int prob_mode,
                              uint64_t rng_key, void* stream_, gs_blocks** out) {
  gs_status st = check_batches(g, seeds, num_seeds, batch_size, batch_index_base, n_per_layer,
                               num_layers, out);
  if (st) return st;
  if (prob_mode < 0 || prob_mode > 2) return fail(GS_ERR_INVALID_ARGUMENT, "unknown prob_mode %d", prob_mode);
  for (int l = 0; l < num_layers; ++l)
    if (n_per_layer[l] > 4096) return fail(GS_ERR_NOT_SUPPORTED, "n_per_layer must be <= 4096");
  if (batch_size > 4096) return fail(GS_ERR_NOT_SUPPORTED, "layer-wise batch_size must be <= 4096");
  cudaStream_t stream = (cudaStream_t)stream_;
  if ((st = prepare_blocks(out, stream, g))) return st;
  return run_layerwise(g, seeds, num_seeds, batch_size, batch_index_base, n_per_layer, num_layers,
                       prob_mode, rng_key, stream, *out);
}

gs_status gs_random_walk(const gs_graph* g, const int32_t* starts, int64_t num_walkers,
                         int64_t walker_index_base, int length, float p, float q,
                         uint64_t rng_key, uint32_t flags, void* stream_, int32_t* traces) {
  if (!g || (!starts && num_walkers > 0) || (!traces && num_walkers > 0))
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_random_walk: null pointer");
  if (num_walkers < 0 || length < 0 || length >= (1 << 24) || walker_index_base < 0)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_random_walk: bad num_walkers/length/base");
  if (!(p > 0.0f) || !(q > 0.0f)) return fail(GS_ERR_INVALID_ARGUMENT, "gs_random_walk: p, q must be > 0");
  const bool n2v = (flags & GS_WALK_FORCE_NODE2VEC) || p != 1.0f || q != 1.0f;
  if (n2v && !g->sorted)
    return fail(GS_ERR_UNSORTED_GRAPH, "gs_random_walk: Node2Vec needs ascending CSC columns");
  return launch_walk(g, starts, num_walkers, walker_index_base, length, p, q, rng_key, n2v,
                     (flags & GS_WALK_PLAIN_CSC) != 0, (cudaStream_t)stream_, traces);
}

gs_status gs_walk_check(const gs_graph* g, void* stream_) {
  if (!g) return fail(GS_ERR_INVALID_ARGUMENT, "gs_walk_check: null graph");
  cudaStream_t stream = (cudaStream_t)stream_;
  int h = 0;
  GS_CUDA_TRY(cudaMemcpyAsync(&h, g->d_err, 4, cudaMemcpyDeviceToHost, stream));
  GS_CUDA_TRY(cudaStreamSynchronize(stream));
  GS_CUDA_TRY(cudaMemsetAsync(g->d_err, 0, 4, stream));
  if (h & ERR_SEED_RANGE) return fail(GS_ERR_INDEX_OUT_OF_RANGE, "a start node is outside [0, N)");
  return GS_OK;
}

gs_status gs_blocks_sync(gs_blocks* b) {
  if (!b) return fail(GS_ERR_INVALID_ARGUMENT, "gs_blocks_sync: null");
  GS_CUDA_TRY(cudaStreamSynchronize(b->stream));
  const int L = b->num_layers;
  b->h_meta.assign((size_t)b->num_batches * L * GS_META_FIELDS, 0);
  if (b->num_batches > 0)
    GS_CUDA_TRY(cudaMemcpy(b->h_meta.data(), b->b_meta.ptr, b->h_meta.size() * 8,
                           cudaMemcpyDeviceToHost));
  int err[4] = {0};
  unsigned long long ctr[MAX_LAYERS + 2] = {0};
  GS_CUDA_TRY(cudaMemcpy(err, b->b_err.ptr, 16, cudaMemcpyDeviceToHost));
  GS_CUDA_TRY(cudaMemcpy(ctr, b->b_ctr.ptr, std::min<size_t>(sizeof(ctr), b->b_ctr.bytes),
                         cudaMemcpyDeviceToHost));
  // views only of a result whose every block is complete (out-of-range seeds
  // leave valid, empty columns; an overflowed or inconsistent block does not)
  b->synced = (err[0] & (ERR_CAPACITY | ERR_INTERNAL)) == 0;
  if (err[0] & ERR_INTERNAL) return fail(GS_ERR_CUDA, "internal consistency check failed in a sampling kernel");
  if (err[0] & ERR_SEED_RANGE) return fail(GS_ERR_INDEX_OUT_OF_RANGE, "a seed id is outside [0, N)");
  if (err[0] & ERR_CAPACITY) {
    if (b->kind == gs_blocks::SHADOW) {
      b->sh_edge_hint = (int64_t)(ctr[0] + ctr[0] / 4 + 1024);
    } else {
      for (int l = 0; l < b->num_layers; ++l)
        b->lw_edge_hint[l] = std::max<int64_t>(b->lw_edge_hint[l], (int64_t)(ctr[l] + ctr[l] / 4 + 1024));
      b->lw_tab_hint = std::max<int64_t>(b->lw_tab_hint, (int64_t)ctr[MAX_LAYERS]);
      if (ctr[MAX_LAYERS + 1]) b->lw_big = true;  // re-run on the global-table kernel
    }
    return fail(GS_ERR_CAPACITY,
                "a device-side capacity was exceeded; call again with this gs_blocks (it has grown)");
  }
  return GS_OK;
}

gs_status gs_blocks_shape(const gs_blocks* b, int64_t* num_batches, int* num_layers) {
  if (!b) return fail(GS_ERR_INVALID_ARGUMENT, "gs_blocks_shape: null");
  if (num_batches) *num_batches = b->num_batches;
  if (num_layers) *num_layers = b->num_layers;
  return GS_OK;
}

gs_status gs_blocks_view(const gs_blocks* b, int64_t batch, int layer, gs_block_view* out) {
  if (!b || !out) return fail(GS_ERR_INVALID_ARGUMENT, "gs_blocks_view: null");
  if (!b->synced) return fail(GS_ERR_INVALID_ARGUMENT, "gs_blocks_view: call gs_blocks_sync first");
  if (batch < 0 || batch >= b->num_batches || layer < 0 || layer >= b->num_layers)
    return fail(GS_ERR_INVALID_ARGUMENT, "gs_blocks_view: batch/layer out of range");
  const int64_t* m = b->h_meta.data() + (batch * b->num_layers + layer) * GS_META_FIELDS;
  const gs_layer_buffers& lb = b->layers[layer];
  out->n_cols = m[0];
  out->n_rows = m[1];
  out->n_edges = m[2];
  out->col_map = lb.col_map + m[3];
  out->row_map = lb.row_map + m[4];
  out->indptr = lb.indptr + m[5];
  out->row_local = lb.row_local + m[6];
  out->eid = lb.eid + m[6];
  out->val = lb.val ? lb.val + m[6] : nullptr;
  out->row_prob = lb.row_prob ? lb.row_prob + m[4] : nullptr;
  return GS_OK;
}

gs_status gs_blocks_device_meta(const gs_blocks* b, const int64_t** meta) {
  if (!b || !meta) return fail(GS_ERR_INVALID_ARGUMENT, "gs_blocks_device_meta: null");
  *meta = (const int64_t*)b->b_meta.ptr;
  return GS_OK;
}

gs_status gs_blocks_layer(const gs_blocks* b, int layer, gs_layer_buffers* out) {
  if (!b || !out) return fail(GS_ERR_INVALID_ARGUMENT, "gs_blocks_layer: null");
  if (layer < 0 || layer >= b->num_layers) return fail(GS_ERR_INVALID_ARGUMENT, "gs_blocks_layer: bad layer");
  *out = b->layers[layer];
  return GS_OK;
}

void gs_blocks_destroy(gs_blocks* b) {
  if (!b) return;
  if (b->aux) gs_blocks_destroy(b->aux);
  if (b->side) {
    cudaStreamSynchronize(b->side);
    cudaStreamDestroy(b->side);
  }
  if (b->ev_fork) cudaEventDestroy(b->ev_fork);
  if (b->ev_join) cudaEventDestroy(b->ev_join);
  cudaStream_t s = b->stream;
  for (int l = 0; l < MAX_LAYERS; ++l) {
    b->b_col[l].reset(b->al, s);
    b->b_row[l].reset(b->al, s);
    b->b_indptr[l].reset(b->al, s);
    b->b_rowl[l].reset(b->al, s);
    b->b_eid[l].reset(b->al, s);
    b->b_val[l].reset(b->al, s);
    b->b_rprob[l].reset(b->al, s);
  }
  b->b_meta.reset(b->al, s);
  b->b_err.reset(b->al, s);
  b->b_ws.reset(b->al, s);
  b->b_gen.reset(b->al, s);
  b->b_ctr.reset(b->al, s);
  b->b_sched.reset(b->al, s);
  b->b_pack.reset(b->al, s);
  b->b_trace.reset(b->al, s);
  delete b;
}

}  // extern "C"
