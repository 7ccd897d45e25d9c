// gs_internal.h -- host/device shared structures of libgsb200 (not part of the ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/gs.h"

namespace gsb {

constexpr int MAX_LAYERS = 8;
constexpr int MAX_FANOUT = 32;
constexpr int64_t MAX_SLOTS_PER_BATCH = (1ll << 25);  // table value field (R3 positions)

// ---- kernel launches enqueued by this thread (gs_kernel_launches) ----
extern thread_local int64_t g_launches;
extern bool g_profiling;  // gs_set_profiling
inline void count_launch(int n = 1) { g_launches += n; }

// ---- error reporting (thread-local message) ----
void set_error(const char* fmt, ...);
gs_status fail(gs_status st, const char* fmt, ...);
gs_status cuda_fail(cudaError_t e, const char* what);
#define GS_CUDA_TRY(expr)                                   \
  do {                                                      \
    cudaError_t _e = (expr);                                \
    if (_e != cudaSuccess) return ::gsb::cuda_fail(_e, #expr); \
  } while (0)

// ---- allocator hook ----
struct Allocator {
  gs_alloc_fn alloc = nullptr;
  gs_free_fn free_fn = nullptr;
  void* ctx = nullptr;
  void* allocate(size_t bytes, cudaStream_t s) const;
  void release(void* p, size_t bytes, cudaStream_t s) const;
};
Allocator current_allocator();

// A growable device buffer owned through an Allocator.
struct DevBuf {
  void* ptr = nullptr;
  size_t bytes = 0;
  // Ensures capacity >= need; returns false on allocation failure.
  bool ensure(const Allocator& al, size_t need, cudaStream_t s, bool zero = false);
  void reset(const Allocator& al, cudaStream_t s);
};

// Device error word bits (set by kernels, read by gs_blocks_sync).
enum : int { ERR_SEED_RANGE = 1, ERR_CAPACITY = 2, ERR_INTERNAL = 4 };

}  // namespace gsb

struct gs_graph {
  int64_t num_nodes = 0, num_edges = 0;
  int64_t* indptr = nullptr;
  int32_t* indices = nullptr;
  float* weights = nullptr;
  float* colsum = nullptr;   // weighted graphs: fp32(sum_fp64 w) per column (a0 pre-processing)
  int32_t* poscnt = nullptr; // weighted graphs: #{w > 0} per column (a0; the A-Res sample count)
  bool owns = false;
  int sorted = 0;
  int64_t max_in_degree = 0;
  gsb::Allocator al;
  gsb::DevBuf b_indptr, b_indices, b_weights, b_colsum, b_poscnt, b_err, b_deg, b_degsrc;
  int32_t* deg = nullptr;    // FastGCN a0 pre-processing: in-degree per node (built on first use)
  int32_t* degsrc = nullptr; // FastGCN a0: in-degree of every CSC entry's row (deg[indices[e]]), if it fits
  gsb::DevBuf b_walk;        // walk index (walk.cu): 16 B per CSC entry, built on the first walk
  const int4* walk_rec = nullptr;
  bool walk_index_failed = false;
  int* d_err = nullptr;  // walk error word
  bool host_mapped = false;  // indices (+ weights) read from pinned host memory (UVA)
  void* host_reg[2] = {nullptr, nullptr};  // ranges this graph registered (unregistered at destroy)
  // hot-page HBM cache of a host-mapped graph (gs_graph_cache_hot): ptab[page] =
  // slot of the page in cidx / cw, or -1; pages of 1 << cpsh entries
  gsb::DevBuf b_ptab, b_cidx, b_cw;
  int32_t* ptab = nullptr;
  int32_t* cidx = nullptr;
  float* cw = nullptr;
  int cpsh = 14;
  int64_t cached_pages = 0;
  int n_reg = 0;
};

struct gs_blocks {
  enum Kind { NODEWISE = 0, LAYERWISE = 1, SHADOW = 2 };
  gsb::Allocator al;
  cudaStream_t stream = nullptr;
  int kind = NODEWISE;
  int64_t num_batches = 0;
  int num_layers = 0;
  gs_layer_buffers layers[gsb::MAX_LAYERS] = {};
  // owned buffers per layer: col_map (layer 0 / layer-wise), row_map, indptr,
  // row_local, eid, val, row_prob
  gsb::DevBuf b_col[gsb::MAX_LAYERS], b_row[gsb::MAX_LAYERS], b_indptr[gsb::MAX_LAYERS],
      b_rowl[gsb::MAX_LAYERS], b_eid[gsb::MAX_LAYERS], b_val[gsb::MAX_LAYERS],
      b_rprob[gsb::MAX_LAYERS];
  gsb::DevBuf b_meta, b_err, b_ws, b_gen, b_ctr, b_sched, b_pack;
  gsb::DevBuf b_trace;         // GraphSAINT-RW: walk traces between the walk and the induce launch
  std::vector<int64_t> h_meta;
  int64_t sh_edge_hint = 0;    // ShaDow edge capacity learnt from an overflow
  int64_t ws_stride_prev = -1; // workspace layout of the previous launch
  unsigned int launch_id = 0;  // per-call tag for device-side flags
  int ws_kind_prev = 0;        // workspace layout tag of the previous launch (per kernel family)
  int64_t lw_edge_hint[gsb::MAX_LAYERS] = {};  // layer-wise edge capacity learnt from an overflow
  int64_t lw_tab_hint = 0;     // layer-wise per-CTA table size learnt from an overflow
  bool lw_big = false;         // a batch-layer outgrew the shared-memory layer-wise kernel
  bool synced = false;
  gs_blocks* aux = nullptr;    // ShaDow: the internal node-wise result
  int64_t num_seeds = 0, batch_size = 0;  // node-wise: the seeds and (fixed) batch size sampled
  int64_t graph_edges = 0;     // num_edges of the graph sampled (gs_blocks_pack_narrow's check)
  const int64_t* bptr_dev = nullptr;       // node-wise (hop engine): device seed offsets [nb + 1]
  cudaStream_t side = nullptr; // node-wise: second stream (groups of batches alternate), forked/joined by events
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  std::vector<std::pair<std::string, double>> prof;  // per-kernel ms of the last call (profiling on)
};
