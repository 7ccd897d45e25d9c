/*
 * gs.h -- C ABI of the B200-native gSampler ECSF sampling hot path.
 *
 * The library (libgsb200.so, sources in paper_conf_sosp_gonglmc0lwl23_b200/csrc)
 * runs every step of the path in hand-written sm_100a CUDA kernels:
 *   Extract  A[:, frontiers]                      PAPER.md Table 4
 *   Compute  row/column sums, broadcast divides    Table 4, Fig. 3(b)/(c)
 *   Select   individual_sample / collective_sample Table 4; walks P:75
 *   Finalize row()/column(), relabel, compaction   Table 4
 * ("P:n" = line n of the paper text /root/reference/PAPER.md.)
 * The paper fixes WHAT is sampled, not HOW; the readings (sampling algorithms,
 * Philox keying, output order) are listed in DESIGN.md "Readings" (R1..R25).
 *
 * Conventions (all entry points):
 *  - Plain pointers and sizes only.  "device" pointers must be CUDA device (or
 *    managed) memory of the current device; "host" pointers are CPU memory.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *    Calls are stream-ordered: they validate host-side arguments, enqueue
 *    kernels and return without synchronising unless stated otherwise.
 *  - Every call returns gs_status; on failure gs_last_error() (thread-local)
 *    holds a message.  No C++ exception crosses the ABI.
 *  - Node ids are int32 (N < 2^31); indptr and edge ids are int64.
 *  - Results depend only on (graph, seeds, batch_size, batch_index_base,
 *    rng_key, parameters): not on stream, device, launch geometry or the
 *    number of ranks sharing an epoch.
 */
#ifndef GS_H
#define GS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum gs_status {
  GS_OK = 0,
  GS_ERR_INVALID_ARGUMENT = 1,   /* bad pointer / size / mode (host-side check)   */
  GS_ERR_OUT_OF_MEMORY = 2,      /* allocation through the allocator hook failed  */
  GS_ERR_CUDA = 3,               /* a CUDA runtime call or kernel launch failed   */
  GS_ERR_UNSORTED_GRAPH = 4,     /* Node2Vec needs ascending CSC columns          */
  GS_ERR_INDEX_OUT_OF_RANGE = 5, /* a seed/start id outside [0, N) (device-detected) */
  GS_ERR_NOT_SUPPORTED = 6,      /* parameter outside the implemented envelope    */
  GS_ERR_CAPACITY = 7,           /* a device-side output capacity was exceeded    */
  GS_ERR_INVALID_GRAPH = 8       /* CSC validation failed in gs_graph_create      */
} gs_status;

const char* gs_last_error(void);
const char* gs_status_string(gs_status s);
/* Library version: major*10000 + minor*100 + patch. */
int gs_version(void);
/* Kernels this library has enqueued from the calling thread so far (a
 * cumulative counter: the difference around a call = its kernel launches). */
int64_t gs_kernel_launches(void);

/* Device-memory hook.  Every device buffer the library owns (graph copies,
 * blocks, workspaces) is obtained through alloc(bytes, stream, ctx) and
 * returned through free(ptr, bytes, stream, ctx).  Default (both NULL):
 * cudaMalloc / cudaFree.  The Python binding installs PyTorch's caching
 * allocator here, so PyTorch owns the device memory.  Not thread-safe: set it
 * before creating objects; objects remember the hook they were created with. */
typedef void* (*gs_alloc_fn)(size_t bytes, void* stream, void* ctx);
typedef void (*gs_free_fn)(void* ptr, size_t bytes, void* stream, void* ctx);
gs_status gs_set_allocator(gs_alloc_fn alloc, gs_free_fn free_fn, void* ctx);

/* ------------------------------------------------------------------------ */
/* Graph (a0): CSC adjacency, column v = in-neighbours of v.          */
/* ------------------------------------------------------------------------ */
typedef struct gs_graph gs_graph;

enum {
  GS_GRAPH_HOST_PTRS = 1, /* indptr/indices/weights are host pointers (copied to HBM)      */
  GS_GRAPH_BORROW = 2,    /* device pointers are used in place; caller keeps them alive    */
  GS_GRAPH_HOST_MAPPED = 4 /* with HOST_PTRS: indices / weights stay in host memory, pinned
                             and mapped (cudaHostRegister), read by every kernel over the
                             host link (UVA; graphs beyond 180 GB of HBM, SURVEY
                             8(f) f4); indptr is copied to HBM; the caller keeps the host
                             arrays alive until gs_graph_destroy                          */
};                        /* default (0): device pointers, copied into library-owned HBM  */

/* Validates the CSC on the device (indptr[0] == 0, monotone, indptr[N] ==
 * num_edges, 0 <= indices < N) and records whether every column is sorted
 * ascending (needed by Node2Vec).  Synchronises `stream` once (one-off).
 *   indptr  int64[num_nodes + 1], indices int32[num_edges],
 *   weights fp32[num_edges] or NULL (unweighted: w == 1).
 * Returns GS_ERR_INVALID_GRAPH if validation fails. */
gs_status gs_graph_create(const int64_t* indptr, const int32_t* indices, const float* weights,
                          int64_t num_nodes, int64_t num_edges, uint32_t flags, void* stream,
                          gs_graph** out);

typedef struct gs_graph_info {
  int64_t num_nodes, num_edges;
  int weighted;       /* weights present */
  int sorted;         /* every column ascending */
  int64_t max_in_degree;
  const int64_t* indptr;   /* device */
  const int32_t* indices;  /* device */
  const float* weights;    /* device or NULL */
  int host_mapped;         /* indices / weights are mapped host memory (GS_GRAPH_HOST_MAPPED) */
  int64_t cached_pages;    /* HBM cache of a host-mapped graph (gs_graph_cache_hot): pages held, */
  int64_t cache_page_entries; /* CSC entries per page                                           */
} gs_graph_info;
gs_status gs_graph_get_info(const gs_graph* g, gs_graph_info* out);
/* Replaces the edge weights (device float[num_edges]) and recomputes the a0
 * column sums; copied unless flags has GS_GRAPH_BORROW (then used in place and
 * kept alive by the caller).  Structure, validation and derived index arrays
 * are unchanged.  Used to sample over a computed bias (PASS att, R29). */
gs_status gs_graph_set_weights(gs_graph* g, const float* weights, uint32_t flags, void* stream);
/* Hot-column cache of a host-mapped graph (GS_GRAPH_HOST_MAPPED; P:490's
 * "caching hot data in GPU"): copies the hottest pages of the
 * index (and weight) array -- pages of 16,384 CSC entries, scored by the sum
 * over their entries of min(32, in-degree of the entry's column), i.e. the
 * expected node-wise accesses per entry when frontier nodes are drawn in
 * proportion to degree -- into HBM, at most budget_bytes of them; the
 * node-wise sampler then reads cached entries from HBM and the rest over the
 * host link.  Results are unchanged (tested).  A second call replaces the
 * cache; budget_bytes = 0 drops it.  GS_ERR_INVALID_ARGUMENT for a graph that
 * is not host-mapped.  Synchronises the stream (page scores come to the host). */
gs_status gs_graph_cache_hot(gs_graph* g, int64_t budget_bytes, void* stream);
void gs_graph_destroy(gs_graph* g);

/* ------------------------------------------------------------------------ */
/* Sample blocks: the result of the sampling calls.                           */
/* ------------------------------------------------------------------------ */
/* A gs_blocks object owns device buffers holding, for every (batch, layer),
 * one sampled sub-matrix of A ("block") over local ids plus its relabel
 * maps (A.column(), A.row()).  Seeds are cut into batches of
 * batch_size (the last may be shorter); batch b is independent of every other
 * (super-batch sampling with per-batch id spaces).
 *
 * Reuse: pass `*out == NULL` to create a new object, or a previous result to
 * reuse its buffers (grown through the allocator when too small; reuse with
 * unchanged shapes performs no allocation and is CUDA-graph capturable). */
typedef struct gs_blocks gs_blocks;

typedef struct gs_block_view {
  int64_t n_cols, n_rows, n_edges;
  const int32_t* col_map;   /* [n_cols]  local column -> global node (the frontier)      */
  const int32_t* row_map;   /* [n_rows]  local row -> global node; next layer's frontier */
  const int64_t* indptr;    /* [n_cols+1] CSC over local ids, indptr[0] == 0             */
  const int32_t* row_local; /* [n_edges] local row of each edge                           */
  const int64_t* eid;       /* [n_edges] global edge id (position in indices)            */
  const float* val;         /* [n_edges] or NULL: LADIES/FastGCN edge value, PASS prob   */
  const float* row_prob;    /* [n_rows] or NULL: layer-wise p(u) = b(u)/B                */
} gs_block_view;            /* all pointers are DEVICE pointers into the gs_blocks object */

/* Waits for the stream the blocks were produced on, copies the per-(batch,
 * layer) counts to the host and reports device-detected errors
 * (GS_ERR_INDEX_OUT_OF_RANGE, GS_ERR_CAPACITY). */
gs_status gs_blocks_sync(gs_blocks* b);
gs_status gs_blocks_shape(const gs_blocks* b, int64_t* num_batches, int* num_layers);
/* Device pointers of one block; requires a prior gs_blocks_sync. */
gs_status gs_blocks_view(const gs_blocks* b, int64_t batch, int layer, gs_block_view* out);
/* Sync-free access: device int64 [num_batches][num_layers][GS_META_FIELDS]:
 * (n_cols, n_rows, n_edges, col_offset, row_offset, indptr_offset,
 * edge_offset, 0) -- the offsets locate the block inside the layer-wide
 * arrays of gs_blocks_layer. */
enum { GS_META_FIELDS = 8 };
gs_status gs_blocks_device_meta(const gs_blocks* b, const int64_t** meta);

typedef struct gs_layer_buffers {   /* whole-layer device arrays of one layer */
  int32_t* col_map;   int64_t col_capacity;
  int32_t* row_map;   int64_t row_capacity;
  int64_t* indptr;    int64_t indptr_capacity;
  int32_t* row_local; int64_t* eid; float* val; int64_t edge_capacity; /* val may be NULL */
  float* row_prob;    /* [row_capacity] or NULL */
} gs_layer_buffers;
gs_status gs_blocks_layer(const gs_blocks* b, int layer, gs_layer_buffers* out);

/* Packs layer `layer` of every batch into dense, batch-ordered DEVICE arrays
 * (caller-owned, each at least the layer's capacity from gs_blocks_layer):
 * batch b's edges (row_local, eid), its block indptr (n_cols + 1 entries,
 * block-relative: starts at 0) and its row_map follow those of batch b - 1.
 * totals: DEVICE int64[3] <- (edges, indptr entries, rows) of the layer.
 * Stream-ordered, no host sync: the sampling kernels write every batch into a
 * fixed padded region; this lets a host copy move only
 * the sampled data (read `totals` first).  Errors: GS_ERR_INVALID_ARGUMENT
 * (null pointer, bad layer), GS_ERR_OUT_OF_MEMORY, GS_ERR_CUDA. */
gs_status gs_blocks_pack(const gs_blocks* b, int layer, int32_t* row_local, int64_t* eid,
                         int64_t* indptr, int32_t* row_map, int64_t* totals, void* stream);
/* As gs_blocks_pack with 32-bit edge ids and block-relative 32-bit indptr
 * entries (a smaller host copy): the sampled graph must have fewer than 2^31
 * entries (else GS_ERR_NOT_SUPPORTED, host-side); block indptr values are
 * always < 2^25.  Buffers are int32 arrays of the same capacities. */
gs_status gs_blocks_pack_narrow(const gs_blocks* b, int layer, int32_t* row_local, int32_t* eid,
                                int32_t* indptr, int32_t* row_map, int64_t* totals, void* stream);
void gs_blocks_destroy(gs_blocks* b);
/* Profiling (diagnostic, off by default): while on, the node-wise sampler
 * records a CUDA event after each of its kernels, runs them on one stream and
 * synchronises at the end of the call; gs_blocks_profile(b, i, &name, &ms)
 * then returns the i-th (kernel, milliseconds) pair of that call
 * (GS_ERR_INVALID_ARGUMENT past the last).  name stays valid until the next
 * call on b. */
gs_status gs_set_profiling(int on);
gs_status gs_blocks_profile(const gs_blocks* b, int i, const char** name, double* ms);

/* ------------------------------------------------------------------------ */
/* Node-wise sampling (a1 + a3 + a6; + a2 for PASS-style).                    */
/* ------------------------------------------------------------------------ */
enum {
  GS_W_UNIFORM = 0,      /* GraphSAGE: uniform without replacement (Floyd, R5)            */
  GS_W_EDGE = 1,         /* weighted without replacement, A-Res keys on w_e (R6)          */
  GS_W_PASS_COLNORM = 2  /* as EDGE, plus val_e = w_e / sum(w over column v): PASS A3 (R11) */
};
/* individual_sample, layer by layer:
 *   seeds   device int32[num_seeds], 0 <= id < N (violations are reported by
 *           gs_blocks_sync as GS_ERR_INDEX_OUT_OF_RANGE; such columns are empty)
 *   batch_size > 0; batch b holds seeds [b*batch_size, min(num_seeds, (b+1)*batch_size))
 *   batch_index_base: global index of batch 0 (keys the RNG; shard invariance)
 *   fanouts host int32[num_layers], 1 <= fanouts[l] <= 32, fanouts[0] applies to
 *           the seeds (R15); 1 <= num_layers <= 8
 *   replace 0: without replacement (GraphSAGE); 1: with replacement (KGCN, R10,
 *           bias_mode must be GS_W_UNIFORM)
 *   rng_key Philox key; counters (v, slot, layer|tag<<24, global batch) (R4)
 * Output per (b, l): col_map = frontier (l = 0: the batch's seeds; l > 0: the
 * previous layer's row_map, R2), edges in column order then ascending position
 * (slot order with replacement), row_map = the block's distinct rows ascending (R3).
 * Envelope: batch_size * prod(fanouts[0..l]) <= 2^25 for every l. */
gs_status gs_sample_neighbors(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                              int64_t batch_size, int64_t batch_index_base,
                              const int32_t* fanouts, int num_layers, int replace, int bias_mode,
                              uint64_t rng_key, void* stream, gs_blocks** out);

/* Ragged mini-batches (super-batch with per-batch ID spaces):
 * as gs_sample_neighbors, but batch b holds seeds [batch_ptr[b],
 * batch_ptr[b+1]) for any non-decreasing HOST int64[num_batches + 1] with
 * batch_ptr[0] == 0 and batch_ptr[num_batches] == num_seeds (empty batches
 * allowed; copied, the caller may free it on return).  Batch b's blocks live
 * in the fixed regions starting at batch_ptr[b].
 * Envelope: max batch size * prod(fanouts) <= 2^25.  Errors as
 * gs_sample_neighbors, plus GS_ERR_INVALID_ARGUMENT for a malformed batch_ptr. */
gs_status gs_sample_neighbors_ragged(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                                     const int64_t* batch_ptr, int64_t num_batches, int64_t batch_index_base,
                                     const int32_t* fanouts, int num_layers, int replace, int bias_mode,
                                     uint64_t rng_key, void* stream, gs_blocks** out);

/* Induce ("induce a subgraph using all the sampled nodes", P:113;
 * R12) over an existing node-wise result `sampled` (from gs_sample_neighbors
 * or gs_sample_neighbors_ragged, same stream order): for every batch, U = its
 * seeds and the rows of every layer, ascending; one block per batch
 * (num_layers == 1 in *out): col_map == row_map == U, the edges u->v of A with
 * u, v in U in CSC order.  *out (NULL or a previous result, != sampled) is
 * library-owned.  Edge overflow -> GS_ERR_CAPACITY at gs_blocks_sync (the
 * object has grown: call again).  Envelope: N within the cluster shared-
 * memory bitmap (GS_ERR_NOT_SUPPORTED otherwise). */
gs_status gs_induce_subgraph(const gs_graph* g, const gs_blocks* sampled, void* stream, gs_blocks** out);

/* ShaDow (R12): node-wise sampling as gs_sample_neighbors
 * (bias_mode UNIFORM or EDGE, no replacement), then for every batch the
 * subgraph of A induced on U = the union of the seeds and all sampled rows,
 * ascending (R12).  One block per batch (num_layers == 1 in the result):
 * col_map == row_map == U, edges u->v with u, v in U in CSC order. */
gs_status gs_sample_shadow(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                           int64_t batch_size, int64_t batch_index_base, const int32_t* fanouts,
                           int num_layers, int bias_mode, uint64_t rng_key, void* stream,
                           gs_blocks** out);

/* GraphSAINT-RW (Table 2: "conduct vanilla random walk and induce
 * subgraph according to sampled nodes"; DESIGN R26).
 *   roots       device int32[num_roots], cut into batches of batch_size (the
 *               last may be shorter); root i walks walk_length DeepWalk steps
 *               (R13) keyed by the global walker index
 *               batch_index_base * batch_size + i (Philox tag 5, R4)
 *   walk_length >= 0; batch_size * (walk_length + 1) <= 2^25 and the global
 *               walker ids must fit 32 bits (else GS_ERR_NOT_SUPPORTED)
 * Output: one block per batch (num_layers == 1), exactly as gs_sample_shadow:
 * col_map == row_map == U = the distinct nodes the batch's walks visited,
 * ascending; edges u->v of A with u, v in U in CSC order.  Roots outside
 * [0, N) are reported by gs_blocks_sync (GS_ERR_INDEX_OUT_OF_RANGE); edge
 * overflow as GS_ERR_CAPACITY (the object has grown: call again).
 * Two launches: the walk kernel (traces kept in the result object) and the
 * cluster induce kernel. */
gs_status gs_sample_saint_rw(const gs_graph* g, const int32_t* roots, int64_t num_roots,
                             int64_t batch_size, int64_t batch_index_base, int walk_length,
                             uint64_t rng_key, void* stream, gs_blocks** out);

/* PinSAGE-style (Table 2: "random walks ... using restarts, select
 * top-k visited neighbors as sampled nodes"; DESIGN R27).
 * Per (batch b, layer l) and frontier column v: num_walks walks from v of at
 * most walk_length steps; before step t of walk w, r = philox(v,
 * w*walk_length + t-1, l | 7<<24, batch_index_base + b): the walk ends if
 * fp32((r2>>8) 2^-24) < restart_prob (the next walk restarts at v) or at a
 * node with no in-neighbours, else it moves to in-neighbour draw_below(d).
 * Every visit of a node x != v counts; v's neighbours are its topk[l] most
 * visited nodes (count descending, id ascending), in that order.
 *   seeds       device int32[num_seeds], batches of batch_size (last ragged)
 *   topk        host int32[num_layers], 1..32; 1 <= num_layers <= 8
 *   num_walks, walk_length >= 1, num_walks * walk_length <= 2048
 *   restart_prob in [0, 1]
 * Output per (b, l) like gs_sample_neighbors: col_map = frontier (l = 0 the
 * seeds, else the previous layer's row_map, R2), row_map = the selected nodes
 * ascending (R3), CSC over local ids with each column in rank order,
 * val = fp32(visit count), eid = -1 (these are not edges of A).
 * Envelope: batch_size * prod(topk[0..l]) <= 2^25.  Seeds outside [0, N) are
 * reported by gs_blocks_sync; their columns are empty.  One kernel launch. */
gs_status gs_sample_pinsage(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                            int64_t batch_size, int64_t batch_index_base, const int32_t* topk,
                            int num_layers, int num_walks, int walk_length, float restart_prob,
                            uint64_t rng_key, void* stream, gs_blocks** out);

/* ------------------------------------------------------------------------ */
/* Matrix-centric operators (Table 4).            */
/* A gs_matrix is a materialised sub-matrix of A over GLOBAL node ids:        */
/* local columns `cols` with a CSC indptr, and per entry its global row id,   */
/* its edge id (position in the graph's indices) and an fp32 value (the edge  */
/* weight, 1 if unweighted).  Device-resident, library-owned (allocator hook), */
/* freed by gs_matrix_destroy.  These are the unfused operators a new         */
/* algorithm composes; the samplers above fuse them.              */
/* Calls that size an output (slice_columns, slice_rows, row_ids) synchronise */
/* the stream once; the others only enqueue.  Node ids outside [0, N) ->      */
/* GS_ERR_INDEX_OUT_OF_RANGE.                                                 */
/* ------------------------------------------------------------------------ */
typedef struct gs_matrix gs_matrix;
typedef struct gs_matrix_view {
  int64_t num_nodes, n_cols, nnz;
  const int32_t* cols;    /* [n_cols]   global id of each local column        */
  const int64_t* indptr;  /* [n_cols+1] CSC over the local columns            */
  const int32_t* row;     /* [nnz]      global row id of each entry           */
  const int64_t* eid;     /* [nnz]      edge id of each entry                 */
  float* val;             /* [nnz]      entry value (mutable in place)        */
} gs_matrix_view;
enum { GS_OP_ADD = 0, GS_OP_SUB = 1, GS_OP_MUL = 2, GS_OP_DIV = 3, GS_OP_POW = 4 };
/* A[:, cols] (Extract): cols device int32[n_cols] (duplicates allowed);
 * each column's entries in the graph's CSC order.  *out may be NULL (a new
 * object) or a previous result (reused). */
gs_status gs_matrix_slice_columns(const gs_graph* g, const int32_t* cols, int64_t n_cols, void* stream,
                                  gs_matrix** out);
/* A[rows, :] (Extract): the entries whose row is in rows (device
 * int32[n_rows]); same columns; *out must differ from in. */
gs_status gs_matrix_slice_rows(const gs_matrix* in, const int32_t* rows, int64_t n_rows, void* stream,
                               gs_matrix** out);
/* A.sum(axis) (Compute; R1): axis 0 -> out device float[n_cols], the
 * per-column sums; axis 1 -> out device float[num_nodes], the per-row sums by
 * global row id (0 for rows without entries).  fp64 accumulation, one fp32
 * rounding (R19). */
gs_status gs_matrix_sum(const gs_matrix* m, int axis, float* out, void* stream);
/* A.<op>(V, axis) in place (Compute): val = val op V[c] (axis 0,
 * V device float[n_cols]) or val op V[row] (axis 1, V device float[num_nodes]).
 * op: GS_OP_ADD/SUB/MUL/DIV/POW (IEEE fp32; POW = fp32(pow_fp64)). */
gs_status gs_matrix_broadcast(gs_matrix* m, int op, const float* V, int axis, void* stream);
/* A <op> v in place (Compute), e.g. A ** 2 (LADIES, Fig. 2). */
gs_status gs_matrix_elementwise(gs_matrix* m, int op, float v, void* stream);
/* A.row() (Finalize; R3): distinct row ids ascending into out (device
 * int32, capacity >= min(nnz, num_nodes)); *n_out (host) = their number. */
gs_status gs_matrix_row_ids(const gs_matrix* m, int32_t* out, int64_t* n_out, void* stream);
/* A.individual_sample(K, probs) (Select): every column
 * (frontier) samples K of its entries independently; returns the sub-matrix
 * of the kept entries (ascending position; slot order with replacement).
 * use_values 0: uniform -- without replacement Floyd (R5, all of a column with
 * <= K entries), replace 1: K i.i.d. draws (R10); use_values 1: weighted
 * without replacement on the matrix's values (A-Res, R6; values <= 0
 * ineligible).  RNG: the samplers' keying (R4) with the column node, the
 * entry's position in the column, `layer` and `batch_index` -- on A[:, F] the
 * result is exactly that layer of gs_sample_neighbors (Extract-Select fusion,
 * P:289).  1 <= K <= 32.  Synchronises the stream once (output size). */
gs_status gs_matrix_individual_sample(const gs_matrix* in, int K, int use_values, int replace, uint64_t rng_key,
                                      int layer, int64_t batch_index, void* stream, gs_matrix** out);
/* A.collective_sample(K, node_probs) (Select): K of the
 * matrix's row nodes by the bias node_probs (device float[num_nodes], indexed
 * by global id, unnormalised) or, node_probs NULL, the rows' entry counts;
 * b <= 0 ineligible; every eligible row when at most K (R24), else the K
 * smallest A-Res keys (R6, layer-wise keying R4; ties -> smaller id); returns
 * the sub-matrix of the entries whose row was selected (CSC order; its
 * gs_matrix_row_ids = S ascending).  With node_probs = (A[:,F] ** 2).sum(1)
 * it is one layer of gs_sample_layerwise(LADIES).  K <= 2048.  Synchronises. */
gs_status gs_matrix_collective_sample(const gs_matrix* in, int K, const float* node_probs, uint64_t rng_key,
                                      int layer, int64_t batch_index, void* stream, gs_matrix** out);
/* Fused Edge-Map chain (+ Edge-Reduce): the element-wise
 * operators (ops[i], scalars[i]), i < n_ops <= 8, applied in order to every
 * entry value -- identical to n_ops gs_matrix_elementwise calls -- in one
 * pass; axis -1: written back in place (Edge-Map fusion); axis 0 / 1: not
 * written, summed per column / per global row into out (float[n_cols] /
 * float[num_nodes], fp64 accumulation, Edge-MapReduce fusion). */
gs_status gs_matrix_map_reduce(gs_matrix* m, const int* ops, const float* scalars, int n_ops, int axis, float* out,
                               void* stream);
/* AS-GCN-style learned layer-wise bias (Table 2; R30): out[u] =
 * fp32(s(u) * relu(fp32(sum_f X[u][f] wg[f]))) with s = A.sum(axis=1) (fp64
 * accumulation), X device bf16 [num_nodes][F] row-major, wg device float[F]
 * (the trainable projection); 0 for nodes that are not rows of m.  The
 * node_probs of gs_matrix_collective_sample. */
gs_status gs_matrix_asgcn_bias(const gs_matrix* m, const void* X, int F, const float* wg, float* out, void* stream);
gs_status gs_matrix_get_view(const gs_matrix* m, gs_matrix_view* out);
void      gs_matrix_destroy(gs_matrix* m);

/* ------------------------------------------------------------------------ */
/* Heterogeneous graphs ("each type of edges is modeled as a sparse    */
/* matrix to conduct the same sampling workflow as homogeneous graphs";      */
/* SURVEY 8(f) f4).                                                           */
/* ------------------------------------------------------------------------ */
typedef struct gs_hetero gs_hetero;
/* One mini-batch of node-wise (GraphSAGE, R5) sampling over num_relations
 * edge types.  Relation r: graphs[r] is the CSC matrix of that edge type --
 * column v = the in-neighbours of destination node v of type dst_type[r], row
 * ids = source nodes of type src_type[r], both in per-type local ids; it has
 * max(num_nodes[src], num_nodes[dst]) columns (columns past the destination
 * type's count empty).  seeds[t] (device int32[num_seeds[t]], NULL when 0) are
 * the layer-0 frontier of node type t.  Layer l, relation r: every frontier
 * node of type dst_type[r] samples fanouts[l * num_relations + r] (0..32; 0
 * skips the relation at that layer) of its in-neighbours in graphs[r] --
 * A_r[:, F].individual_sample(k), so the RNG keying is the homogeneous one
 * (R4, layer l, batch 0) under the key rng_key XOR (r + 1) * 0x9E3779B97F4A7C15
 * (R33); the frontier of type t at layer l + 1 is the union of the sampled
 * rows of every relation with src_type == t, ascending (A.row()).
 * Results: gs_hetero_block (layer, relation) -> the sampled sub-matrix (global
 * per-type ids, COO + CSC over the frontier; NULL when skipped), borrowed
 * from the gs_hetero; gs_hetero_frontier (layer 0..num_layers, type) -> device
 * ids + count.  Synchronises the stream (sizes).  Errors: GS_ERR_INVALID_ARGUMENT
 * (counts, types, fanouts, a graph with too few columns), GS_ERR_INDEX_OUT_OF_RANGE
 * (a seed or row id outside its type). */
gs_status gs_sample_neighbors_hetero(const gs_graph* const* graphs, const int32_t* src_type,
                                     const int32_t* dst_type, int num_relations, int num_node_types,
                                     const int64_t* num_nodes, const int32_t* const* seeds,
                                     const int64_t* num_seeds, const int32_t* fanouts, int num_layers,
                                     uint64_t rng_key, void* stream, gs_hetero** out);
gs_status gs_hetero_block(const gs_hetero* h, int layer, int relation, const gs_matrix** out);
gs_status gs_hetero_frontier(const gs_hetero* h, int layer, int node_type, const int32_t** ids, int64_t* n);
void      gs_hetero_destroy(gs_hetero* h);

/* PASS learned bias in full (Fig. 3(c) lines 3-9; DESIGN R29; SURVEY
 * 8(f) f2).  att[e] for every edge e = (u -> v) of g (weight w_e, 1 if unweighted):
 *   A1 = w_e <X_u W1, X_v W1>, A2 = w_e <X_u W2, X_v W2>, A3 = fp32(w_e / colsum_v),
 *   att = fp32(relu((s0 A1 + s1 A2) + s2 A3)), s = softmax(W3) (fp64).
 *   X   device bf16 [num_nodes][F] row-major (node features)
 *   W1, W2 device bf16 [F][H] row-major, H in {8, 16, 32, 64}
 *   W3  host float[3] (mixing logits)
 *   att device float[num_edges] (caller-owned), CSC order
 * The projections X [W1 | W2] are one dense bf16 GEMM on the tensor cores
 * (cuBLAS, fp32 accumulate); the SDDMM + mix is a hand-written kernel.  Exact
 * (order-independent) for the grid-valued inputs of R29.  Line 10
 * (individual_sample(k, att)) = gs_graph_set_weights(att) + gs_sample_neighbors
 * with GS_W_EDGE.  Stream-ordered; workspace through the allocator hook. */
gs_status gs_pass_attention(const gs_graph* g, const void* X, int F, const void* W1, const void* W2,
                            int H, const float* W3, void* stream, float* att);

/* ------------------------------------------------------------------------ */
/* Layer-wise sampling (a1 + a2 + a4 + a6): FastGCN / LADIES.                 */
/* ------------------------------------------------------------------------ */
enum {
  GS_PROB_LADIES = 0, /* b(u) = sum over extracted edges of w^2 (Fig. 2)  */
  GS_PROB_DEGREE = 1, /* b(u) = in-degree of u (FastGCN)                       */
  GS_PROB_COUNT = 2   /* b(u) = number of extracted edges of u (node_probs omitted)  */
};
/* collective_sample: per (batch, layer) with frontier F, C =
 * unique rows of A[:, F]; S = all u in C with b(u) > 0 if at most K of them,
 * else the K smallest A-Res keys (R6/R7); S ascending; block = edges of
 * A[:, F] whose row is in S (CSC order); row_prob p(u) = b(u)/B with
 * B = sum of b over C; val_e = a_e / sum_column(a), a_e = w_e / p(u)
 * (Fig. 3(b) lines 5-7).  Next frontier = S.
 *   n_per_layer host int32[num_layers], 1 <= K <= 4096. */
gs_status gs_sample_layerwise(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                              int64_t batch_size, int64_t batch_index_base,
                              const int32_t* n_per_layer, int num_layers, int prob_mode,
                              uint64_t rng_key, void* stream, gs_blocks** out);

/* ------------------------------------------------------------------------ */
/* Random walks (a5): DeepWalk / Node2Vec.                                   */
/* ------------------------------------------------------------------------ */
enum { GS_WALK_FORCE_NODE2VEC = 1,  /* use the Node2Vec sampler even at p == q == 1 */
       GS_WALK_PLAIN_CSC = 2 };     /* walk the plain CSC: do not build / use the walk index */
/* One walker per start node.  traces: caller-owned device
 * int32 [num_walkers][length + 1]; traces[i][0] = starts[i]; a walker at a
 * node with no in-neighbours stops and the rest of its row is -1 (R13).
 * p == q == 1 (and no FORCE flag): DeepWalk, uniform in-neighbour per step.
 * Otherwise Node2Vec with bias 1/p (x == prev), 1 (x in column(prev)), 1/q
 * (else), by rejection sampling (R14); needs a sorted graph
 * (GS_ERR_UNSORTED_GRAPH otherwise).  walker_index_base keys the RNG by the
 * global walker index (R4).  p, q > 0; 0 <= length < 2^24.
 * The first walk on a graph builds a walk index (16 bytes per CSC entry: each
 * position's neighbour with that neighbour's column range, a0 pre-processing)
 * when memory allows, so that a step is one dependent random read instead of
 * two; results are identical either way (GS_WALK_PLAIN_CSC disables it). */
gs_status gs_random_walk(const gs_graph* g, const int32_t* starts, int64_t num_walkers,
                         int64_t walker_index_base, int length, float p, float q,
                         uint64_t rng_key, uint32_t flags, void* stream, int32_t* traces);
/* Device-detected errors of the last gs_random_walk on this thread's graph
 * (out-of-range starts); synchronises the stream. */
gs_status gs_walk_check(const gs_graph* g, void* stream);

#ifdef __cplusplus
}
#endif
#endif /* GS_H */
