/*
 * gso.h -- CPU ORACLE for the gSampler ECSF sampling hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_sosp_gonglmc0lwl23_b200/, include/gs.h) never
 * links, imports or calls anything in oracle/; the two share no code.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, "P:n" = line n):
 *   - Extract  A[:, frontiers]          Table 4
 *   - Compute  row sums / column sums / broadcast divides  Table 4,
 *              LADIES Fig. 3(b), PASS A3
 *   - Select   individual_sample (node-wise),
 *              collective_sample (layer-wise),
 *              random walks (DeepWalk P:75, Node2Vec P:82)
 *   - Finalize row()/column() + relabel/compaction,
 *              ShaDow induced subgraph,
 *              GraphSAINT-RW walk + induce,
 *              PinSAGE-style restart walks + top-k visited
 * The paper does not fix the sampling algorithms, the RNG or the output order;
 * the readings used here are DESIGN.md section "Readings" (R1..R25), which
 * follow SURVEY.md section 8(c).  Every random draw is Philox4x32-10 keyed by
 * (rng_key; subject, slot, layer|tag<<24, global batch index).
 *
 * Arithmetic: IEEE fp32/fp64 round-to-nearest, built with -ffp-contract=off and
 * without -ffast-math.  Sums are accumulated in fp64 and rounded once to fp32.
 *
 * Parity status: every function below is pinned by tests/test_oracle_*.py
 * (KAT vectors, exact laws by enumeration + chi-square, the paper's worked
 * LADIES example B_f = 0.58, closed forms, brute force).
 */
#ifndef GSO_H
#define GSO_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { GSO_OK = 0, GSO_ERR_INVALID_ARGUMENT = 1, GSO_ERR_INDEX_OUT_OF_RANGE = 5,
       GSO_ERR_UNSORTED_GRAPH = 4 };

/* node-wise bias modes (R6, R11) */
enum { GSO_W_UNIFORM = 0, GSO_W_EDGE = 1, GSO_W_PASS_COLNORM = 2 };
/* layer-wise node-bias modes (R7-R9) */
enum { GSO_PROB_LADIES = 0, GSO_PROB_DEGREE = 1, GSO_PROB_COUNT = 2 };

/* CSC adjacency: column v lists the in-neighbours u of v; edge id =
 * position in indices.  weights may be NULL (unweighted: w == 1). Host memory. */
typedef struct gso_graph {
  int64_t num_nodes;
  int64_t num_edges;
  const int64_t* indptr;   /* [num_nodes+1] */
  const int32_t* indices;  /* [num_edges]   */
  const float* weights;    /* [num_edges] or NULL */
} gso_graph;

/* One sampled block of one (batch, layer): a sub-matrix of A over local ids. */
typedef struct gso_block_view {
  int64_t n_cols, n_rows, n_edges;
  const int32_t* col_map;   /* [n_cols] local col -> global node (the frontier) */
  const int32_t* row_map;   /* [n_rows] local row -> global node (A.row()) */
  const int64_t* indptr;    /* [n_cols+1] CSC over local ids */
  const int32_t* row_local; /* [n_edges] */
  const int64_t* eid;       /* [n_edges] global edge ids */
  const float* val;         /* [n_edges] or NULL (LADIES val, PASS prob) */
  const float* row_prob;    /* [n_rows] or NULL (layer-wise p(u)) */
} gso_block_view;

typedef struct gso_result gso_result;

/* Philox4x32-10 (Salmon et al. SC'11), out = philox(ctr, key). */
void gso_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
/* floor(((r1<<32)|r0) * n / 2^64): integer draw in [0, n) (R23). */
uint64_t gso_uniform_below(uint64_t n, uint32_t r0, uint32_t r1);
/* A-Res exponential key -log((r+0.5)*2^-32) / bias in fp64 (R6). */
double gso_ares_key(uint32_t r, double bias);

/* Node-wise sampling: GraphSAGE (replace=0, UNIFORM), KGCN (replace=1),
 * weighted A-Res (EDGE), PASS-style A3 probabilities (PASS_COLNORM).
 * Seeds are cut into batches of batch_size (the last may be shorter); batch b
 * uses global batch index batch_index_base + b in every Philox counter.
 * fanouts[l] applies to the frontier of layer l (fanouts[0] -> seeds). */
int gso_sample_neighbors(const gso_graph* g, const int32_t* seeds, int64_t num_seeds,
                         int64_t batch_size, int64_t batch_index_base,
                         const int32_t* fanouts, int num_layers, int replace, int bias_mode,
                         uint64_t rng_key, int num_threads, gso_result** out);

/* Layer-wise sampling: LADIES / FastGCN (DEGREE) / COUNT, K = n_per_layer[l]. */
int gso_sample_layerwise(const gso_graph* g, const int32_t* seeds, int64_t num_seeds,
                         int64_t batch_size, int64_t batch_index_base,
                         const int32_t* n_per_layer, int num_layers, int prob_mode,
                         uint64_t rng_key, int num_threads, gso_result** out);

/* ShaDow: node-wise sampling for the given fanouts, then the subgraph induced
 * on the union of all sampled nodes of each batch (one block per batch). */
int gso_shadow(const gso_graph* g, const int32_t* seeds, int64_t num_seeds,
               int64_t batch_size, int64_t batch_index_base,
               const int32_t* fanouts, int num_layers, int bias_mode,
               uint64_t rng_key, int num_threads, gso_result** out);

/* GraphSAINT-RW (Table 2; R26): a DeepWalk walk of walk_length steps
 * from every root (global walker index batch_index_base * batch_size + i),
 * then per batch of batch_size roots the subgraph induced on the visited nodes
 * (as ShaDow: U ascending, one block per batch). */
int gso_saint_rw(const gso_graph* g, const int32_t* roots, int64_t num_roots, int64_t batch_size,
                 int64_t batch_index_base, int walk_length, uint64_t rng_key, int num_threads,
                 gso_result** out);

/* PinSAGE-style (Table 2; R27): per frontier v, num_walks walks of at
 * most walk_length steps, each step preceded by an end-with-probability
 * restart_prob test; the topk[l] most visited nodes != v (count descending,
 * id ascending) are v's neighbours (val = visit count, eid = -1).  Next
 * frontier = row_map (the selected nodes, ascending). */
int gso_pinsage(const gso_graph* g, const int32_t* seeds, int64_t num_seeds, int64_t batch_size,
                int64_t batch_index_base, const int32_t* topk, int num_layers, int num_walks,
                int walk_length, float restart_prob, uint64_t rng_key, int num_threads,
                gso_result** out);

/* DeepWalk (p == q == 1 and !force_node2vec) / Node2Vec random walks.
 * traces: caller-owned int32 [num_walkers][length+1], -1 after a dead end. */
int gso_random_walk(const gso_graph* g, const int32_t* starts, int64_t num_walkers,
                    int64_t walker_index_base, int length, float p, float q,
                    uint64_t rng_key, int force_node2vec, int num_threads, int32_t* traces);

int64_t gso_result_num_batches(const gso_result* r);
int gso_result_num_layers(const gso_result* r);
int gso_result_view(const gso_result* r, int64_t batch, int layer, gso_block_view* out);
void gso_result_free(gso_result* r);

#ifdef __cplusplus
}
#endif
#endif
