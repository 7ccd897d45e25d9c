// gso.cpp -- CPU ORACLE for the gSampler ECSF hot path (test infrastructure
// only; see gso.h for who may load it).  Plain, slow, single-threaded per
// batch; OpenMP only over independent batches / walkers.  Shares no code with
// the CUDA path.  "P:n" = line n of the paper text; "R<n>" = the
// reading n listed in DESIGN.md (which follows SURVEY.md section 8(c)).
//
// Build: g++ -O2 -std=c++17 -ffp-contract=off -fopenmp -shared -fPIC
#include "gso.h"

#include <algorithm>
#include <cmath>
#include <cstring>
#include <unordered_map>
#include <utility>
#include <map>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {

// ---------------------------------------------------------------------------
// Philox4x32-10 (Salmon, Moraes, Dror, Shaw, SC'11), R-keying in DESIGN.md R4.
// ---------------------------------------------------------------------------
const uint32_t PHILOX_M0 = 0xD2511F53u, PHILOX_M1 = 0xCD9E8D57u;
const uint32_t PHILOX_W0 = 0x9E3779B9u, PHILOX_W1 = 0xBB67AE85u;

struct Word4 { uint32_t v[4]; };

Word4 philox(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3, uint64_t rng_key) {
  uint32_t c[4] = {c0, c1, c2, c3};
  uint32_t k0 = (uint32_t)(rng_key & 0xffffffffu), k1 = (uint32_t)(rng_key >> 32);
  for (int round = 0; round < 10; ++round) {
    uint64_t p0 = (uint64_t)PHILOX_M0 * c[0];
    uint64_t p1 = (uint64_t)PHILOX_M1 * c[2];
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c[1] ^ k0;
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c[3] ^ k1;
    uint32_t n3 = lo0;
    c[0] = n0; c[1] = n1; c[2] = n2; c[3] = n3;
    if (round < 9) { k0 += PHILOX_W0; k1 += PHILOX_W1; }
  }
  Word4 w;
  for (int i = 0; i < 4; ++i) w.v[i] = c[i];
  return w;
}

// Tags of the counter word c2 = layer_or_step | tag << 24 (R4).
enum { TAG_FLOYD = 1, TAG_REPLACE = 2, TAG_ARES_NODE = 3, TAG_ARES_LAYER = 4,
       TAG_DEEPWALK = 5, TAG_NODE2VEC = 6, TAG_PINSAGE = 7 };

uint32_t c2_of(int layer, int tag) { return (uint32_t)layer | ((uint32_t)tag << 24); }

// R23: floor(r * n / 2^64) with r = r1:r0, exact 128-bit product.
uint64_t uniform_below(uint64_t n, uint32_t r0, uint32_t r1) {
  unsigned __int128 r = ((unsigned __int128)r1 << 32) | r0;
  return (uint64_t)((r * n) >> 64);
}

// R6: exponential key of Efraimidis-Spirakis A-Res, fp64.
double ares_key(uint32_t r, double bias) {
  double u = ((double)r + 0.5) * 0x1p-32;
  double e = -std::log(u);
  return e / bias;
}

// ---------------------------------------------------------------------------
// Result storage
// ---------------------------------------------------------------------------
struct Block {
  std::vector<int32_t> col_map, row_map, row_local;
  std::vector<int64_t> indptr, eid;
  std::vector<float> val, row_prob;
  bool has_val = false, has_row_prob = false;
};

struct Graph {
  int64_t n, nnz;
  const int64_t* indptr;
  const int32_t* indices;
  const float* weights;
  int64_t off(int32_t v) const { return indptr[v]; }
  int64_t deg(int32_t v) const { return indptr[v + 1] - indptr[v]; }
  float w(int64_t e) const { return weights ? weights[e] : 1.0f; }
};

// Finalize (R3): row_map = A.row() = the unique rows of the
// block in ascending node-id order (the row set of a sparse matrix);
// row_local[e] = index of the edge's row in row_map.
void finalize_rows_ascending(const std::vector<int32_t>& edge_u, Block& blk) {
  blk.row_map = edge_u;
  std::sort(blk.row_map.begin(), blk.row_map.end());
  blk.row_map.erase(std::unique(blk.row_map.begin(), blk.row_map.end()), blk.row_map.end());
  blk.row_local.resize(edge_u.size());
  for (size_t e = 0; e < edge_u.size(); ++e)
    blk.row_local[e] = (int32_t)(std::lower_bound(blk.row_map.begin(), blk.row_map.end(),
                                                  edge_u[e]) - blk.row_map.begin());
}

// ---------------------------------------------------------------------------
// Select, node-wise (individual_sample)
// Returns positions inside column v (0..d-1) in output order.
// ---------------------------------------------------------------------------

// R5: Robert Floyd's algorithm for a uniform k-subset of {0..d-1}.
std::vector<int64_t> select_floyd(const Graph& g, int32_t v, int k, int layer, uint32_t batch,
                                  uint64_t key) {
  int64_t d = g.deg(v);
  std::vector<int64_t> pos;
  if (d <= k) {  // take every neighbour, no randomness consumed
    for (int64_t i = 0; i < d; ++i) pos.push_back(i);
    return pos;
  }
  for (int s = 0; s < k; ++s) {
    Word4 r = philox((uint32_t)v, (uint32_t)s, c2_of(layer, TAG_FLOYD), batch, key);
    int64_t m = d - k + s;
    int64_t t = (int64_t)uniform_below((uint64_t)(m + 1), r.v[0], r.v[1]);
    bool seen = std::find(pos.begin(), pos.end(), t) != pos.end();
    pos.push_back(seen ? m : t);
  }
  std::sort(pos.begin(), pos.end());  // R4/Q4: ascending position
  return pos;
}

// R10: KGCN -- k i.i.d. uniform positions with replacement, in slot order.
std::vector<int64_t> select_replace(const Graph& g, int32_t v, int k, int layer, uint32_t batch,
                                    uint64_t key) {
  int64_t d = g.deg(v);
  std::vector<int64_t> pos;
  if (d == 0) return pos;
  for (int s = 0; s < k; ++s) {
    Word4 r = philox((uint32_t)v, (uint32_t)s, c2_of(layer, TAG_REPLACE), batch, key);
    pos.push_back((int64_t)uniform_below((uint64_t)d, r.v[0], r.v[1]));
  }
  return pos;
}

// R6: weighted without replacement, A-Res keys over eligible (w > 0) positions.
std::vector<int64_t> select_ares(const Graph& g, int32_t v, int k, int layer, uint32_t batch,
                                 uint64_t key) {
  int64_t d = g.deg(v), off = g.off(v);
  std::vector<int64_t> eligible;
  for (int64_t i = 0; i < d; ++i)
    if (g.w(off + i) > 0.0f) eligible.push_back(i);
  if ((int64_t)eligible.size() <= k) return eligible;
  std::vector<std::pair<double, int64_t>> keyed;
  for (int64_t i : eligible) {
    Word4 r = philox((uint32_t)v, (uint32_t)(i >> 2), c2_of(layer, TAG_ARES_NODE), batch, key);
    keyed.push_back({ares_key(r.v[i & 3], (double)g.w(off + i)), i});
  }
  std::sort(keyed.begin(), keyed.end());  // ties -> smaller position
  std::vector<int64_t> pos;
  for (int s = 0; s < k; ++s) pos.push_back(keyed[s].second);
  std::sort(pos.begin(), pos.end());
  return pos;
}

// One node-wise layer: Extract + Select + Finalize; PASS-style A3
// probabilities prob_e = w_e / sum(w over the whole column) (R11).
Block nodewise_layer(const Graph& g, const std::vector<int32_t>& frontier, int k, int layer,
                     uint32_t batch, int replace, int bias_mode, uint64_t key) {
  Block blk;
  blk.col_map = frontier;
  blk.indptr.push_back(0);
  blk.has_val = (bias_mode == GSO_W_PASS_COLNORM);
  std::vector<int32_t> edge_u;
  for (int32_t v : frontier) {
    std::vector<int64_t> pos;
    if (replace) pos = select_replace(g, v, k, layer, batch, key);
    else if (bias_mode == GSO_W_UNIFORM) pos = select_floyd(g, v, k, layer, batch, key);
    else pos = select_ares(g, v, k, layer, batch, key);
    int64_t off = g.off(v);
    float colsum = 0.0f;
    if (blk.has_val) {
      double s = 0.0;
      for (int64_t i = 0; i < g.deg(v); ++i) s += (double)g.w(off + i);
      colsum = (float)s;
    }
    for (int64_t p : pos) {
      edge_u.push_back(g.indices[off + p]);
      blk.eid.push_back(off + p);
      if (blk.has_val) blk.val.push_back(g.w(off + p) / colsum);
    }
    blk.indptr.push_back((int64_t)edge_u.size());
  }
  finalize_rows_ascending(edge_u, blk);
  return blk;
}

bool frontier_in_range(const Graph& g, const int32_t* f, int64_t n) {
  for (int64_t i = 0; i < n; ++i)
    if (f[i] < 0 || (int64_t)f[i] >= g.n) return false;
  return true;
}

// ---------------------------------------------------------------------------
// Select, layer-wise (collective_sample) with the LADIES
// compute/finalize of Fig. 3(b) and Table 2; R7-R9, R24.
// ---------------------------------------------------------------------------
Block layerwise_layer(const Graph& g, const std::vector<int32_t>& frontier, int K, int layer,
                      uint32_t batch, int prob_mode, uint64_t key) {
  Block blk;
  blk.col_map = frontier;
  blk.has_val = true;
  blk.has_row_prob = true;
  // Extract A[:, F] and Compute the per-candidate bias b(u) (row sum, R1).
  std::unordered_map<int32_t, double> sum_w2;
  std::unordered_map<int32_t, int64_t> count;
  std::vector<int32_t> cand;  // C in first-seen order (order irrelevant)
  for (int32_t v : frontier) {
    int64_t off = g.off(v);
    for (int64_t i = 0; i < g.deg(v); ++i) {
      int32_t u = g.indices[off + i];
      float w = g.w(off + i);
      float w2 = w * w;  // (A ** 2), pre-computable per P:300
      if (!count.count(u)) cand.push_back(u);
      sum_w2[u] += (double)w2;
      count[u] += 1;
    }
  }
  std::unordered_map<int32_t, float> bias;
  double total = 0.0;
  for (int32_t u : cand) {
    float b;
    if (prob_mode == GSO_PROB_LADIES) b = (float)sum_w2[u];
    else if (prob_mode == GSO_PROB_DEGREE) b = (float)g.deg(u);
    else b = (float)count[u];
    bias[u] = b;
    total += (double)b;
  }
  float B = (float)total;
  std::vector<int32_t> eligible;
  for (int32_t u : cand)
    if (bias[u] > 0.0f) eligible.push_back(u);
  std::vector<int32_t> S;
  if ((int64_t)eligible.size() <= K) {
    S = eligible;
  } else {
    std::vector<std::pair<double, int32_t>> keyed;
    for (int32_t u : eligible) {
      Word4 r = philox((uint32_t)u, 0u, c2_of(layer, TAG_ARES_LAYER), batch, key);
      keyed.push_back({ares_key(r.v[0], (double)bias[u]), u});
    }
    std::sort(keyed.begin(), keyed.end());  // ties -> smaller node id
    for (int s = 0; s < K; ++s) S.push_back(keyed[s].second);
  }
  std::sort(S.begin(), S.end());
  std::unordered_map<int32_t, int32_t> local;
  for (size_t i = 0; i < S.size(); ++i) {
    local[S[i]] = (int32_t)i;
    blk.row_map.push_back(S[i]);
    blk.row_prob.push_back(bias[S[i]] / B);  // p(u) = b(u) / B
  }
  // Finalize: keep E_F edges whose row is in S (CSC order), divide by p(u),
  // then normalise each column by its sum (Fig. 3(b) lines 5-7).
  blk.indptr.push_back(0);
  for (int32_t v : frontier) {
    int64_t off = g.off(v);
    std::vector<float> a_col;
    for (int64_t i = 0; i < g.deg(v); ++i) {
      int32_t u = g.indices[off + i];
      auto it = local.find(u);
      if (it == local.end()) continue;
      float p = blk.row_prob[it->second];
      float a = g.w(off + i) / p;
      blk.row_local.push_back(it->second);
      blk.eid.push_back(off + i);
      a_col.push_back(a);
    }
    double csum = 0.0;
    for (float a : a_col) csum += (double)a;
    float c = (float)csum;
    for (float a : a_col) blk.val.push_back(a / c);
    blk.indptr.push_back((int64_t)blk.eid.size());
  }
  return blk;
}

}  // namespace

struct gso_result {
  int64_t num_batches = 0;
  int num_layers = 0;
  std::vector<Block> blocks;  // [batch][layer]
};

extern "C" {

void gso_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
  Word4 w = philox(ctr[0], ctr[1], ctr[2], ctr[3], ((uint64_t)key[1] << 32) | key[0]);
  for (int i = 0; i < 4; ++i) out[i] = w.v[i];
}

uint64_t gso_uniform_below(uint64_t n, uint32_t r0, uint32_t r1) { return uniform_below(n, r0, r1); }

double gso_ares_key(uint32_t r, double bias) { return ares_key(r, bias); }

static int set_threads(int num_threads) {
#ifdef _OPENMP
  if (num_threads > 0) omp_set_num_threads(num_threads);
#endif
  (void)num_threads;
  return 0;
}

static int check_common(const gso_graph* g, const int32_t* seeds, int64_t num_seeds,
                        int64_t batch_size, int num_layers, const int32_t* per_layer,
                        gso_result** out) {
  if (!g || !out || (!seeds && num_seeds > 0) || num_seeds < 0 || batch_size <= 0 ||
      num_layers < 1 || num_layers > 8 || !per_layer)
    return GSO_ERR_INVALID_ARGUMENT;
  for (int l = 0; l < num_layers; ++l)
    if (per_layer[l] <= 0) return GSO_ERR_INVALID_ARGUMENT;
  Graph gg{g->num_nodes, g->num_edges, g->indptr, g->indices, g->weights};
  if (!frontier_in_range(gg, seeds, num_seeds)) return GSO_ERR_INDEX_OUT_OF_RANGE;
  return GSO_OK;
}

int gso_sample_neighbors(const gso_graph* g, const int32_t* seeds, int64_t num_seeds,
                         int64_t batch_size, int64_t batch_index_base, const int32_t* fanouts,
                         int num_layers, int replace, int bias_mode, uint64_t rng_key,
                         int num_threads, gso_result** out) {
  int st = check_common(g, seeds, num_seeds, batch_size, num_layers, fanouts, out);
  if (st) return st;
  if (bias_mode < 0 || bias_mode > 2 || (replace && bias_mode != GSO_W_UNIFORM))
    return GSO_ERR_INVALID_ARGUMENT;
  Graph gg{g->num_nodes, g->num_edges, g->indptr, g->indices, g->weights};
  gso_result* r = new gso_result();
  r->num_batches = (num_seeds + batch_size - 1) / batch_size;
  r->num_layers = num_layers;
  r->blocks.resize((size_t)r->num_batches * num_layers);
  set_threads(num_threads);
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t b = 0; b < r->num_batches; ++b) {
    int64_t lo = b * batch_size, hi = std::min(num_seeds, lo + batch_size);
    std::vector<int32_t> frontier(seeds + lo, seeds + hi);
    uint32_t gb = (uint32_t)(batch_index_base + b);
    for (int l = 0; l < num_layers; ++l) {
      Block blk = nodewise_layer(gg, frontier, fanouts[l], l, gb, replace, bias_mode, rng_key);
      frontier = blk.row_map;  // next frontiers = sample_A.row() (R2)
      r->blocks[(size_t)b * num_layers + l] = std::move(blk);
    }
  }
  *out = r;
  return GSO_OK;
}

int gso_sample_layerwise(const gso_graph* g, const int32_t* seeds, int64_t num_seeds,
                         int64_t batch_size, int64_t batch_index_base,
                         const int32_t* n_per_layer, int num_layers, int prob_mode,
                         uint64_t rng_key, int num_threads, gso_result** out) {
  int st = check_common(g, seeds, num_seeds, batch_size, num_layers, n_per_layer, out);
  if (st) return st;
  if (prob_mode < 0 || prob_mode > 2) return GSO_ERR_INVALID_ARGUMENT;
  Graph gg{g->num_nodes, g->num_edges, g->indptr, g->indices, g->weights};
  gso_result* r = new gso_result();
  r->num_batches = (num_seeds + batch_size - 1) / batch_size;
  r->num_layers = num_layers;
  r->blocks.resize((size_t)r->num_batches * num_layers);
  set_threads(num_threads);
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t b = 0; b < r->num_batches; ++b) {
    int64_t lo = b * batch_size, hi = std::min(num_seeds, lo + batch_size);
    std::vector<int32_t> frontier(seeds + lo, seeds + hi);
    uint32_t gb = (uint32_t)(batch_index_base + b);
    for (int l = 0; l < num_layers; ++l) {
      Block blk = layerwise_layer(gg, frontier, n_per_layer[l], l, gb, prob_mode, rng_key);
      frontier = blk.row_map;  // F_{l+1} = S
      r->blocks[(size_t)b * num_layers + l] = std::move(blk);
    }
  }
  *out = r;
  return GSO_OK;
}

// Induce (R12): U = unique(nodes) in ascending order, then
// every edge u->v of A with u, v in U, columns in U order, CSC order inside.
static Block induce(const Graph& gg, std::vector<int32_t> all) {
  Block ind;
  std::sort(all.begin(), all.end());
  all.erase(std::unique(all.begin(), all.end()), all.end());
  ind.row_map = all;
  std::unordered_map<int32_t, int32_t> local;
  for (size_t i = 0; i < all.size(); ++i) local[all[i]] = (int32_t)i;
  ind.col_map = ind.row_map;
  ind.indptr.push_back(0);
  for (int32_t v : ind.col_map) {
    int64_t off = gg.off(v);
    for (int64_t i = 0; i < gg.deg(v); ++i) {
      auto it = local.find(gg.indices[off + i]);
      if (it == local.end()) continue;
      ind.row_local.push_back(it->second);
      ind.eid.push_back(off + i);
    }
    ind.indptr.push_back((int64_t)ind.eid.size());
  }
  return ind;
}

int gso_shadow(const gso_graph* g, const int32_t* seeds, int64_t num_seeds, int64_t batch_size,
               int64_t batch_index_base, const int32_t* fanouts, int num_layers, int bias_mode,
               uint64_t rng_key, int num_threads, gso_result** out) {
  int st = check_common(g, seeds, num_seeds, batch_size, num_layers, fanouts, out);
  if (st) return st;
  if (bias_mode < 0 || bias_mode > 1) return GSO_ERR_INVALID_ARGUMENT;
  Graph gg{g->num_nodes, g->num_edges, g->indptr, g->indices, g->weights};
  gso_result* r = new gso_result();
  r->num_batches = (num_seeds + batch_size - 1) / batch_size;
  r->num_layers = 1;
  r->blocks.resize((size_t)r->num_batches);
  set_threads(num_threads);
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t b = 0; b < r->num_batches; ++b) {
    int64_t lo = b * batch_size, hi = std::min(num_seeds, lo + batch_size);
    std::vector<int32_t> frontier(seeds + lo, seeds + hi);
    uint32_t gb = (uint32_t)(batch_index_base + b);
    // U = unique of (F0, row_map_0, row_map_1, ...) in ascending order (R12)
    std::vector<int32_t> all(frontier);
    for (int l = 0; l < num_layers; ++l) {
      Block blk = nodewise_layer(gg, frontier, fanouts[l], l, gb, 0, bias_mode, rng_key);
      frontier = blk.row_map;
      all.insert(all.end(), blk.row_map.begin(), blk.row_map.end());
    }
    Block ind = induce(gg, std::move(all));
    r->blocks[(size_t)b] = std::move(ind);
  }
  *out = r;
  return GSO_OK;
}

int gso_random_walk(const gso_graph* g, const int32_t* starts, int64_t num_walkers,
                    int64_t walker_index_base, int length, float p, float q, uint64_t rng_key,
                    int force_node2vec, int num_threads, int32_t* traces) {
  if (!g || (!starts && num_walkers > 0) || !traces || num_walkers < 0 || length < 0 ||
      !(p > 0.0f) || !(q > 0.0f))
    return GSO_ERR_INVALID_ARGUMENT;
  Graph gg{g->num_nodes, g->num_edges, g->indptr, g->indices, g->weights};
  if (!frontier_in_range(gg, starts, num_walkers)) return GSO_ERR_INDEX_OUT_OF_RANGE;
  const bool node2vec = force_node2vec || p != 1.0f || q != 1.0f;
  const float bp = 1.0f / p, bq = 1.0f / q;
  const float bmax = std::max(bp, std::max(1.0f, bq));
  const int64_t L1 = (int64_t)length + 1;
  set_threads(num_threads);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < num_walkers; ++i) {
    int32_t* tr = traces + i * L1;
    uint32_t walker = (uint32_t)(walker_index_base + i);
    tr[0] = starts[i];
    for (int t = 1; t <= length; ++t) {
      int32_t v = tr[t - 1];
      if (v < 0 || gg.deg(v) == 0) {  // dead end -> -1 padding (R13)
        tr[t] = -1;
        continue;
      }
      int64_t off = gg.off(v), d = gg.deg(v);
      if (!node2vec) {  // DeepWalk: uniform in-neighbour
        Word4 r = philox(walker, 0u, c2_of(t, TAG_DEEPWALK), 0u, rng_key);
        tr[t] = gg.indices[off + (int64_t)uniform_below((uint64_t)d, r.v[0], r.v[1])];
        continue;
      }
      if (t == 1) {  // Node2Vec first step has no previous node: uniform
        Word4 r = philox(walker, 0u, c2_of(t, TAG_NODE2VEC), 0u, rng_key);
        tr[t] = gg.indices[off + (int64_t)uniform_below((uint64_t)d, r.v[0], r.v[1])];
        continue;
      }
      // Node2Vec second-order bias 1/p (return), 1 (distance 1), 1/q,
      // realised by rejection sampling against bmax (R14).
      int32_t prev = tr[t - 2];
      const int32_t* pb = gg.indices + gg.off(prev);
      const int32_t* pe = pb + gg.deg(prev);
      for (uint32_t trial = 0;; ++trial) {
        Word4 r = philox(walker, trial, c2_of(t, TAG_NODE2VEC), 0u, rng_key);
        int32_t x = gg.indices[off + (int64_t)uniform_below((uint64_t)d, r.v[0], r.v[1])];
        float bias;
        if (x == prev) bias = bp;
        else if (std::binary_search(pb, pe, x)) bias = 1.0f;
        else bias = bq;
        float y = (float)(r.v[2] >> 8) * 0x1p-24f;
        y = y * bmax;
        if (y < bias || trial == 4095u) {
          tr[t] = x;
          break;
        }
      }
    }
  }
  return GSO_OK;
}

int64_t gso_result_num_batches(const gso_result* r) { return r ? r->num_batches : 0; }
int gso_result_num_layers(const gso_result* r) { return r ? r->num_layers : 0; }

int gso_result_view(const gso_result* r, int64_t batch, int layer, gso_block_view* out) {
  if (!r || !out || batch < 0 || batch >= r->num_batches || layer < 0 || layer >= r->num_layers)
    return GSO_ERR_INVALID_ARGUMENT;
  const Block& b = r->blocks[(size_t)batch * r->num_layers + layer];
  out->n_cols = (int64_t)b.col_map.size();
  out->n_rows = (int64_t)b.row_map.size();
  out->n_edges = (int64_t)b.eid.size();
  out->col_map = b.col_map.data();
  out->row_map = b.row_map.data();
  out->indptr = b.indptr.data();
  out->row_local = b.row_local.data();
  out->eid = b.eid.data();
  out->val = b.has_val ? b.val.data() : nullptr;
  out->row_prob = b.has_row_prob ? b.row_prob.data() : nullptr;
  return GSO_OK;
}

void gso_result_free(gso_result* r) { delete r; }

}  // extern "C"

int gso_saint_rw(const gso_graph* g, const int32_t* roots, int64_t num_roots, int64_t batch_size,
                 int64_t batch_index_base, int walk_length, uint64_t rng_key, int num_threads,
                 gso_result** out) {
  if (!g || !out || (!roots && num_roots > 0) || num_roots < 0 || batch_size <= 0 ||
      batch_index_base < 0 || walk_length < 0)
    return GSO_ERR_INVALID_ARGUMENT;
  Graph gg{g->num_nodes, g->num_edges, g->indptr, g->indices, g->weights};
  if (!frontier_in_range(gg, roots, num_roots)) return GSO_ERR_INDEX_OUT_OF_RANGE;
  // GraphSAINT-RW (Table 2; R26): a DeepWalk walk from every root,
  // keyed by the global walker index (batch_index_base * batch_size + i) ...
  const int64_t L1 = (int64_t)walk_length + 1;
  std::vector<int32_t> traces((size_t)(num_roots * L1));
  int st = gso_random_walk(g, roots, num_roots, batch_index_base * batch_size, walk_length, 1.0f,
                           1.0f, rng_key, 0, num_threads, traces.data());
  if (st) return st;
  gso_result* r = new gso_result();
  r->num_batches = (num_roots + batch_size - 1) / batch_size;
  r->num_layers = 1;
  r->blocks.resize((size_t)r->num_batches);
  set_threads(num_threads);
  // ... then per batch the subgraph induced on the nodes its walks visited.
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t b = 0; b < r->num_batches; ++b) {
    int64_t lo = b * batch_size, hi = std::min(num_roots, lo + batch_size);
    std::vector<int32_t> all;
    for (int64_t i = lo * L1; i < hi * L1; ++i)
      if (traces[(size_t)i] >= 0) all.push_back(traces[(size_t)i]);  // -1: after a dead end (R13)
    r->blocks[(size_t)b] = induce(gg, std::move(all));
  }
  *out = r;
  return GSO_OK;
}

// PinSAGE-style (Table 2: "random walks ... using restarts, select
// top-k visited neighbors as sampled nodes"; R27).  For every frontier v:
// num_walks walks from v of at most walk_length steps; before each step the
// walk ends with probability restart_prob (the next walk restarts at v), or at
// a node with no in-neighbours; draw r = philox(v, w * walk_length + t - 1,
// layer | 7<<24, b): end if fp32((r2 >> 8) * 2^-24) < restart_prob, else step
// to in-neighbour draw_below(d, r0, r1).  Every visit of a node x != v counts;
// the k most visited (count descending, node id ascending) are v's sampled
// neighbours, in that rank order, with val = fp32(count).  eid = -1: these
// are not edges of A.  row_map = the selected nodes, unique ascending (R3).
static Block pinsage_layer(const Graph& gg, const std::vector<int32_t>& F, int k, int num_walks,
                           int walk_length, float restart_prob, int layer, uint32_t batch,
                           uint64_t key) {
  Block blk;
  blk.col_map = F;
  blk.has_val = true;
  std::vector<std::vector<std::pair<int64_t, int32_t>>> sel(F.size());  // (count, node)
  for (size_t j = 0; j < F.size(); ++j) {
    const int32_t v = F[j];
    std::map<int32_t, int64_t> count;
    for (int w = 0; w < num_walks; ++w) {
      int32_t x = v;
      for (int t = 1; t <= walk_length; ++t) {
        Word4 r = philox((uint32_t)v, (uint32_t)(w * walk_length + t - 1), c2_of(layer, TAG_PINSAGE),
                         batch, key);
        float y = (float)(r.v[2] >> 8) * 0x1p-24f;
        if (y < restart_prob) break;  // restart: the next walk starts at v again
        if (gg.deg(x) == 0) break;    // dead end (R13)
        x = gg.indices[gg.off(x) + (int64_t)uniform_below((uint64_t)gg.deg(x), r.v[0], r.v[1])];
        if (x != v) count[x] += 1;
      }
    }
    std::vector<std::pair<int64_t, int32_t>> ranked;
    for (auto& kv : count) ranked.push_back({kv.second, kv.first});
    std::sort(ranked.begin(), ranked.end(), [](const std::pair<int64_t, int32_t>& a,
                                               const std::pair<int64_t, int32_t>& b) {
      return a.first != b.first ? a.first > b.first : a.second < b.second;
    });
    if ((int)ranked.size() > k) ranked.resize((size_t)k);
    sel[j] = ranked;
  }
  std::vector<int32_t> rows;
  for (auto& sj : sel)
    for (auto& cx : sj) rows.push_back(cx.second);
  std::sort(rows.begin(), rows.end());
  rows.erase(std::unique(rows.begin(), rows.end()), rows.end());
  blk.row_map = rows;
  std::unordered_map<int32_t, int32_t> local;
  for (size_t i = 0; i < rows.size(); ++i) local[rows[i]] = (int32_t)i;
  blk.indptr.push_back(0);
  for (auto& sj : sel) {
    for (auto& cx : sj) {
      blk.row_local.push_back(local[cx.second]);
      blk.eid.push_back(-1);
      blk.val.push_back((float)cx.first);
    }
    blk.indptr.push_back((int64_t)blk.eid.size());
  }
  return blk;
}

int gso_pinsage(const gso_graph* g, const int32_t* seeds, int64_t num_seeds, int64_t batch_size,
                int64_t batch_index_base, const int32_t* topk, int num_layers, int num_walks,
                int walk_length, float restart_prob, uint64_t rng_key, int num_threads,
                gso_result** out) {
  int st = check_common(g, seeds, num_seeds, batch_size, num_layers, topk, out);
  if (st) return st;
  if (num_walks < 1 || walk_length < 1 || !(restart_prob >= 0.0f) || !(restart_prob <= 1.0f))
    return GSO_ERR_INVALID_ARGUMENT;
  Graph gg{g->num_nodes, g->num_edges, g->indptr, g->indices, g->weights};
  gso_result* r = new gso_result();
  r->num_batches = (num_seeds + batch_size - 1) / batch_size;
  r->num_layers = num_layers;
  r->blocks.resize((size_t)r->num_batches * num_layers);
  set_threads(num_threads);
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t b = 0; b < r->num_batches; ++b) {
    int64_t lo = b * batch_size, hi = std::min(num_seeds, lo + batch_size);
    std::vector<int32_t> frontier(seeds + lo, seeds + hi);
    uint32_t gb = (uint32_t)(batch_index_base + b);
    for (int l = 0; l < num_layers; ++l) {
      Block blk = pinsage_layer(gg, frontier, topk[l], num_walks, walk_length, restart_prob, l, gb,
                                rng_key);
      frontier = blk.row_map;  // next frontier = the selected nodes (R2)
      r->blocks[(size_t)b * num_layers + l] = std::move(blk);
    }
  }
  *out = r;
  return GSO_OK;
}
