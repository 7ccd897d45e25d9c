/* gs_c_client.c -- a plain C99 consumer of include/gs.h (no CUDA headers).
 * Builds a 6-node CSC on the host, creates the graph with GS_GRAPH_HOST_PTRS,
 * samples one GraphSAGE [2,2] batch and prints layer 0's block:
 *   "n_cols n_rows n_edges" then the eids, then the row_map.
 * The CUDA runtime entry points it needs are declared here by hand (their C
 * ABI); tests/test_c_abi.py compiles it with gcc -std=c99 -Werror and, on a
 * GPU, compares its output with the oracle. */
#include <stdio.h>
#include <stdlib.h>

#include "gs.h"

int cudaMalloc(void** p, size_t bytes);
int cudaFree(void* p);
int cudaMemcpy(void* dst, const void* src, size_t bytes, int kind);
int cudaDeviceSynchronize(void);
enum { H2D = 1, D2H = 2 };

#define CHECK(x)                                                          \
  do {                                                                    \
    gs_status s_ = (x);                                                   \
    if (s_ != GS_OK) {                                                    \
      fprintf(stderr, "%s -> %s: %s\n", #x, gs_status_string(s_), gs_last_error()); \
      return 1;                                                           \
    }                                                                     \
  } while (0)

int main(void) {
  /* column v lists the in-neighbours of v, ascending */
  const int64_t indptr[7] = {0, 3, 6, 8, 9, 12, 14};
  const int32_t indices[14] = {1, 2, 4, 0, 3, 5, 0, 1, 2, 0, 1, 3, 2, 4};
  const int32_t seeds_h[3] = {0, 1, 4};
  const int32_t fanouts[2] = {2, 2};
  gs_graph* g = NULL;
  gs_blocks* blk = NULL;
  gs_block_view v;
  int32_t* seeds_d = NULL;
  int64_t eid[64];
  int32_t rows[64];
  int64_t i;
  CHECK(gs_graph_create(indptr, indices, NULL, 6, 14, GS_GRAPH_HOST_PTRS, NULL, &g));
  if (cudaMalloc((void**)&seeds_d, sizeof seeds_h) != 0) return 2;
  if (cudaMemcpy(seeds_d, seeds_h, sizeof seeds_h, H2D) != 0) return 2;
  CHECK(gs_sample_neighbors(g, seeds_d, 3, 3, 0, fanouts, 2, 0, GS_W_UNIFORM, 42u, NULL, &blk));
  CHECK(gs_blocks_sync(blk));
  CHECK(gs_blocks_view(blk, 0, 0, &v));
  if (v.n_edges > 64 || v.n_rows > 64) return 3;
  if (cudaMemcpy(eid, v.eid, (size_t)v.n_edges * 8, D2H) != 0) return 2;
  if (cudaMemcpy(rows, v.row_map, (size_t)v.n_rows * 4, D2H) != 0) return 2;
  printf("%lld %lld %lld\n", (long long)v.n_cols, (long long)v.n_rows, (long long)v.n_edges);
  for (i = 0; i < v.n_edges; ++i) printf("%lld ", (long long)eid[i]);
  printf("\n");
  for (i = 0; i < v.n_rows; ++i) printf("%d ", rows[i]);
  printf("\n");
  gs_blocks_destroy(blk);
  gs_graph_destroy(g);
  cudaFree(seeds_d);
  return 0;
}
