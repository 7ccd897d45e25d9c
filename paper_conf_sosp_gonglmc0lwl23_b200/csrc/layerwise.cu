// layerwise.cu -- layer-wise ECSF sampling (FastGCN / LADIES / COUNT).
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "gs_internal.h"

namespace gsb {

gs_status run_layerwise(const gs_graph* g, const int32_t* seeds, int64_t num_seeds,
                        int64_t batch_size, int64_t batch_base, const int32_t* n_per_layer,
                        int L, int prob_mode, uint64_t key, cudaStream_t stream, gs_blocks* blk) {
  (void)g; (void)seeds; (void)num_seeds; (void)batch_size; (void)batch_base; (void)n_per_layer;
  (void)L; (void)prob_mode; (void)key; (void)stream; (void)blk;
  return fail(GS_ERR_NOT_SUPPORTED, "layer-wise sampling: not built yet");
}

}  // namespace gsb
