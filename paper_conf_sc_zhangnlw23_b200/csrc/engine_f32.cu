// Grid- and cluster-engine kernels instantiated for key type F32 (see engine_grid.cuh).
#include "engine_batch.cuh"
#include "engine_resident.cuh"
#include "engine_cluster.cuh"
#include "engine_grid.cuh"

namespace airtopk {
AIRTOPK_INSTANTIATE_GRID(K_F32)
AIRTOPK_INSTANTIATE_CLUSTER(K_F32)
AIRTOPK_INSTANTIATE_BATCH(K_F32)
AIRTOPK_INSTANTIATE_RESIDENT(K_F32)

int grid_occupancy_f32(int idx64) {
  int n = 0;
  cudaError_t e = idx64 ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, pass_kernel<K_F32, uint64_t, 1, 1, false>, kBlock, hist_smem_bytes<K_F32, uint64_t, 1, 1>())
                        : cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, pass_kernel<K_F32, uint32_t, 1, 1, false>, kBlock, hist_smem_bytes<K_F32, uint32_t, 1, 1>());
  return e == cudaSuccess ? n : -1;
}
}  // namespace airtopk
