// Grid- and cluster-engine kernels instantiated for key type F64 (see engine_grid.cuh).
#include "engine_batch.cuh"
#include "engine_resident.cuh"
#include "engine_cluster.cuh"
#include "engine_grid.cuh"

namespace airtopk {
AIRTOPK_INSTANTIATE_GRID(K_F64)
AIRTOPK_INSTANTIATE_CLUSTER(K_F64)
AIRTOPK_INSTANTIATE_BATCH(K_F64)
AIRTOPK_INSTANTIATE_RESIDENT(K_F64)
}  // namespace airtopk
