// Instantiation unit: tree traversal kernels for d = any (runtime d).
#include "knn_tree.cuh"

namespace psb {
template int launch_tree_v<0>(int, const DevIndex &, const float *, int64_t, int, int32_t *, float *,
                                cudaStream_t, uint32_t, int64_t *, cudaMemPool_t, int);
}
