// Instantiation unit: tree traversal kernels for any d (runtime), fanout 64.
#include "knn_tree.cuh"

namespace psb {
template int launch_tree_ks<0, 2>(int, const DevIndex &, const float *, int64_t, int, int32_t *, float *,
                                     cudaStream_t, uint32_t, int64_t *, cudaMemPool_t, int,
                                     const TraceOut &);
}
