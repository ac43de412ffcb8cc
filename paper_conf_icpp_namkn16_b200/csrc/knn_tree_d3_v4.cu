// Instantiation unit: tree traversal kernels for d = 3, fanout 128.
#include "knn_tree.cuh"

namespace psb {
template int launch_tree_ks<3, 4>(int, const DevIndex &, const float *, int64_t, int, int32_t *, float *,
                                     cudaStream_t, uint32_t, int64_t *, cudaMemPool_t, int,
                                     const TraceOut &);
}
