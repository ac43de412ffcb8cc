// Instantiation unit: brute-force kernels for d = 3.
#include "knn_brute.cuh"

namespace psb {
template int launch_brute_v<3>(const DevIndex &, const float *, int64_t, int, int32_t *, float *, cudaStream_t,
                                 int, cudaMemPool_t);
}
