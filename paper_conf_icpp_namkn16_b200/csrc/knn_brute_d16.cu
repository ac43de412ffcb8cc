// Instantiation unit: brute-force kernels for d = 16.
#include "knn_brute.cuh"

namespace psb {
template int launch_brute_v<16>(const DevIndex &, const float *, int64_t, int, int32_t *, float *, cudaStream_t,
                                 int, cudaMemPool_t);
}
