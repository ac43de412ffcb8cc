// Instantiation unit: brute-force kernels for d = 3, fanout 64.
#include "knn_brute.cuh"

namespace psb {
template int launch_brute_ks<3, 2>(const DevIndex &, const float *, int64_t, int, int32_t *, float *,
                                      cudaStream_t, int, cudaMemPool_t);
}
