// Instantiation unit: brute-force kernels for any d (runtime), fanout 128.
#include "knn_brute.cuh"

namespace psb {
template int launch_brute_ks<0, 4>(const DevIndex &, const float *, int64_t, int, int32_t *, float *,
                                      cudaStream_t, int, cudaMemPool_t);
}
