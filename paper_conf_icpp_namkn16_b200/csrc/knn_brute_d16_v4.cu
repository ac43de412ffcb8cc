// Instantiation unit: brute-force kernels for d = 16, fanout 128.
#include "knn_brute.cuh"

namespace psb {
template int launch_brute_ks<16, 4>(const DevIndex &, const float *, int64_t, int, int32_t *, float *,
                                      cudaStream_t, int, cudaMemPool_t);
}
