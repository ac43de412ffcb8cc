// psb_probe.cu — measured memory ceilings for the rooflines bench.py reports
// (SURVEY.md §8(d) "which roofline binds": at C2-C5 the traversal's node and
// leaf blocks are served mostly from L2, so the ceiling that bounds their
// algorithmic bytes is the L2 read bandwidth, measured here on the same GPU in
// the same run instead of a guide figure).
#include <cuda_runtime.h>

#include "psb_launch.h"

namespace psb {

// Every thread streams 16-byte loads over its grid-strided share of the buffer,
// `passes` times. ld.global.cg caches in L2 only, so no pass is served from L1
// and every byte crosses the L2 -> SM path; the xor keeps the loads alive.
__global__ void __launch_bounds__(512) l2_read_kernel(const uint4 *__restrict__ buf, int64_t n16, int passes,
                                                      unsigned *__restrict__ sink)
{
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    unsigned acc = 0;
    for (int p = 0; p < passes; ++p) {
        for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += stride) {
            uint4 v = __ldcg(buf + i);
            acc ^= v.x ^ v.y ^ v.z ^ v.w;
        }
    }
    if (acc == 0x9e3779b9u) sink[0] = acc;   // practically never taken; defeats dead-code elimination
}

}  // namespace psb

using namespace psb;

extern "C" int psb_probe_l2_read(int64_t bytes, int32_t passes, int32_t reps, double *gbs)
{
    if (!gbs || bytes < (1 << 20) || passes < 1 || reps < 1) {
        psb_set_error("psb_probe_l2_read: bad argument");
        return PSB_EINVAL;
    }
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t n16 = bytes / 16;
    uint4 *buf = nullptr;
    unsigned *sink = nullptr;
    cudaEvent_t a = nullptr, b = nullptr;
    cudaStream_t st = nullptr;
    cudaError_t e;
    int rc = PSB_OK;
    double best = 0.0;
    if ((e = cudaMalloc((void **)&buf, n16 * 16)) != cudaSuccess || (e = cudaMalloc((void **)&sink, 4)) != cudaSuccess ||
        (e = cudaMemset(buf, 0x5a, n16 * 16)) != cudaSuccess || (e = cudaEventCreate(&a)) != cudaSuccess ||
        (e = cudaEventCreate(&b)) != cudaSuccess ||
        (e = cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking)) != cudaSuccess) {
        rc = report_cuda(e, "psb_probe_l2_read: setup");
    }
    const unsigned grid = (unsigned)sms * 4;   // 4 x 512 threads per SM: full occupancy
    if (rc == PSB_OK) {
        l2_read_kernel<<<grid, 512, 0, st>>>(buf, n16, 2, sink);   // warm: the buffer into L2
        for (int r = 0; r < reps && rc == PSB_OK; ++r) {
            cudaEventRecord(a, st);
            l2_read_kernel<<<grid, 512, 0, st>>>(buf, n16, passes, sink);
            cudaEventRecord(b, st);
            if ((e = cudaEventSynchronize(b)) != cudaSuccess) { rc = report_cuda(e, "psb_probe_l2_read"); break; }
            float ms = 0.f;
            cudaEventElapsedTime(&ms, a, b);
            const double g = (double)n16 * 16 * passes / (ms * 1e-3) / 1e9;
            if (g > best) best = g;
        }
    }
    if (st) cudaStreamDestroy(st);
    if (a) cudaEventDestroy(a);
    if (b) cudaEventDestroy(b);
    cudaFree(buf);
    cudaFree(sink);
    *gbs = best;
    return rc;
}
