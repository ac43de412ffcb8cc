// psb_probe.cu — measured memory ceilings for the rooflines bench.py reports
// (SURVEY.md §8(d) "which roofline binds": at C2-C5 the traversal's node and
// leaf blocks are served mostly from L2, so the ceiling that bounds their
// algorithmic bytes is the L2 read bandwidth, measured here on the same GPU in
// the same run instead of a guide figure).
#include <cuda_runtime.h>

#include "psb_launch.h"

namespace psb {

// Every thread streams loads over its grid-strided share of the buffer, `passes`
// times, with U independent loads in flight; W = 16 (ld.global.cg.v4.b32) or 32
// bytes (ld.global.cg.v8.b32, sm_100). .cg caches in L2 only, so no pass is served
// from L1 and every byte crosses the L2 -> SM path; the xor keeps the loads alive.
// Round 2 measured one 16-byte load per thread at 15.3 TB/s, four in flight at
// 18.4 TB/s and one 32-byte load at 19.4 TB/s on the same B200 (64 MiB,
// tools/micro_l2.cu, profiles/r02cf): the probe reports the best of its shapes, so
// the roofline's ceiling is what the L2 can deliver, not what one load shape gets.
template <int W, int U>
__global__ void __launch_bounds__(512) l2_read_kernel(const uint4 *__restrict__ buf, int64_t n16, int passes,
                                                      unsigned *__restrict__ sink)
{
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t n = n16 / (W / 16);                  // W-byte elements
    unsigned acc = 0;
    for (int p = 0; p < passes; ++p) {
        int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
        for (; i + (U - 1) * stride < n; i += U * stride) {
            unsigned r[U][W / 4];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint4 *a = buf + (i + u * stride) * (W / 16);
                if constexpr (W == 32) {
                    asm volatile("ld.global.cg.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                                 : "=r"(r[u][0]), "=r"(r[u][1]), "=r"(r[u][2]), "=r"(r[u][3]), "=r"(r[u][4]),
                                   "=r"(r[u][5]), "=r"(r[u][6]), "=r"(r[u][7])
                                 : "l"(a));
                } else {
                    const uint4 v = __ldcg(a);
                    r[u][0] = v.x; r[u][1] = v.y; r[u][2] = v.z; r[u][3] = v.w;
                }
            }
#pragma unroll
            for (int u = 0; u < U; ++u)
#pragma unroll
                for (int w = 0; w < W / 4; ++w) acc ^= r[u][w];
        }
        for (; i < n; i += stride) {
            const uint4 v = __ldcg(buf + i * (W / 16));
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
    using K = void (*)(const uint4 *, int64_t, int, unsigned *);
    const K shapes[] = {l2_read_kernel<16, 1>, l2_read_kernel<16, 4>, l2_read_kernel<32, 1>, l2_read_kernel<32, 2>};
    for (K kern : shapes) {
        if (rc != PSB_OK) break;
        kern<<<grid, 512, 0, st>>>(buf, n16, 2, sink);   // warm: the buffer into L2
        for (int r = 0; r < reps && rc == PSB_OK; ++r) {
            cudaEventRecord(a, st);
            kern<<<grid, 512, 0, st>>>(buf, n16, passes, sink);
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
