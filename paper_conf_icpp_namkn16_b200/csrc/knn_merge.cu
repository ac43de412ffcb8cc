// knn_merge.cu — k-way merge of sorted per-part (dist, id) lists: the step after
// the data-sharded all-gather and the second stage of a
// chunked brute-force scan.
#include <cuda_runtime.h>

#include "psb_device.cuh"
#include "psb_launch.h"

namespace psb {

template <int KS>
__global__ void __launch_bounds__(128)
merge_kernel(const int32_t *__restrict__ ids, const float *__restrict__ dists, int parts, int64_t nq,
             int k, int32_t *__restrict__ out_ids, float *__restrict__ out_dists)
{
    __shared__ u64 scratch_all[4 * 32];
    u64 *scratch = scratch_all + (threadIdx.x >> 5) * 32;
    const int lane = threadIdx.x & 31;
    const int64_t qi = (int64_t)blockIdx.x * 4 + (threadIdx.x >> 5);
    if (qi >= nq) return;
    TopK<KS> T;
#pragma unroll
    for (int s = 0; s < KS; ++s) {
        const int r = s * 32 + lane;
        T.key[s] = r < k ? make_key(__ldg(dists + qi * k + r), __ldg(ids + qi * k + r)) : PAD_KEY;
    }
    u64 thr = T.kth(k);
    for (int p = 1; p < parts; ++p) {
        const int64_t row = ((int64_t)p * nq + qi) * k;
        u64 cand[KS];
#pragma unroll
        for (int s = 0; s < KS; ++s) {
            const int r = s * 32 + lane;
            cand[s] = r < k ? make_key(__ldg(dists + row + r), __ldg(ids + row + r)) : ~0ull;
        }
        T.template offer<KS>(cand, k, lane, thr, scratch);
    }
    T.store(k, lane, out_ids + qi * k, out_dists + qi * k);
}

int launch_merge(const int32_t *ids, const float *dists, int parts, int64_t nq, int k, int32_t *oi,
                 float *od, cudaStream_t st)
{
    const unsigned blocks = (unsigned)((nq + 3) / 4);
    if (k <= 32) merge_kernel<1><<<blocks, 128, 0, st>>>(ids, dists, parts, nq, k, oi, od);
    else if (k <= 64) merge_kernel<2><<<blocks, 128, 0, st>>>(ids, dists, parts, nq, k, oi, od);
    else merge_kernel<4><<<blocks, 128, 0, st>>>(ids, dists, parts, nq, k, oi, od);
    return report_cuda(cudaGetLastError(), "merge kernel launch");
}

// Dispatch on d: specialised instantiations for the configs' d, runtime-d otherwise.
int launch_tree(int algo, const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi,
                float *od, cudaStream_t st, uint32_t variant, int64_t *stats, cudaMemPool_t pool)
{
    int rc = PSB_NOT_INSTANTIATED;
    switch (ix.d) {
    case 2: rc = launch_tree_v<2>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool); break;
    case 3: rc = launch_tree_v<3>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool); break;
    case 8: rc = launch_tree_v<8>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool); break;
    case 16: rc = launch_tree_v<16>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool); break;
    default: break;
    }
    if (rc == PSB_NOT_INSTANTIATED) rc = launch_tree_v<0>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool);
    return rc == PSB_NOT_INSTANTIATED ? PSB_EUNSUPPORTED : rc;
}

int launch_brute(const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi, float *od,
                 cudaStream_t st, int sm_count, cudaMemPool_t pool)
{
    int rc = PSB_NOT_INSTANTIATED;
    switch (ix.d) {
    case 2: rc = launch_brute_v<2>(ix, queries, nq, k, oi, od, st, sm_count, pool); break;
    case 3: rc = launch_brute_v<3>(ix, queries, nq, k, oi, od, st, sm_count, pool); break;
    case 8: rc = launch_brute_v<8>(ix, queries, nq, k, oi, od, st, sm_count, pool); break;
    case 16: rc = launch_brute_v<16>(ix, queries, nq, k, oi, od, st, sm_count, pool); break;
    default: break;
    }
    if (rc == PSB_NOT_INSTANTIATED) rc = launch_brute_v<0>(ix, queries, nq, k, oi, od, st, sm_count, pool);
    return rc == PSB_NOT_INSTANTIATED ? PSB_EUNSUPPORTED : rc;
}

}  // namespace psb
