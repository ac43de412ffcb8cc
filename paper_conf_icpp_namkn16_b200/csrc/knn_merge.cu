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
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const size_t per_warp = 32 + (KS == 0 ? (size_t)k : 0);
    u64 *scratch = reinterpret_cast<u64 *>(smem_raw) + (threadIdx.x >> 5) * per_warp;
    const int lane = threadIdx.x & 31;
    const int64_t qi = (int64_t)blockIdx.x * 4 + (threadIdx.x >> 5);
    if (qi >= nq) return;
    TopK<KS> T;
    T.init(scratch + 32, k);
    u64 thr = PAD_KEY;
    constexpr int C = KS == 0 ? 4 : KS;      // keys per lane per offer round
    for (int p = 0; p < parts; ++p) {
        const int64_t row = ((int64_t)p * nq + qi) * k;
        for (int r0 = 0; r0 < k; r0 += 32 * C) {
            u64 cand[C];
#pragma unroll
            for (int s = 0; s < C; ++s) {
                const int r = r0 + s * 32 + lane;
                cand[s] = r < k ? make_key(__ldg(dists + row + r), __ldg(ids + row + r)) : ~0ull;
            }
            T.template offer<C>(cand, k, lane, thr, scratch);
        }
    }
    T.store(k, lane, out_ids + qi * k, out_dists + qi * k);
}

// Latency-mode merge: one CTA of MP_WARPS warps per query. Only keys with dist <=
// the query's final shared pruning distance can belong to the answer (every true
// neighbour is, and few others are), so the whole [parts][k] block is first read
// at once by all threads (one L2 round trip) and the survivors are collected in
// shared memory (the per-warp lists' space); one warp then keeps the k smallest.
// If more keys survive than that space holds (ties at the bound), the per-warp
// merge below runs instead.
constexpr int MP_WARPS = 32;

template <int KS>
__global__ void __launch_bounds__(MP_WARPS * 32)
merge_parts_kernel(const int32_t *__restrict__ ids, const float *__restrict__ dists, const float *__restrict__ gpd,
                   int parts, int k, int32_t *__restrict__ out_ids, float *__restrict__ out_dists)
{
    __shared__ u64 lists[MP_WARPS][KS * 32];
    __shared__ u64 scratch_all[MP_WARPS][32];
    __shared__ int nbuf;
    constexpr int MP_BUF = MP_WARPS * KS * 32;
    u64 *const buf = &lists[0][0];                   // the fast path's survivors
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t qi = blockIdx.x;
    const float lim = __ldg(gpd + qi);
    TopK<KS> T;
    T.init();
    u64 thr = PAD_KEY;
    if (threadIdx.x == 0) nbuf = 0;
    __syncthreads();
    {
        const int total = parts * k;
        const float *dq = dists + qi * (int64_t)total;
        const int32_t *iq = ids + qi * (int64_t)total;
#pragma unroll 8
        for (int i = threadIdx.x; i < total; i += MP_WARPS * 32) {
            const float dv = __ldg(dq + i);
            if (dv <= lim) {
                const int pos = atomicAdd(&nbuf, 1);
                if (pos < MP_BUF) buf[pos] = make_key(dv, __ldg(iq + i));
            }
        }
    }
    __syncthreads();
    const int nb = nbuf;
    if (nb <= MP_BUF) {
        if (w == 0) {
            for (int c = 0; c < nb; c += 32) {
                u64 cand[1] = {c + lane < nb ? buf[c + lane] : ~0ull};
                T.template offer<1>(cand, k, lane, thr, scratch_all[0]);
            }
            T.store(k, lane, out_ids + qi * k, out_dists + qi * k);
        }
        return;
    }
    constexpr int U = 4;
    for (int p0 = w; p0 < parts; p0 += MP_WARPS * U) {
        float dv[U][KS];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int p = p0 + u * MP_WARPS;
#pragma unroll
            for (int s = 0; s < KS; ++s) {
                const int r = s * 32 + lane;
                dv[u][s] = (p < parts && r < k) ? __ldg(dists + (qi * parts + p) * (int64_t)k + r) : INFINITY;
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int p = p0 + u * MP_WARPS;
            u64 cand[KS];
            bool any = false;
#pragma unroll
            for (int s = 0; s < KS; ++s) {
                const int r = s * 32 + lane;
                const bool ok = p < parts && r < k && dv[u][s] <= lim;
                cand[s] = ok ? make_key(dv[u][s], __ldg(ids + (qi * parts + p) * (int64_t)k + r)) : ~0ull;
                any |= ok;
            }
            if (__any_sync(FULL, any)) T.template offer<KS>(cand, k, lane, thr, scratch_all[w]);
        }
    }
#pragma unroll
    for (int s = 0; s < KS; ++s) lists[w][s * 32 + lane] = T.key[s];
    __syncthreads();
    if (w == 0) {
        for (int o = 1; o < MP_WARPS; ++o) {
            u64 cand[KS];
#pragma unroll
            for (int s = 0; s < KS; ++s) cand[s] = s * 32 + lane < k ? lists[o][s * 32 + lane] : ~0ull;
            T.template offer<KS>(cand, k, lane, thr, scratch_all[0]);
        }
        T.store(k, lane, out_ids + qi * k, out_dists + qi * k);
    }
}

__global__ void fill_inf(float *__restrict__ p, int64_t n, unsigned long long *__restrict__ queue)
{
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) p[i] = INFINITY;
    if (queue && i == 0) *queue = 0ull;
}

void init_shared_pd(float *gpd, int64_t nq, unsigned long long *queue, cudaStream_t st)
{
    fill_inf<<<(unsigned)((nq + 255) / 256), 256, 0, st>>>(gpd, nq, queue);
}

// Few parts per query (split batches): one warp per query over its [parts][k]
// lists, same filter.
template <int KS>
__global__ void __launch_bounds__(128)
merge_parts_small_kernel(const int32_t *__restrict__ ids, const float *__restrict__ dists,
                         const float *__restrict__ gpd, int parts, int64_t nq, int k, int32_t *__restrict__ out_ids,
                         float *__restrict__ out_dists)
{
    __shared__ u64 scratch_all[4][32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t qi = (int64_t)blockIdx.x * 4 + w;
    if (qi >= nq) return;
    const float lim = __ldg(gpd + qi);
    TopK<KS> T;
    T.init();
    u64 thr = PAD_KEY;
    for (int p = 0; p < parts; ++p) {
        const int64_t row = (qi * parts + p) * (int64_t)k;
        u64 cand[KS];
        bool any = false;
#pragma unroll
        for (int s = 0; s < KS; ++s) {
            const int r = s * 32 + lane;
            const float dv = r < k ? __ldg(dists + row + r) : INFINITY;
            const bool ok = r < k && dv <= lim;
            cand[s] = ok ? make_key(dv, __ldg(ids + row + r)) : ~0ull;
            any |= ok;
        }
        if (__any_sync(FULL, any)) T.template offer<KS>(cand, k, lane, thr, scratch_all[w]);
    }
    T.store(k, lane, out_ids + qi * k, out_dists + qi * k);
}

int launch_merge_parts(const int32_t *ids, const float *dists, const float *gpd, int parts, int64_t nq, int k,
                       int32_t *oi, float *od, cudaStream_t st)
{
    if (parts <= 8) {
        const unsigned blocks = (unsigned)((nq + 3) / 4);
        if (k <= 32) merge_parts_small_kernel<1><<<blocks, 128, 0, st>>>(ids, dists, gpd, parts, nq, k, oi, od);
        else if (k <= 64) merge_parts_small_kernel<2><<<blocks, 128, 0, st>>>(ids, dists, gpd, parts, nq, k, oi, od);
        else merge_parts_small_kernel<4><<<blocks, 128, 0, st>>>(ids, dists, gpd, parts, nq, k, oi, od);
        return report_cuda(cudaGetLastError(), "merge_parts kernel launch");
    }
    if (k <= 32) merge_parts_kernel<1><<<(unsigned)nq, MP_WARPS * 32, 0, st>>>(ids, dists, gpd, parts, k, oi, od);
    else if (k <= 64) merge_parts_kernel<2><<<(unsigned)nq, MP_WARPS * 32, 0, st>>>(ids, dists, gpd, parts, k, oi, od);
    else merge_parts_kernel<4><<<(unsigned)nq, MP_WARPS * 32, 0, st>>>(ids, dists, gpd, parts, k, oi, od);
    return report_cuda(cudaGetLastError(), "merge_parts kernel launch");
}

int launch_merge(const int32_t *ids, const float *dists, int parts, int64_t nq, int k, int32_t *oi,
                 float *od, cudaStream_t st)
{
    const unsigned blocks = (unsigned)((nq + 3) / 4);
    const size_t s0 = 4 * 32 * 8;
    if (k <= 32) merge_kernel<1><<<blocks, 128, s0, st>>>(ids, dists, parts, nq, k, oi, od);
    else if (k <= 64) merge_kernel<2><<<blocks, 128, s0, st>>>(ids, dists, parts, nq, k, oi, od);
    else if (k <= 128) merge_kernel<4><<<blocks, 128, s0, st>>>(ids, dists, parts, nq, k, oi, od);
    else {
        const size_t sb = 4 * (32 + (size_t)k) * 8;         // NEXT-3: list in shared memory
        if (sb > 48 * 1024) {
            cudaError_t ea = cudaFuncSetAttribute(merge_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sb);
            if (ea != cudaSuccess) return report_cuda(ea, "cudaFuncSetAttribute (merge)");
        }
        merge_kernel<0><<<blocks, 128, sb, st>>>(ids, dists, parts, nq, k, oi, od);
    }
    return report_cuda(cudaGetLastError(), "merge kernel launch");
}

// Dispatch on (d, fanout): the configs' specialisations, runtime-d otherwise.
#define PSB_SPECIALISED(X) X(2, 1) X(3, 2) X(3, 4) X(8, 4) X(16, 4)

int launch_tree(int algo, const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi,
                float *od, cudaStream_t st, uint32_t variant, int64_t *stats, cudaMemPool_t pool, int parts,
                const TraceOut &tr)
{
    int rc = PSB_NOT_INSTANTIATED;
    const int V = ix.F / 32;
#define TRY(DD, VV)                                                                                  \
    if (rc == PSB_NOT_INSTANTIATED && ix.d == DD && V == VV)                                        \
        rc = launch_tree_ks<DD, VV>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool, parts, tr);
    PSB_SPECIALISED(TRY)
#undef TRY
    if (rc == PSB_NOT_INSTANTIATED) {
        switch (V) {
        case 1: rc = launch_tree_ks<0, 1>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool, parts, tr); break;
        case 2: rc = launch_tree_ks<0, 2>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool, parts, tr); break;
        case 4: rc = launch_tree_ks<0, 4>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool, parts, tr); break;
        case 8: rc = launch_tree_ks<0, 8>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool, parts, tr); break;
        case 16: rc = launch_tree_ks<0, 16>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool, parts, tr); break;
        default: break;
        }
    }
    return rc == PSB_NOT_INSTANTIATED ? PSB_EUNSUPPORTED : rc;
}

int launch_brute(const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi, float *od,
                 cudaStream_t st, int sm_count, cudaMemPool_t pool)
{
    int rc = PSB_NOT_INSTANTIATED;
    const int V = ix.F / 32;
#define TRY(DD, VV)                                                                                  \
    if (rc == PSB_NOT_INSTANTIATED && ix.d == DD && V == VV)                                        \
        rc = launch_brute_ks<DD, VV>(ix, queries, nq, k, oi, od, st, sm_count, pool);
    PSB_SPECIALISED(TRY)
#undef TRY
    if (rc == PSB_NOT_INSTANTIATED) {
        switch (V) {
        case 1: rc = launch_brute_ks<0, 1>(ix, queries, nq, k, oi, od, st, sm_count, pool); break;
        case 2: rc = launch_brute_ks<0, 2>(ix, queries, nq, k, oi, od, st, sm_count, pool); break;
        case 4: rc = launch_brute_ks<0, 4>(ix, queries, nq, k, oi, od, st, sm_count, pool); break;
        case 8: rc = launch_brute_ks<0, 8>(ix, queries, nq, k, oi, od, st, sm_count, pool); break;
        case 16: rc = launch_brute_ks<0, 16>(ix, queries, nq, k, oi, od, st, sm_count, pool); break;
        default: break;
        }
    }
    return rc == PSB_NOT_INSTANTIATED ? PSB_EUNSUPPORTED : rc;
}

}  // namespace psb
