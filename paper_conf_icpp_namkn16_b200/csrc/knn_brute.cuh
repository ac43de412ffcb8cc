#pragma once
// knn_brute.cuh — GPU brute-force kNN (the paper's exhaustive baseline, PAPER.md
// P:L79-84 §I, §V-D) and the k-way merge of sorted per-part lists
// (data-sharded mode; also the second stage of a chunked scan).
//
// Brute force uses the index's leaf-blocked SoA point array (every point exactly
// once, pad slots at +inf) and the same binary32 distance as the traversals, so
// all three algorithms return bit-identical rows. No GEMM expansion
// (|x|^2 - 2x.y + |y|^2 rounds differently and would break bit-exactness).
#include <cuda_runtime.h>

#include "psb_device.cuh"
#include "psb_launch.h"

namespace psb {

constexpr int BF_WARPS = 4;

// One warp scores QW queries against leaves [l0, l1): each leaf row is loaded
// once and used for all QW queries.
template <int D, int V, int KS, int QW>
__global__ void __launch_bounds__(BF_WARPS * 32)
brute_kernel(DevIndex ix, const float *__restrict__ queries, int64_t nq, int k, int64_t leaves_per_chunk,
             int32_t *__restrict__ out_ids, float *__restrict__ out_dists)
{
    constexpr int F = 32 * V;
    extern __shared__ __align__(16) unsigned char smem[];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t q0 = ((int64_t)blockIdx.x * BF_WARPS + w) * QW;
    if (q0 >= nq) return;
    const int d = ix.d;
    // per warp: 32-key merge scratch, then (large k) QW lists of k keys; queries after all warps
    const size_t per_warp = 32 + (KS == 0 ? (size_t)QW * k : 0);
    u64 *scratch = reinterpret_cast<u64 *>(smem) + (size_t)w * per_warp;
    u64 *lists = scratch + 32;
    float *qs = reinterpret_cast<float *>(smem + BF_WARPS * per_warp * 8) + (size_t)w * QW * PSB_DMAX;

    Query<D> q[QW];
#pragma unroll
    for (int i = 0; i < QW; ++i) {
        const int64_t qi = q0 + i < nq ? q0 + i : nq - 1;   // clamp: duplicates are never stored
        q[i].load(queries + qi * d, d, qs + i * PSB_DMAX);
    }
    TopK<KS> T[QW];
    u64 thr[QW];
#pragma unroll
    for (int i = 0; i < QW; ++i) { T[i].init(lists + (size_t)i * k, k); thr[i] = PAD_KEY; }

    const int64_t l0 = (int64_t)blockIdx.y * leaves_per_chunk;
    const int64_t l1 = l0 + leaves_per_chunk < ix.L ? l0 + leaves_per_chunk : ix.L;
    for (int64_t leaf = l0; leaf < l1; ++leaf) {
        const float *lp = ix.pts + leaf * (int64_t)d * F + lane * V;
        float dist[QW][V];
#pragma unroll
        for (int i = 0; i < QW; ++i)
#pragma unroll
            for (int t = 0; t < V; ++t) dist[i][t] = 0.f;
        for_dims<D>(d, [&](int j) {
            float p[V];
            ldv<V>(lp + j * F, p);
#pragma unroll
            for (int i = 0; i < QW; ++i) acc_sq_diff<V, PackedSum<D>::value>(dist[i], p, q[i][j], j == 0);
        });
        const int32_t *lid = ix.ids + leaf * F + lane * V;
#pragma unroll
        for (int i = 0; i < QW; ++i) {
            const float td = key_dist(thr[i]);
            bool any = false;
#pragma unroll
            for (int t = 0; t < V; ++t) any |= dist[i][t] <= td;
            if (__any_sync(FULL, any)) {
                u64 cand[V];
#pragma unroll
                for (int t = 0; t < V; ++t)
                    cand[t] = dist[i][t] <= td ? make_key(dist[i][t], __ldg(lid + t)) : ~0ull;
                T[i].template offer<V>(cand, k, lane, thr[i], scratch);
            }
        }
    }
    const int64_t part = (int64_t)blockIdx.y * nq;
#pragma unroll
    for (int i = 0; i < QW; ++i)
        if (q0 + i < nq) T[i].store(k, lane, out_ids + (part + q0 + i) * k, out_dists + (part + q0 + i) * k);
}

template <int D, int V, int KS>
static int launch_brute_t(const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi,
                          float *od, cudaStream_t st, int sm_count, cudaMemPool_t pool)
{
    constexpr int QW = KS == 0 ? 1 : (KS >= 4 ? 2 : 4);
    const int64_t warps_q = (nq + QW - 1) / QW;
    const int64_t blocks_q = (warps_q + BF_WARPS - 1) / BF_WARPS;
    // enough warps to cover ~48 per SM; chunks never smaller than 4 leaves
    int64_t S = ((int64_t)sm_count * 48 + warps_q - 1) / warps_q;
    const int64_t smax = (ix.L + 3) / 4;
    if (S > smax) S = smax;
    if (S > 1024) S = 1024;
    if (S < 1) S = 1;
    const int64_t per = (ix.L + S - 1) / S;
    S = (ix.L + per - 1) / per;
    const size_t smem = BF_WARPS * (32 + (KS == 0 ? (size_t)QW * k : 0)) * 8 +
                        (D == 0 ? (size_t)BF_WARPS * QW * PSB_DMAX * 4 : 0);
    if (smem > 48 * 1024) {
        cudaError_t ea = cudaFuncSetAttribute(brute_kernel<D, V, KS, QW>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                              (int)smem);
        if (ea != cudaSuccess) return report_cuda(ea, "cudaFuncSetAttribute (brute)");
    }
    int32_t *pi = oi;
    float *pd = od;
    if (S > 1) {
        cudaError_t e = cudaMallocFromPoolAsync((void **)&pi, sizeof(int32_t) * (size_t)(S * nq * k), pool, st);
        if (e != cudaSuccess) return report_cuda(e, "cudaMallocAsync (brute scratch)");
        e = cudaMallocFromPoolAsync((void **)&pd, sizeof(float) * (size_t)(S * nq * k), pool, st);
        if (e != cudaSuccess) { cudaFreeAsync(pi, st); return report_cuda(e, "cudaMallocAsync (brute scratch)"); }
    }
    dim3 grid((unsigned)blocks_q, (unsigned)S);
    brute_kernel<D, V, KS, QW><<<grid, BF_WARPS * 32, smem, st>>>(ix, queries, nq, k, per, pi, pd);
    int rc = report_cuda(cudaGetLastError(), "brute kernel launch");
    if (S > 1) {
        if (rc == PSB_OK) rc = launch_merge(pi, pd, (int)S, nq, k, oi, od, st);
        cudaFreeAsync(pi, st);
        cudaFreeAsync(pd, st);
    }
    return rc;
}

template <int D, int V>
int launch_brute_ks(const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi,
                           float *od, cudaStream_t st, int sm, cudaMemPool_t pool)
{
    if (k <= 32) return launch_brute_t<D, V, 1>(ix, queries, nq, k, oi, od, st, sm, pool);
    if (k <= 64) return launch_brute_t<D, V, 2>(ix, queries, nq, k, oi, od, st, sm, pool);
    if constexpr (D == 0) {
        if (k <= 128) return launch_brute_t<D, V, 4>(ix, queries, nq, k, oi, od, st, sm, pool);
        return launch_brute_t<D, V, 0>(ix, queries, nq, k, oi, od, st, sm, pool);   // NEXT-3
    }
    return PSB_NOT_INSTANTIATED;   // k > 64: generic-d kernels
}

}  // namespace psb
