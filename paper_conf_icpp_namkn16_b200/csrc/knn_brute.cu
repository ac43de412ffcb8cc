// knn_brute.cu — GPU brute-force kNN (the paper's exhaustive baseline, PAPER.md
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
    float *qs = reinterpret_cast<float *>(smem) + (size_t)w * QW * PSB_DMAX;

    Query<D> q[QW];
#pragma unroll
    for (int i = 0; i < QW; ++i) {
        const int64_t qi = q0 + i < nq ? q0 + i : nq - 1;   // clamp: duplicates are never stored
        q[i].load(queries + qi * d, d, qs + i * PSB_DMAX);
    }
    TopK<KS> T[QW];
    u64 thr[QW];
#pragma unroll
    for (int i = 0; i < QW; ++i) { T[i].init(); thr[i] = PAD_KEY; }

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
            for (int i = 0; i < QW; ++i) {
                const float qj = q[i][j];
#pragma unroll
                for (int t = 0; t < V; ++t) dist[i][t] = __fadd_rn(dist[i][t], sq_diff(p[t], qj));
            }
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
                T[i].template offer<V>(cand, k, lane, thr[i]);
            }
        }
    }
    const int64_t part = (int64_t)blockIdx.y * nq;
#pragma unroll
    for (int i = 0; i < QW; ++i)
        if (q0 + i < nq) T[i].store(k, lane, out_ids + (part + q0 + i) * k, out_dists + (part + q0 + i) * k);
}

template <int KS>
__global__ void __launch_bounds__(128)
merge_kernel(const int32_t *__restrict__ ids, const float *__restrict__ dists, int parts, int64_t nq,
             int k, int32_t *__restrict__ out_ids, float *__restrict__ out_dists)
{
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
        T.template offer<KS>(cand, k, lane, thr);
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

template <int D, int V, int KS>
static int launch_brute_t(const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi,
                          float *od, cudaStream_t st, int sm_count)
{
    constexpr int QW = KS >= 4 ? 2 : 4;
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
    const size_t smem = D == 0 ? (size_t)BF_WARPS * QW * PSB_DMAX * 4 : 0;
    int32_t *pi = oi;
    float *pd = od;
    if (S > 1) {
        cudaError_t e = cudaMallocAsync((void **)&pi, sizeof(int32_t) * (size_t)(S * nq * k), st);
        if (e != cudaSuccess) return report_cuda(e, "cudaMallocAsync (brute scratch)");
        e = cudaMallocAsync((void **)&pd, sizeof(float) * (size_t)(S * nq * k), st);
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
static int launch_brute_ks(const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi,
                           float *od, cudaStream_t st, int sm)
{
    if (k <= 32) return launch_brute_t<D, V, 1>(ix, queries, nq, k, oi, od, st, sm);
    if (k <= 64) return launch_brute_t<D, V, 2>(ix, queries, nq, k, oi, od, st, sm);
    return launch_brute_t<D, V, 4>(ix, queries, nq, k, oi, od, st, sm);
}

template <int D>
static int launch_brute_v(const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi,
                          float *od, cudaStream_t st, int sm)
{
    switch (ix.F) {
    case 32: return launch_brute_ks<D, 1>(ix, queries, nq, k, oi, od, st, sm);
    case 64: return launch_brute_ks<D, 2>(ix, queries, nq, k, oi, od, st, sm);
    case 128: return launch_brute_ks<D, 4>(ix, queries, nq, k, oi, od, st, sm);
    default: break;
    }
    if constexpr (D == 0) {
        if (ix.F == 256) return launch_brute_ks<0, 8>(ix, queries, nq, k, oi, od, st, sm);
        if (ix.F == 512) return launch_brute_ks<0, 16>(ix, queries, nq, k, oi, od, st, sm);
        return PSB_EUNSUPPORTED;
    } else {
        return launch_brute_v<0>(ix, queries, nq, k, oi, od, st, sm);
    }
}

int launch_brute(const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi, float *od,
                 cudaStream_t st, int sm_count)
{
    switch (ix.d) {
    case 2: return launch_brute_v<2>(ix, queries, nq, k, oi, od, st, sm_count);
    case 3: return launch_brute_v<3>(ix, queries, nq, k, oi, od, st, sm_count);
    case 8: return launch_brute_v<8>(ix, queries, nq, k, oi, od, st, sm_count);
    case 16: return launch_brute_v<16>(ix, queries, nq, k, oi, od, st, sm_count);
    default: return launch_brute_v<0>(ix, queries, nq, k, oi, od, st, sm_count);
    }
}

}  // namespace psb
