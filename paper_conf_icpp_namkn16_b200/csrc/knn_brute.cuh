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

#include <algorithm>
#include <cstdlib>

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

// Brute force staged through shared memory (compile-time d, k <= 64). A CTA of
// BS_WARPS warps scores BS_WARPS * QW queries against a chunk of leaves: the
// leaf blocks stream through a BS_STAGES-deep shared-memory ring filled with
// cp.async (16-byte LDGSTS by all threads, one commit group per leaf, one
// barrier per leaf), so every point is read from L2 once per CTA instead of once
// per warp, and its latency hides behind the scoring of the previous leaves. Lane l scores its V points of
// the leaf against the warp's QW queries, whose coordinates sit in shared memory
// as packed (q, q) pairs (one broadcast LDS.64 per query and dimension); each
// (point pair, dimension) costs one packed subtract, square and add (FADD2 /
// FFMA2 with the -0 addend / FADD2), the minimum for the RN distance.
constexpr int BS_WARPS = 8;
constexpr int BS_STAGES = 3;
#ifndef PSB_BS_PACKED_SUM
#define PSB_BS_PACKED_SUM 1     // running sums as FADD2 pairs (1) or scalar FADD (0)
#endif

__device__ __forceinline__ void cp_async16(void *smem_dst, const void *gmem_src)
{
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem_dst);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(s), "l"(gmem_src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

template <int D, int V>
struct BruteSmem {
    static constexpr int F = 32 * V;
    static constexpr size_t leaf_floats = (size_t)D * F;
    static constexpr size_t bytes(int qw)
    {
        return BS_STAGES * leaf_floats * 4 + (size_t)BS_WARPS * qw * D * 8 + (size_t)BS_WARPS * 32 * 8;
    }
};

template <int D, int V, int KS, int QW>
__global__ void __launch_bounds__(BS_WARPS * 32)
brute_smem_kernel(DevIndex ix, const float *__restrict__ queries, int64_t nq, int k, int64_t leaves_per_chunk,
                  int32_t *__restrict__ out_ids, float *__restrict__ out_dists)
{
    constexpr int F = 32 * V;
    constexpr int LEAF = D * F;
    extern __shared__ __align__(16) unsigned char smem[];
    float *stage = reinterpret_cast<float *>(smem);                         // [BS_STAGES][D][F]
    u64 *qpair = reinterpret_cast<u64 *>(stage + BS_STAGES * LEAF);         // [BS_WARPS * QW][D]
    u64 *scratch_all = qpair + BS_WARPS * QW * D;                           // [BS_WARPS][32]
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t cq0 = (int64_t)blockIdx.x * BS_WARPS * QW;
    for (int i = threadIdx.x; i < BS_WARPS * QW * D; i += blockDim.x) {
        int64_t qi = cq0 + i / D;
        qi = qi < nq ? qi : nq - 1;                                        // clamp: duplicates are never stored
        const float v = __ldg(queries + qi * D + i % D);
        qpair[i] = f2_pack(v, v);
    }
    const int64_t l0 = (int64_t)blockIdx.y * leaves_per_chunk;
    const int64_t l1 = l0 + leaves_per_chunk < ix.L ? l0 + leaves_per_chunk : ix.L;
    auto issue = [&](int64_t leaf, int st) {
        if (leaf < l1) {
            const float *src = ix.pts + leaf * LEAF;
            float *dst = stage + st * LEAF;
            for (int o = threadIdx.x * 4; o < LEAF; o += BS_WARPS * 32 * 4) cp_async16(dst + o, src + o);
        }
        cp_async_commit();                                                 // one group per leaf, empty at the end
    };
#pragma unroll
    for (int st = 0; st < BS_STAGES - 1; ++st) issue(l0 + st, st);

    const int64_t q0 = cq0 + (int64_t)w * QW;
    const bool active = q0 < nq;
    const u64 *myq = qpair + (size_t)w * QW * D;
    u64 *scratch = scratch_all + w * 32;
    TopK<KS> T[QW];
    u64 thr[QW];
#pragma unroll
    for (int i = 0; i < QW; ++i) { T[i].init(); thr[i] = PAD_KEY; }

    int st = 0;
    for (int64_t leaf = l0; leaf < l1; ++leaf) {
        cp_async_wait<BS_STAGES - 2>();                                    // this leaf's group has landed
        __syncthreads();            // ... for every thread's copies; and every warp is done with the last stage
        issue(leaf + BS_STAGES - 1, st == 0 ? BS_STAGES - 1 : st - 1);    // refill the stage read last round
        if (active) {
            const float *lp = stage + st * LEAF + lane * V;
            float dist[QW][V];
#pragma unroll
            for (int j = 0; j < D; ++j) {
                float p[V];
                if constexpr (V == 4) {
                    const float4 x = *reinterpret_cast<const float4 *>(lp + j * F);
                    p[0] = x.x; p[1] = x.y; p[2] = x.z; p[3] = x.w;
                } else if constexpr (V == 2) {
                    const float2 x = *reinterpret_cast<const float2 *>(lp + j * F);
                    p[0] = x.x; p[1] = x.y;
                } else {
#pragma unroll
                    for (int t = 0; t < V; ++t) p[t] = lp[j * F + t];
                }
#pragma unroll
                for (int i = 0; i < QW; ++i) {
                    const u64 qq = myq[i * D + j];
                    if constexpr (V % 2 == 0) {
#pragma unroll
                        for (int t = 0; t < V; t += 2)
                            f2_acc_sq<PSB_BS_PACKED_SUM != 0>(dist[i][t], dist[i][t + 1],
                                                              f2_sub(f2_pack(p[t], p[t + 1]), qq), j == 0);
                    } else {
                        float qa, qb;
                        f2_unpack(qq, qa, qb);
#pragma unroll
                        for (int t = 0; t < V; ++t) {
                            const float x = sq_diff(p[t], qa);
                            dist[i][t] = j == 0 ? x : __fadd_rn(dist[i][t], x);
                        }
                    }
                }
            }
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
        st = st + 1 == BS_STAGES ? 0 : st + 1;
    }
    cp_async_wait<0>();
    const int64_t part = (int64_t)blockIdx.y * nq;
#pragma unroll
    for (int i = 0; i < QW; ++i)
        if (q0 + i < nq) T[i].store(k, lane, out_ids + (part + q0 + i) * k, out_dists + (part + q0 + i) * k);
}

template <int D, int V, int KS>
static int launch_brute_smem(const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi, float *od,
                             cudaStream_t st, int sm_count, cudaMemPool_t pool)
{
    constexpr int QW = 4;
    const int64_t blocks_q = (nq + BS_WARPS * QW - 1) / (BS_WARPS * QW);
    const size_t smem = BruteSmem<D, V>::bytes(QW);
    auto kern = brute_smem_kernel<D, V, KS, QW>;
    cudaError_t e;
    if (smem > 48 * 1024 && (e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) !=
                                cudaSuccess)
        return report_cuda(e, "cudaFuncSetAttribute (brute smem)");
    int per_sm = cached_occupancy((const void *)kern, BS_WARPS * 32, smem);
    if (per_sm < 1) per_sm = 1;
    // Split the leaves into S chunks. A small batch (too few CTAs to fill the GPU
    // twice with chunks of >= 2048 leaves: single-query latency) gets about two
    // CTAs per slot, chunks down to 8 leaves. A large batch gets chunks of >= 2048
    // leaves, and since every CTA then does the same work, the launch takes
    // ceil(blocks / slots) waves of equal length: take the smallest S whose waves
    // are >= 90 % full on average (at least two waves' worth of CTAs), else the
    // fullest up to S = 64. More chunks cost partial lists and a longer merge, so
    // the threshold is not higher. C4 (313 query blocks on 296 slots): round 1's
    // "two CTAs per slot" rule gave S = 2, 2.11 waves with a third wave of 34 CTAs
    // (22 % achieved occupancy), 317 ms; S = 6 takes 279 ms, S = 12 286 ms,
    // S = 24 293 ms (profiles/r02bh).
    const int64_t slots = (int64_t)sm_count * per_sm;
    const int64_t smax_big = std::min<int64_t>(ix.L / 2048, 64);
    const int64_t smax = std::max<int64_t>(1, std::min<int64_t>((ix.L + 7) / 8, 1024));
    int64_t S = 1;
    if (blocks_q * smax_big < 2 * slots) {
        S = std::min<int64_t>(smax, (2 * slots + blocks_q - 1) / blocks_q);
    } else {
        double best = -1.0;
        for (int64_t c = 1; c <= smax_big; ++c) {
            const int64_t blocks = blocks_q * c;
            const int64_t waves = (blocks + slots - 1) / slots;
            const double eff = (double)blocks / ((double)waves * slots);
            if (blocks >= 2 * slots && eff >= 0.90) { S = c; break; }
            if (eff > best + 1e-9) { S = c; best = eff; }
        }
    }
    if (const char *ev = getenv("PSB_BRUTE_CHUNKS")) S = std::max<int64_t>(1, std::min<int64_t>(atoll(ev), smax));   // A/B
    const int64_t per = (ix.L + S - 1) / S;
    S = (ix.L + per - 1) / per;
    int32_t *pi = oi;
    float *pd = od;
    if (S > 1) {
        if ((e = cudaMallocFromPoolAsync((void **)&pi, sizeof(int32_t) * (size_t)(S * nq * k), pool, st)) != cudaSuccess)
            return report_cuda(e, "cudaMallocAsync (brute scratch)");
        if ((e = cudaMallocFromPoolAsync((void **)&pd, sizeof(float) * (size_t)(S * nq * k), pool, st)) != cudaSuccess) {
            cudaFreeAsync(pi, st);
            return report_cuda(e, "cudaMallocAsync (brute scratch)");
        }
    }
    kern<<<dim3((unsigned)blocks_q, (unsigned)S), BS_WARPS * 32, smem, st>>>(ix, queries, nq, k, per, pi, pd);
    int rc = report_cuda(cudaGetLastError(), "brute smem kernel launch");
    if (S > 1) {
        if (rc == PSB_OK) rc = launch_merge(pi, pd, (int)S, nq, k, oi, od, st);
        cudaFreeAsync(pi, st);
        cudaFreeAsync(pd, st);
    }
    return rc;
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
    if constexpr (D > 0) {                    // compile-time d: the shared-memory kernel
        if (k <= 32) return launch_brute_smem<D, V, 1>(ix, queries, nq, k, oi, od, st, sm, pool);
        if (k <= 64) return launch_brute_smem<D, V, 2>(ix, queries, nq, k, oi, od, st, sm, pool);
        return PSB_NOT_INSTANTIATED;          // k > 64: generic-d kernels
    }
    if (k <= 32) return launch_brute_t<D, V, 1>(ix, queries, nq, k, oi, od, st, sm, pool);
    if (k <= 64) return launch_brute_t<D, V, 2>(ix, queries, nq, k, oi, od, st, sm, pool);
    if constexpr (D == 0) {
        if (k <= 128) return launch_brute_t<D, V, 4>(ix, queries, nq, k, oi, od, st, sm, pool);
        return launch_brute_t<D, V, 0>(ix, queries, nq, k, oi, od, st, sm, pool);   // NEXT-3
    }
    return PSB_NOT_INSTANTIATED;   // k > 64: generic-d kernels
}

}  // namespace psb
