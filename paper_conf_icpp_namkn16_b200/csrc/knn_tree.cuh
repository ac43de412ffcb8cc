#pragma once
// knn_tree.cuh — the two tree traversals on sm_100a, one warp per query:
//   psb_kernel : Parallel Scan and Backtrack (Alg. 1, §III)
//   bnb_kernel : classic branch-and-bound (Roussopoulos [17]) made
//                stackless with parent links as the paper ran it
// Step names S1..S11 follow SURVEY.md §8(a); readings R1..R16 follow DESIGN.md §2.
#include <cuda_runtime.h>

#include <cstdlib>

#include "psb_device.cuh"
#include "psb_launch.h"


namespace psb {

constexpr int WARPS_PER_CTA = 4;
// Batches are reordered by closest leaf (knn_order.cu) by default when they have
// at least this many queries and the leaves (points + ids) do not sit in L2
// anyway (profiles/r01_query_order.md: a loss at C2's 16 MB, a gain from C3's 146 MB).
constexpr int64_t REORDER_MIN_QUERIES = 1024;
constexpr double REORDER_MIN_BYTES = 64.0 * (1 << 20);
// Resident CTAs per SM the traversal kernels are compiled for (register cap
// 65536 / (128 * blocks)): 8 (<= 64 registers) measured best at d <= 8, 6 (<= 80)
// at d = 16 and for the runtime-d kernels (profiles/r01_occupancy.md).
#ifndef PSB_MINBLOCKS_SMALL_D
#define PSB_MINBLOCKS_SMALL_D 8
#endif
#ifndef PSB_MINBLOCKS_LARGE_D
#define PSB_MINBLOCKS_LARGE_D 6
#endif
// PSB prefetched the right sibling's coordinates and the scanned leaf's ids by
// default at compile-time d = 16 in round 1; covering the whole 8 KB block made it
// a loss (C4 15.3-15.5 ms without it, 16.5-16.7 with both prefetches,
// profiles/r02_experiments.md). The variant bits PSB_VAR_PREFETCH_NEXT / _IDS now
// run the runtime-d kernels, which keep the prefetch code; the compile-time-d
// kernels carry no prefetch test in their leaf step (2.5 % of the C5 slab's
// instructions, profiles/r02_experiments.md).
#ifndef PSB_REUSE_L1_MIN_D
#define PSB_REUSE_L1_MIN_D 8   // eligibility reuse in pass 2 for compile-time d >= this (psb_query)
#endif
template <int D>
struct MinBlocks {
    static constexpr int value = (D == 0 || D >= 16) ? PSB_MINBLOCKS_LARGE_D : PSB_MINBLOCKS_SMALL_D;
};

struct WarpState {
    float *cache_md;     // [(H+1)][F] child MINDISTs of the node cached per level
    int32_t *cache_node; // [(H+1)] node id cached per level (-1 = none)
    u64 *scratch;        // [32] top-k merge scratch
    u64 *list;           // [k] large-k list (KS == 0 kernels)
    float *qsmem;        // query (D == 0 only)
    unsigned pf;         // scan_leaf prefetch flags (PF_NEXT, PF_IDS)
    TraceOut tr;         // psb_knn_trace output (counting kernels only)
};

__device__ __forceinline__ WarpState warp_state(unsigned char *smem, int H, int F, bool qsmem, int kbig = 0)
{
    const int w = threadIdx.x >> 5;
    unsigned char *base = smem + (size_t)w * WarpSmem::bytes(H, F, qsmem, kbig);
    WarpState s;
    s.cache_md = reinterpret_cast<float *>(base);
    size_t off = (WarpSmem::cache_floats(H, F) * 4 + 15) & ~(size_t)15;
    s.cache_node = reinterpret_cast<int32_t *>(base + off);
    off += (size_t)(H + 1) * 4;
    off = (off + 15) & ~(size_t)15;
    s.scratch = reinterpret_cast<u64 *>(base + off);
    off += 32 * 8;
    s.list = reinterpret_cast<u64 *>(base + off);
    off += (size_t)kbig * 8;
    s.qsmem = reinterpret_cast<float *>(base + off);
    s.pf = 0;
    s.tr = TraceOut{nullptr, nullptr, 0};
    return s;
}

// S3+S4+S5 with the S7 path cache: child MINDISTs of internal node (lvl, node).
// A node already cached at its level is not fetched again: MINDIST is a pure
// function of (query, node), and its k-th-MAXDIST bound was applied when it was
// first fetched (re-applying it could not lower pd further).
template <int D, int V, bool SPH>
__device__ __forceinline__ bool internal_md(const DevIndex &ix, int lvl, int node,
                                            const Query<D> &q, int lane, const WarpState &ws,
                                            bool use_cache, bool use_max, int k, float &pd,
                                            float (&md)[V], float (&Md)[V])
{
    constexpr int F = 32 * V;
    float *cm = ws.cache_md + (size_t)lvl * F + lane * V;
    if (use_cache && ws.cache_node[lvl] == node) {
#pragma unroll
        for (int t = 0; t < V; ++t) md[t] = cm[t];
        return false;
    }
    // block size: compile-time for MBR nodes of a compile-time d
    const int64_t bf = (D > 0 && !SPH) ? 2 * D * F : ix.blk_floats;
    const float *blk = ix.nodes + ix.level_off[lvl] + (int64_t)node * bf;
    if (use_max) {
        if constexpr (SPH) sphere_bounds<D, V, true>(blk, q, ix.d, lane, md, Md);
        else node_bounds<D, V, true>(blk, q, ix.d, lane, md, Md);
        if (k <= ix.F && !(ws.pf & PF_KTH_RULE)) {
            // Alg. 1 l.13-15 with point counts (R3): every child subtree but the
            // last holds >= F >= k points, all within its MAXDIST, so the smallest
            // MAXDIST over children holding >= k points bounds d_k.
            const int lim = ix.kcnt_lim[lvl] - (node * F + lane * V);
            float m = pd;
#pragma unroll
            for (int t = 0; t < V; ++t)
                if (t <= lim) m = fminf(m, Md[t]);
            pd = warp_min_f(m);
        } else {
            pd = kth_bound<V>(Md, k, pd);                // the k-th smallest MAXDIST
        }
    } else {
        if constexpr (SPH) sphere_bounds<D, V, false>(blk, q, ix.d, lane, md, Md);
        else node_bounds<D, V, false>(blk, q, ix.d, lane, md, Md);
    }
    if (use_cache) {
#pragma unroll
        for (int t = 0; t < V; ++t) cm[t] = md[t];
        __syncwarp();
        if (lane == 0) ws.cache_node[lvl] = node;
        __syncwarp();
    }
    return true;
}

// Pass-1 child choice (S2, R4): among this node's children c in [c_lo, c_hi),
// the argmin of (MINDIST, MAXDIST, c). A query inside several overlapping boxes
// has MINDIST 0 to all of them; the smaller MAXDIST picks the box that hugs it,
// which makes ClosestLeaf, hence the initial pruning distance, much tighter
// (profiles/r01_closest_leaf.md). With index_tie the order is (MINDIST, c).
template <int V>
__device__ __forceinline__ int closest_child(const float (&md)[V], const float (&Md)[V], int c_lo, int c_hi,
                                             int lane, bool index_tie)
{
    u64 best = ~0ull;
#pragma unroll
    for (int t = 0; t < V; ++t) {
        const int cc = lane * V + t;
        const u64 kk = index_tie ? make_key(md[t], cc) : ((u64)__float_as_uint(md[t]) << 32) | __float_as_uint(Md[t]);
        if (cc >= c_lo && cc < c_hi) best = kk < best ? kk : best;
    }
    best = warp_min_u64(best);
    if (index_tie) return (int)(best & 0xffffffffu);
    unsigned mine = 0;
#pragma unroll
    for (int t = 0; t < V; ++t) {
        const int cc = lane * V + t;
        const u64 kk = ((u64)__float_as_uint(md[t]) << 32) | __float_as_uint(Md[t]);
        mine |= (unsigned)(cc >= c_lo && cc < c_hi && kk == best) << t;
    }
    const unsigned bal = __ballot_sync(FULL, mine != 0);
    const int src = __ffs(bal) - 1;
    return src * V + (__ffs(__shfl_sync(FULL, mine, src)) - 1);
}

// Last leaf under (lvl, node): min((node+1)*F^lvl, L) - 1. With span clamped at
// L and node < F*nlev[lvl], the product stays below 2L < 2^27 (n < 2^31, F >= 32).
__device__ __forceinline__ int max_leaf(const DevIndex &ix, int lvl, int node)
{
    const int e = (node + 1) * (int)ix.span[lvl];
    return (e < (int)ix.L ? e : (int)ix.L) - 1;
}

template <int F>
struct Log2 {
    static constexpr int value = F == 32 ? 5 : F == 64 ? 6 : F == 128 ? 7 : F == 256 ? 8 : 9;
};

// PSB for query qi, executed by one warp (Alg. 1 with the readings of DESIGN.md §2).
template <int D, int V, int KS, bool ST, bool SPH>
__device__ __forceinline__ void psb_query(const DevIndex &ix, const float *__restrict__ queries, int64_t qi,
                                          int k, int32_t *__restrict__ out_ids, float *__restrict__ out_dists,
                                          int64_t *__restrict__ stats, const WarpState &ws, bool use_cache,
                                          bool use_max, int lane)
{
    constexpr int F = 32 * V;
    constexpr int LOGF = Log2<F>::value;
    const int H = ix.H;

    // S1: query to registers, kNNs <- {inf} (Alg. 1 l.1-2)
    Query<D> q;
    q.load(queries + qi * ix.d, ix.d, ws.qsmem);
    for (int l = lane; l <= H; l += 32) ws.cache_node[l] = -1;
    __syncwarp();
    TopK<KS> T;
    T.init(ws.list, k);
    u64 thr = PAD_KEY;
    float pd = __int_as_float(0x7f800000);
    Stats<ST> S;

    // One loop runs both passes so that each step (node bounds, leaf scan, top-k
    // merge) is inlined once: the kernel's code size decides its instruction-cache
    // hit rate (profiles/r01_icache.md).
    //
    // S2: pass 1, getInitialPruningDistance(Q, ClosestLeaf) (Alg. 1 l.3; R4):
    // greedy descent by (MINDIST, MAXDIST, child index) argmin, k-th-MAXDIST
    // bounds on the way, to ClosestLeaf; then ClosestLeaf and the other leaves of
    // its parent N* in increasing (MINDIST, index) order while their MINDIST is
    // <= the running pruning distance (at most 32 leaves). N*'s child MINDISTs
    // were computed on the way down, so choosing them costs no fetch, and the
    // k-th distance falls fast: the initial bound is close to d_k. Their points
    // go straight into the kNN list (allowed by R4); pass 2 treats these leaves
    // as scanned without a change (R25).
    // Pass 2 (Alg. 1 l.6-47): leftmost eligible descent, left-to-right leaf scan,
    // parent-link backtrack.
    bool pass1 = true;
    const bool p1_index_tie = (ws.pf & PF_P1_INDEX_TIE) != 0;
    int lvl = H;
    int node = 0;
    // Pass-1 state lives in the path cache's unused level-0 slot (no registers
    // held across the loop): p1md[c] = MINDIST of N*'s child c, set to -1 once
    // that leaf is scanned in pass 1; `nstar` = N* (level-1 node id) once pass 1
    // is over (-1 before), so pass 2's skip test is one compare in registers.
    float *const p1md = ws.cache_md;
    int nstar = -1;                                              // N* once pass 1 is over
    int visited = -1;                                            // R10
    // Pass 2's eligibility at the current level-1 node (the node every non-changing
    // leaf returns to, Alg. 1 l.44): this lane's bits of {c < c_end : MINDIST <= pd}
    // for node enode. While the walk returns to the same node and pd has not moved,
    // the set is the same (the node is in the path cache, MINDIST is a pure function
    // of (query, node)), so the next child is the next bit above `visited` without
    // re-reading or re-testing the MINDISTs.
    // The set stays valid until pd can change: a leaf scan that changed the list, or
    // a node fetch (its MAXDIST bound); both reset enode.
    constexpr bool REUSE_L1 = D == 0 || D >= PSB_REUSE_L1_MIN_D;
    unsigned emask = 0;
    int enode = -1;
    while (true) {
        if (lvl > 0) {
            float md[V], Md[V];
            const bool fetched = internal_md<D, V, SPH>(ix, lvl, node, q, lane, ws, use_cache, use_max, k, pd, md, Md);
            if (REUSE_L1 && fetched) enode = -1;                 // pd may have fallen
            S.node(fetched);
            S.step(ws.tr, qi, lane, lvl, node, (pass1 ? TR_PASS1 : 0u) | (fetched ? TR_FETCHED : 0u));
            const int base = node * F;
            int c;
            if (pass1) {
                c = closest_child<V>(md, Md, 0, (int)ix.nlev[lvl - 1] - base, lane, p1_index_tie);
            } else {
                // S6: eligible(c) = MINDIST <= pd (R5) and unvisited leaves below (R8).
                // Subtree leaf ranges are contiguous and increasing in c, so
                // maxLeaf(child c) > visited  <=>  visited+1 < L  and
                // base + c >= (visited+1) / F^(lvl-1)   (a warp-uniform threshold).
                const int c_end = min(F, (int)ix.nlev[lvl - 1] - base);
                const int c_min = visited + 1 < (int)ix.L ? ((visited + 1) >> ((lvl - 1) * LOGF)) - base : F;
                // this lane's children lane*V+t with c_min <= c < c_end, as a bit range
                const int lo_b = min(max(c_min - lane * V, 0), V), hi_b = min(max(c_end - lane * V, 0), V);
                unsigned under = 0;
#pragma unroll
                for (int t = 0; t < V; ++t) under |= (unsigned)(md[t] <= pd) << t;
                under &= (1u << hi_b) - 1u;
                if (REUSE_L1 && lvl == 1) {                      // remembered for the next returns
                    emask = under;
                    enode = node;
                }
                const unsigned mine = under & ~((1u << lo_b) - 1u);
                const unsigned bal = __ballot_sync(FULL, mine != 0);
                c = F;
                if (bal) {                                       // leftmost (R6, R7)
                    const int src = __ffs(bal) - 1;
                    const unsigned m = __shfl_sync(FULL, mine, src);
                    c = src * V + (__ffs(m) - 1);
                }
            }
            if (c < F) {
                node = base + c;
                if (--lvl == 0 && pass1) {                       // ClosestLeaf; keep N*'s MINDISTs
#pragma unroll
                    for (int t = 0; t < V; ++t) p1md[lane * V + t] = md[t];
                    __syncwarp();
                }
            } else {                                             // S7 backtrack (R9)
                if (lvl == H) break;                             // root exhausted (R10)
                visited = max_leaf(ix, lvl, node);
                node /= F;
                ++lvl;
            }
        } else {
            // S8-S10: leaf j
            const int j = node;
            bool changed = false;
            // a pass-1 leaf is not scanned again in pass 2 (its points are in the list)
            const bool pre = (j >> LOGF) == nstar && p1md[j & (F - 1)] < 0.f;
            if (!pre) changed = scan_leaf<D, V, KS, ST>(ix, j, q, lane, T, k, thr, S, ws.scratch, ws.pf);
            if (REUSE_L1 && changed) enode = -1;                 // pd may have fallen
            S.step(ws.tr, qi, lane, 0, j, (pass1 ? TR_PASS1 : 0u) | (changed ? TR_CHANGED : 0u) | (pre ? TR_SKIPPED : 0u));
            pd = fminf(pd, key_dist(thr));                       // Alg. 1 l.37
            if (pass1) {
                const int b1 = j & ~(F - 1);                     // N*'s first leaf
                if (lane == 0) p1md[j - b1] = -1.f;              // scanned
                __syncwarp();
                // next leaf of N* in (MINDIST, index) order, if its MINDIST <= pd:
                // the smallest MINDIST bit pattern (non-negative floats order like
                // their bits) by one REDUX, then the smallest index holding it
                uint32_t mb = 0xffffffffu, mc = 0xffffffffu;
#pragma unroll
                for (int t = 0; t < V; ++t) {
                    const int cc = lane * V + t;
                    const float v = p1md[cc];
                    const uint32_t bits = (v >= 0.f && b1 + cc < (int)ix.L) ? __float_as_uint(v) : 0xffffffffu;
                    if (bits < mb) { mb = bits; mc = (uint32_t)cc; }
                }
                const uint32_t gm = __reduce_min_sync(FULL, mb);
                const uint32_t gc = __reduce_min_sync(FULL, mb == gm ? mc : 0xffffffffu);
                if (gm != 0xffffffffu && __uint_as_float(gm) <= pd) {
                    node = b1 + (int)gc;
                    continue;
                }
                pass1 = false;                                   // restart at the root
                nstar = j >> LOGF;
                lvl = H;
                node = 0;
                continue;
            }
            visited = j;                                         // l.38
            if (j == (int)ix.L - 1) break;                       // R10
            if (changed) {
                node = j + 1;                                    // l.41 right sibling (R11, R12)
            } else {
                node = j / F;                                    // l.44 parent link
                lvl = 1;
                if (REUSE_L1 && node == enode && use_cache) {
                    // the parent's visit without leaving the leaf step: the same
                    // walk as the generic step on a path-cache hit
                    S.node(false);
                    S.step(ws.tr, qi, lane, 1, node, 0u);
                    const int base = node * F;
                    const int lo_b = min(max(j + 1 - base - lane * V, 0), V);
                    const unsigned mine = emask & ~((1u << lo_b) - 1u);
                    const unsigned bal = __ballot_sync(FULL, mine != 0);
                    if (bal) {                                   // leftmost (R6, R7)
                        const int src = __ffs(bal) - 1;
                        node = base + src * V + (__ffs(__shfl_sync(FULL, mine, src)) - 1);
                        lvl = 0;
                    } else {                                     // S7 backtrack (R9)
                        if (H == 1) break;                       // root exhausted (R10)
                        visited = max_leaf(ix, 1, node);
                        node /= F;
                        lvl = 2;
                    }
                }
            }
        }
    }
    // S11
    T.store(k, lane, out_ids + qi * k, out_dists + qi * k);
    S.write(stats, ws.tr, qi, lane);
}

// Stackless B&B: at an internal node take the next child in
// (MINDIST, index) order after the one we returned from, among those with
// MINDIST <= pd; a leaf always returns to its parent.
template <int D, int V, int KS, bool ST, bool SPH>
__device__ __forceinline__ void bnb_query(const DevIndex &ix, const float *__restrict__ queries, int64_t qi,
                                          int k, int32_t *__restrict__ out_ids, float *__restrict__ out_dists,
                                          int64_t *__restrict__ stats, const WarpState &ws, bool use_cache,
                                          bool use_max, int lane)
{
    constexpr int F = 32 * V;
    const int H = ix.H;

    Query<D> q;
    q.load(queries + qi * ix.d, ix.d, ws.qsmem);
    for (int l = lane; l <= H; l += 32) ws.cache_node[l] = -1;
    __syncwarp();
    TopK<KS> T;
    T.init(ws.list, k);
    u64 thr = PAD_KEY;
    float pd = __int_as_float(0x7f800000);
    Stats<ST> S;

    int lvl = H;
    int node = 0;
    int from_c = -1;                        // child we returned from, -1 = fresh visit
    while (true) {
        if (lvl > 0) {
            float md[V], Md[V];
            const bool fetched = internal_md<D, V, SPH>(ix, lvl, node, q, lane, ws, use_cache, use_max, k, pd, md, Md);
            S.node(fetched);
            S.step(ws.tr, qi, lane, lvl, node, fetched ? TR_FETCHED : 0u);
            u64 from_key = 0;
            if (from_c >= 0) {
                float v = md[0];
#pragma unroll
                for (int t = 1; t < V; ++t)
                    if (t == from_c % V) v = md[t];
                from_key = make_key(__shfl_sync(FULL, v, from_c / V), from_c);
            }
            const int base = node * F, nb = (int)ix.nlev[lvl - 1];
            u64 best = ~0ull;
#pragma unroll
            for (int t = 0; t < V; ++t) {
                const int c = lane * V + t;
                const u64 kk = make_key(md[t], c);
                if (base + c < nb && md[t] <= pd && (from_c < 0 || kk > from_key))
                    best = kk < best ? kk : best;
            }
            best = warp_min_u64(best);
            if (best != ~0ull) {
                node = base + (int)(best & 0xffffffffu);
                --lvl;
                from_c = -1;
            } else {
                if (lvl == H) break;
                from_c = (int)(node % F);
                node /= F;
                ++lvl;
            }
        } else {
            const bool ch = scan_leaf<D, V, KS, ST>(ix, node, q, lane, T, k, thr, S, ws.scratch, ws.pf);
            S.step(ws.tr, qi, lane, 0, node, ch ? TR_CHANGED : 0u);
            pd = fminf(pd, key_dist(thr));
            from_c = (int)(node % F);
            node /= F;
            lvl = 1;
        }
    }
    T.store(k, lane, out_ids + qi * k, out_dists + qi * k);
    S.write(stats, ws.tr, qi, lane);
}


// Batch scheduling (knn_order.cu): the key of query qi is the sequence id of its
// ClosestLeaf, reached by the greedy (MINDIST, child index) descent of PSB's pass
// 1 (Alg. 1 l.3; R4). One warp per query, no cache, no MAXDIST.
template <int D, int V, bool SPH>
__global__ void __launch_bounds__(WARPS_PER_CTA * 32)
closest_leaf_kernel(DevIndex ix, const float *__restrict__ queries, int64_t nq, uint32_t *__restrict__ leaf_key,
                    bool index_tie)
{
    __shared__ float qs[WARPS_PER_CTA][D == 0 ? PSB_DMAX : 1];
    constexpr int F = 32 * V;
    const int lane = threadIdx.x & 31;
    const int64_t qi = (int64_t)blockIdx.x * WARPS_PER_CTA + (threadIdx.x >> 5);
    if (qi >= nq) return;
    Query<D> q;
    q.load(queries + qi * ix.d, ix.d, qs[threadIdx.x >> 5]);
    int node = 0;
    for (int lvl = ix.H; lvl > 0; --lvl) {
        const float *blk = ix.nodes + ix.level_off[lvl] + (int64_t)node * ix.blk_floats;
        float md[V], Md[V];
        if constexpr (SPH) sphere_bounds<D, V, true>(blk, q, ix.d, lane, md, Md);
        else node_bounds<D, V, true>(blk, q, ix.d, lane, md, Md);
        const int base = node * F;
        node = base + closest_child<V>(md, Md, 0, (int)ix.nlev[lvl - 1] - base, lane, index_tie);
    }
    if (lane == 0) leaf_key[qi] = (uint32_t)node;
}

// One warp per query. With `queue` non-null the grid is persistent (as many
// CTAs as fit on the GPU) and each warp takes the next query from an atomic
// counter when it finishes one, so a long query never holds an idle block.
#define PSB_TREE_KERNEL(NAME, BODY)                                                                  \
    template <int D, int V, int KS, bool ST, bool SPH>                                                \
    __global__ void __launch_bounds__(WARPS_PER_CTA * 32, MinBlocks<D>::value)                       \
    NAME(DevIndex ix, const float *__restrict__ queries, int64_t nq, int k,                          \
         int32_t *__restrict__ out_ids, float *__restrict__ out_dists, uint32_t variant,             \
         int64_t *__restrict__ stats, unsigned long long *__restrict__ queue,                        \
         const int32_t *__restrict__ order, TraceOut tr)                                              \
    {                                                                                                 \
        extern __shared__ __align__(16) unsigned char smem[];                                         \
        const int lane = threadIdx.x & 31;                                                            \
        WarpState ws = warp_state(smem, ix.H, 32 * V, D == 0, KS == 0 ? k : 0);                       \
        ws.tr = tr;                                                                                   \
        ws.pf = ((variant & PSB_VAR_PREFETCH_NEXT) ? PF_NEXT : 0u) |                                   \
                ((variant & PSB_VAR_PREFETCH_IDS) ? PF_IDS : 0u) |                                     \
                ((variant & PSB_VAR_P1_INDEX_TIE) ? PF_P1_INDEX_TIE : 0u) |                               \
                ((variant & PSB_VAR_KTH_MAXDIST) || ix.irregular ? PF_KTH_RULE : 0u);                     \
        const bool use_cache = !(variant & PSB_VAR_NOCACHE);                                          \
        const bool use_max = !(variant & PSB_VAR_NOMAXDIST);                                          \
        int64_t qi = (int64_t)blockIdx.x * WARPS_PER_CTA + (threadIdx.x >> 5);                        \
        while (true) {                                                                                \
            if (queue) {                                                                              \
                unsigned long long v = 0;                                                             \
                if (lane == 0) v = atomicAdd(queue, 1ull);                                            \
                qi = (int64_t)__shfl_sync(FULL, v, 0);                                                \
            }                                                                                         \
            if (qi >= nq) break;                                                                      \
            const int64_t row = order ? (int64_t)__ldg(order + qi) : qi;                             \
            BODY<D, V, KS, ST, SPH>(ix, queries, row, k, out_ids, out_dists, stats, ws, use_cache, use_max, lane); \
            if (!queue) break;                                                                        \
        }                                                                                             \
    }

PSB_TREE_KERNEL(psb_kernel, psb_query)
PSB_TREE_KERNEL(bnb_kernel, bnb_query)


// ---------------------------------------------------------------------------
// Split mode (SURVEY.md §8(e) "intra-GPU split"; psb_knn_split, and psb_knn for
// batches too small to fill the GPU): `parts` warps share one query. Part p
// owns the level-1 nodes n with n % parts == p and runs PSB (Alg. 1 with the
// readings of DESIGN.md §2) over their leaves only: at level 2 a child is
// eligible only if it is owned, and a changed leaf's right sibling is scanned
// only inside the same level-1 node (else the parent link). Interleaving the
// nodes, rather than cutting the leaves into contiguous ranges, spreads the
// eligible leaves of a query (which cluster in a few neighbouring nodes) over
// all parts. The parts share the query's pruning distance gpd[qi] through
// atomicMin on its bits (valid: every part's k-th distance and k-th-MAXDIST
// bound is an upper bound on the query's true k-th distance, and distances are
// >= +0 so their bit patterns order like the values). Each part writes its own
// sorted list; the lists are merged afterwards (merge_parts_kernel), keeping only
// keys with dist <= the final gpd. Exact: a point of the true kNN has dist <= d_k
// <= gpd at all times; its leaf belongs to one part, whose walk is never pruned
// away from it, so that part keeps it.
__device__ __forceinline__ float shared_pd(const float *g) { return __ldcg(g); }
__device__ __forceinline__ void publish_pd(float *g, float v)
{
    atomicMin(reinterpret_cast<int *>(g), __float_as_int(v));
}

// Latency mode (few queries): the leaves are cut into `parts` contiguous ranges
// and one warp runs PSB restricted to each range: children whose leaf range
// misses [lo, hi) are never eligible, `visited` starts at lo-1 and the walk ends
// when it passes hi-1. Same shared pruning distance and merge as below. With
// thousands of parts per query, short contiguous ranges balance better than
// whole interleaved nodes (C4 single query 0.25 vs 0.49 ms).
template <int D, int V, int KS, bool ST, bool SPH>
__device__ __forceinline__ void psb_range_query(const DevIndex &ix, const float *__restrict__ queries, int64_t qi,
                                               int part, int parts, int k, int32_t *__restrict__ part_ids,
                                               float *__restrict__ part_dists, float *__restrict__ gpd,
                                               const WarpState &ws, bool use_cache, bool use_max, int lane)
{
    constexpr int F = 32 * V;
    constexpr int LOGF = Log2<F>::value;
    const int H = ix.H;
    const int L = (int)ix.L;
    const int chunk = (L + parts - 1) / parts;
    const int lo = part * chunk, hi = min(lo + chunk, L);
    TopK<KS> T;
    T.init(ws.list, k);
    int32_t *oi = part_ids + (qi * parts + part) * (int64_t)k;
    float *od = part_dists + (qi * parts + part) * (int64_t)k;
    if (lo >= hi) {
        T.store(k, lane, oi, od);
        return;
    }
    float *g = gpd + qi;
    Query<D> q;
    q.load(queries + qi * ix.d, ix.d, ws.qsmem);
    for (int l = lane; l <= H; l += 32) ws.cache_node[l] = -1;
    __syncwarp();
    u64 thr = PAD_KEY;
    float pd = shared_pd(g);
    float published = pd;
    Stats<ST> S;

    // pass 1 inside the range: greedy descent among children overlapping [lo, hi)
    int lvl = H, node = 0;
    while (lvl > 0) {
        float md[V], Md[V];
        internal_md<D, V, SPH>(ix, lvl, node, q, lane, ws, use_cache, use_max, k, pd, md, Md);
        const int base = node * F, sh = (lvl - 1) * LOGF;
        const int c_lo = (lo >> sh) - base, c_hi = min((int)ix.nlev[lvl - 1] - base, ((hi - 1) >> sh) - base + 1);
        node = base + closest_child<V>(md, Md, c_lo, c_hi, lane, (ws.pf & PF_P1_INDEX_TIE) != 0);
        --lvl;
    }
    const int pass1_lo = node;
    int pass1_hi = node - 1;
    int64_t seen = 0;
    while (seen < k && pass1_hi + 1 < hi) {
        ++pass1_hi;
        scan_leaf<D, V, KS, ST>(ix, pass1_hi, q, lane, T, k, thr, S, ws.scratch, ws.pf);
        const int64_t left = ix.n - (int64_t)pass1_hi * F;
        seen += left < F ? left : F;
    }
    pd = fminf(pd, key_dist(thr));
    if (pd < published) { if (lane == 0) publish_pd(g, pd); published = pd; }

    lvl = H;
    node = 0;
    int visited = lo - 1;
    while (true) {
        if (lvl > 0) {
            float md[V], Md[V];
            const float gp = shared_pd(g);                       // issued early, used below
            internal_md<D, V, SPH>(ix, lvl, node, q, lane, ws, use_cache, use_max, k, pd, md, Md);
            pd = fminf(pd, gp);
            const int base = node * F, sh = (lvl - 1) * LOGF;
            const int c_end = min(min(F, (int)ix.nlev[lvl - 1] - base), ((hi - 1) >> sh) - base + 1);
            const int c_min = ((visited + 1) >> sh) - base;
            unsigned mine = 0;
#pragma unroll
            for (int t = 0; t < V; ++t) {
                const int c = lane * V + t;
                const bool e = c >= c_min && c < c_end && md[t] <= pd;
                mine |= (unsigned)e << t;
            }
            const unsigned bal = __ballot_sync(FULL, mine != 0);
            if (bal) {
                const int src = __ffs(bal) - 1;
                const unsigned m = __shfl_sync(FULL, mine, src);
                node = base + src * V + (__ffs(m) - 1);
                --lvl;
            } else {
                if (lvl == H) break;
                visited = max_leaf(ix, lvl, node);
                if (visited >= hi - 1) break;                    // range exhausted
                node /= F;
                ++lvl;
            }
        } else {
            const int j = node;
            bool changed;
            if (j >= pass1_lo && j <= pass1_hi) {
                changed = true;
            } else {
                changed = scan_leaf<D, V, KS, ST>(ix, j, q, lane, T, k, thr, S, ws.scratch, ws.pf);
            }
            pd = fminf(pd, key_dist(thr));
            if (pd < published) { if (lane == 0) publish_pd(g, pd); published = pd; }
            visited = j;
            if (j >= hi - 1) break;
            if (changed) {
                node = j + 1;
            } else {
                node = j / F;
                lvl = 1;
            }
        }
    }
    T.store(k, lane, oi, od);
}

// Batch mode (psb_knn_split with many queries): part p owns the level-1 nodes n
// with n % parts == p (see the comment above shared_pd).
template <int D, int V, int KS, bool ST, bool SPH>
__device__ __forceinline__ void psb_node_query(const DevIndex &ix, const float *__restrict__ queries, int64_t qi,
                                               int part, int parts, int k, int32_t *__restrict__ part_ids,
                                               float *__restrict__ part_dists, float *__restrict__ gpd,
                                               const WarpState &ws, bool use_cache, bool use_max, int lane)
{
    constexpr int F = 32 * V;
    constexpr int LOGF = Log2<F>::value;
    const int H = ix.H;
    const int L = (int)ix.L;
    TopK<KS> T;
    T.init(ws.list, k);
    int32_t *oi = part_ids + (qi * parts + part) * (int64_t)k;
    float *od = part_dists + (qi * parts + part) * (int64_t)k;
    if (H == 1 && part != 0) {                                   // one level-1 node: part 0 owns all
        T.store(k, lane, oi, od);
        return;
    }
    float *g = gpd + qi;
    Query<D> q;
    q.load(queries + qi * ix.d, ix.d, ws.qsmem);
    for (int l = lane; l <= H; l += 32) ws.cache_node[l] = -1;
    __syncwarp();
    u64 thr = PAD_KEY;
    float pd = shared_pd(g);
    float published = pd;
    Stats<ST> S;
    float *const p1md = ws.cache_md;                             // N*'s child MINDISTs (pass 1)
    bool pass1 = true;
    int nstar = -1;                                              // N* once pass 1 is over
    int lvl = H, node = 0, visited = -1;
    while (true) {
        if (lvl > 0) {
            float md[V], Md[V];
            const float gp = shared_pd(g);                       // issued early, used below
            internal_md<D, V, SPH>(ix, lvl, node, q, lane, ws, use_cache, use_max, k, pd, md, Md);
            pd = fminf(pd, gp);
            const int base = node * F;
            const int c_end = min(F, (int)ix.nlev[lvl - 1] - base);
            // this lane's children lane*V+t that exist and, at level 2, are owned
            // (child ids base+lane*V+t are consecutive: one modulo per lane)
            unsigned mine = 0;
            if (lvl == 2) {
                int r = (base + lane * V) % parts;
#pragma unroll
                for (int t = 0; t < V; ++t) {
                    mine |= (unsigned)(lane * V + t < c_end && r == part) << t;
                    r = r + 1 == parts ? 0 : r + 1;
                }
            } else {
#pragma unroll
                for (int t = 0; t < V; ++t) mine |= (unsigned)(lane * V + t < c_end) << t;
            }
            int c = F;
            if (pass1) {                                         // closest owned child (R4)
                u64 best = ~0ull;
#pragma unroll
                for (int t = 0; t < V; ++t) {
                    const u64 kk = ((u64)__float_as_uint(md[t]) << 32) | __float_as_uint(Md[t]);
                    if (((mine >> t) & 1u) && kk < best) best = kk;
                }
                best = warp_min_u64(best);
                // stop descending once the closest owned child lies beyond the shared bound
                if (best != ~0ull && __uint_as_float((uint32_t)(best >> 32)) <= pd) {
                    unsigned hit = 0;
#pragma unroll
                    for (int t = 0; t < V; ++t) {
                        const u64 kk = ((u64)__float_as_uint(md[t]) << 32) | __float_as_uint(Md[t]);
                        hit |= (unsigned)(((mine >> t) & 1u) && kk == best) << t;
                    }
                    const unsigned bal = __ballot_sync(FULL, hit != 0);
                    const int src = __ffs(bal) - 1;
                    c = src * V + (__ffs(__shfl_sync(FULL, hit, src)) - 1);
                } else {
                    pass1 = false;                               // nothing owned below: pass 2 from the root
                    lvl = H;
                    node = 0;
                    continue;
                }
            } else {
                // S6 with ownership: MINDIST <= pd, unvisited leaves below, owned at level 2
                const int c_min = visited + 1 < (int)ix.L ? ((visited + 1) >> ((lvl - 1) * LOGF)) - base : F;
                const int lo_b = min(max(c_min - lane * V, 0), V);
                unsigned el = mine & ~((1u << lo_b) - 1u);
#pragma unroll
                for (int t = 0; t < V; ++t) el &= ~((unsigned)!(md[t] <= pd) << t);
                const unsigned bal = __ballot_sync(FULL, el != 0);
                if (bal) {
                    const int src = __ffs(bal) - 1;
                    c = src * V + (__ffs(__shfl_sync(FULL, el, src)) - 1);
                }
            }
            if (c < F) {
                node = base + c;
                if (--lvl == 0 && pass1) {
#pragma unroll
                    for (int t = 0; t < V; ++t) p1md[lane * V + t] = md[t];
                    __syncwarp();
                }
            } else {                                             // S7 backtrack (R9)
                if (lvl == H) break;
                visited = max_leaf(ix, lvl, node);
                node /= F;
                ++lvl;
            }
        } else {
            const int j = node;
            bool changed = false;
            const bool pre = (j >> LOGF) == nstar && p1md[j & (F - 1)] < 0.f;
            if (!pre) changed = scan_leaf<D, V, KS, ST>(ix, j, q, lane, T, k, thr, S, ws.scratch, ws.pf);
            pd = fminf(pd, key_dist(thr));
            if (pd < published) {
                if (lane == 0) publish_pd(g, pd);
                published = pd;
            }
            if (pass1) {                                         // best-first inside N* (R25)
                const int b1 = j & ~(F - 1);
                if (lane == 0) p1md[j - b1] = -1.f;
                __syncwarp();
                pd = fminf(pd, shared_pd(g));                    // the other parts' progress
                u64 best = ~0ull;
#pragma unroll
                for (int t = 0; t < V; ++t) {
                    const int cc = lane * V + t;
                    const float v = p1md[cc];
                    const u64 kk = make_key(v, cc);
                    if (v >= 0.f && b1 + cc < L && kk < best) best = kk;
                }
                best = warp_min_u64(best);
                if (best != ~0ull && key_dist(best) <= pd) {
                    node = b1 + (int)(best & 0xffffffffu);
                    continue;
                }
                pass1 = false;
                nstar = j >> LOGF;
                lvl = H;
                node = 0;
                continue;
            }
            visited = j;
            if (j == L - 1) break;
            if (changed && ((j + 1) >> LOGF) == (j >> LOGF)) {
                node = j + 1;                                    // right sibling in the same (owned) node
            } else {
                node = j / F;                                    // parent link
                lvl = 1;
            }
        }
    }
    T.store(k, lane, oi, od);
}

// One warp per (query, part) task; with `queue` the grid is persistent and
// warps take tasks t = 0, 1, ... from an atomic counter: query order[t / parts]
// (the closest-leaf order when the batch was reordered), part t % parts.
template <int D, int V, int KS, bool ST, bool SPH, bool NODE>
__global__ void __launch_bounds__(WARPS_PER_CTA * 32, MinBlocks<D>::value)
psb_split_kernel(DevIndex ix, const float *__restrict__ queries, int64_t nq, int parts, int k,
                 int32_t *__restrict__ part_ids, float *__restrict__ part_dists, float *__restrict__ gpd,
                 uint32_t variant, unsigned long long *__restrict__ queue, const int32_t *__restrict__ order)
{
    extern __shared__ __align__(16) unsigned char smem[];
    const int lane = threadIdx.x & 31;
    WarpState ws = warp_state(smem, ix.H, 32 * V, D == 0, KS == 0 ? k : 0);
    ws.pf = ((variant & PSB_VAR_PREFETCH_NEXT) ? PF_NEXT : 0u) | ((variant & PSB_VAR_PREFETCH_IDS) ? PF_IDS : 0u) |
            ((variant & PSB_VAR_P1_INDEX_TIE) ? PF_P1_INDEX_TIE : 0u) |
            ((variant & PSB_VAR_KTH_MAXDIST) || ix.irregular ? PF_KTH_RULE : 0u);
    const int64_t tasks = nq * parts;
    int64_t t = (int64_t)blockIdx.x * WARPS_PER_CTA + (threadIdx.x >> 5);
    while (true) {
        if (queue) {
            unsigned long long v = 0;
            if (lane == 0) v = atomicAdd(queue, 1ull);
            t = (int64_t)__shfl_sync(FULL, v, 0);
        }
        if (t >= tasks) break;
        const int64_t qpos = t / parts;
        const int64_t qi = order ? (int64_t)__ldg(order + qpos) : qpos;
        if constexpr (NODE)
            psb_node_query<D, V, KS, ST, SPH>(ix, queries, qi, (int)(t % parts), parts, k, part_ids, part_dists, gpd,
                                              ws, !(variant & PSB_VAR_NOCACHE), !(variant & PSB_VAR_NOMAXDIST), lane);
        else
            psb_range_query<D, V, KS, ST, SPH>(ix, queries, qi, (int)(t % parts), parts, k, part_ids, part_dists, gpd,
                                               ws, !(variant & PSB_VAR_NOCACHE), !(variant & PSB_VAR_NOMAXDIST), lane);
        if (!queue) break;
    }
}

template <int D, int V, int KS>
static int launch_tree_t(int algo, const DevIndex &ix0, const float *queries, int64_t nq, int k,
                         int32_t *oi, float *od, cudaStream_t st, uint32_t variant, int64_t *stats,
                         cudaMemPool_t pool, int parts, const TraceOut &tr)
{
    const size_t smem = WARPS_PER_CTA * WarpSmem::bytes(ix0.H, 32 * V, D == 0, KS == 0 ? k : 0);
    int64_t blocks = (nq + WARPS_PER_CTA - 1) / WARPS_PER_CTA;
    // per-launch view: the count-aware MAXDIST bound's child limit per level (R3)
    DevIndex ix = ix0;
    for (int l = 1; l <= ix.H; ++l) {
        const int64_t lastc = ix.nlev[l - 1] - 1;
        const bool last_ok = ix.n - lastc * ix.span[l - 1] * ix.F >= k;
        ix.kcnt_lim[l] = (int32_t)(last_ok ? lastc : lastc - 1);
    }
    // Counting kernels (stats / trace) are instantiated for the generic-d path
    // and for the compile-time-d MBR kernels, so the counters of a timed
    // configuration come from the same instantiation as its timed kernel
    // (PSB_VAR_GENERIC_D selects the generic one; tests compare the two).
    const bool counting = stats != nullptr || tr.len != nullptr;
    using Kern = void (*)(DevIndex, const float *, int64_t, int, int32_t *, float *, uint32_t, int64_t *,
                          unsigned long long *, const int32_t *, TraceOut);
    Kern kern;
    const bool psbk = algo == PSB_ALGO_PSB;
    if constexpr (D == 0) {
        if (ix.sphere)
            kern = psbk ? (counting ? psb_kernel<D, V, KS, true, true> : psb_kernel<D, V, KS, false, true>)
                        : (counting ? bnb_kernel<D, V, KS, true, true> : bnb_kernel<D, V, KS, false, true>);
        else
            kern = psbk ? (counting ? psb_kernel<D, V, KS, true, false> : psb_kernel<D, V, KS, false, false>)
                        : (counting ? bnb_kernel<D, V, KS, true, false> : bnb_kernel<D, V, KS, false, false>);
    } else {
        if (counting && ix.sphere) return PSB_NOT_INSTANTIATED;
        if (counting) kern = psbk ? psb_kernel<D, V, KS, true, false> : bnb_kernel<D, V, KS, true, false>;
        else if (ix.sphere) kern = psbk ? psb_kernel<D, V, KS, false, true> : bnb_kernel<D, V, KS, false, true>;
        else kern = psbk ? psb_kernel<D, V, KS, false, false> : bnb_kernel<D, V, KS, false, false>;
    }
    cudaError_t e;
    if (smem > 48 * 1024) {
        e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return report_cuda(e, "cudaFuncSetAttribute");
    }
    // Batch scheduling: process the queries in the order of their closest leaf
    // (knn_order.cu) so concurrent warps share leaves in L1/L2. Rows are written
    // to their input positions, so results are unchanged.
    int32_t *order = nullptr;
    const double leaf_bytes = (double)ix.L * ix.F * (ix.d * 4 + 4);
    const bool reorder = (variant & PSB_VAR_LEAF_ORDER) ||
                         (!(variant & PSB_VAR_INPUT_ORDER) && nq >= REORDER_MIN_QUERIES && leaf_bytes >= REORDER_MIN_BYTES);
    // At low d the Hilbert key of the query orders the batch better and costs no
    // node reads (C5 slab: 9.76 -> 9.09 ms with a host-side Hilbert sort; at C3
    // and C4 the closest-leaf order is as good or better, profiles/r02cs, r02ct);
    // PSB_VAR_LEAF_ORDER keeps the closest-leaf order.
    if (reorder && ix.d <= PSB_HILBERT_ORDER_MAX_D && !(variant & PSB_VAR_LEAF_ORDER) && ix.box) {
        if ((e = cudaMallocFromPoolAsync((void **)&order, (size_t)nq * 4, pool, st)) != cudaSuccess)
            return report_cuda(e, "cudaMallocFromPoolAsync (query order)");
        const int rc = hilbert_query_order(queries, nq, ix.d, ix.box, order, pool, st);
        if (rc != PSB_OK) {
            cudaFreeAsync(order, st);
            return rc;
        }
    } else if (reorder) {
        uint32_t *leaf_key = nullptr;
        if ((e = cudaMallocFromPoolAsync((void **)&leaf_key, (size_t)nq * 4, pool, st)) != cudaSuccess ||
            (e = cudaMallocFromPoolAsync((void **)&order, (size_t)nq * 4, pool, st)) != cudaSuccess) {
            if (leaf_key) cudaFreeAsync(leaf_key, st);
            return report_cuda(e, "cudaMallocFromPoolAsync (query order)");
        }
        auto ck = ix.sphere ? closest_leaf_kernel<D, V, true> : closest_leaf_kernel<D, V, false>;
        ck<<<(unsigned)((nq + WARPS_PER_CTA - 1) / WARPS_PER_CTA), WARPS_PER_CTA * 32, 0, st>>>(
            ix, queries, nq, leaf_key, (variant & PSB_VAR_P1_INDEX_TIE) != 0);
        int rc = report_cuda(cudaGetLastError(), "closest-leaf kernel launch");
        if (rc == PSB_OK) rc = sort_query_order(leaf_key, nq, ix.L, order, pool, st);
        cudaFreeAsync(leaf_key, st);
        if (rc != PSB_OK) {
            cudaFreeAsync(order, st);
            return rc;
        }
    }
    if (parts > 1 && algo == PSB_ALGO_PSB && !counting && KS != 0) {
        // split mode: q*parts (query, part) tasks, shared pd per query, then a filtered merge
        // whole interleaved level-1 nodes when the (query, part) tasks fill the GPU
        // (a batch's tail), contiguous leaf ranges otherwise (single-query latency)
        using SK = void (*)(DevIndex, const float *, int64_t, int, int, int32_t *, float *, float *, uint32_t,
                            unsigned long long *, const int32_t *);
        SK skn = ix.sphere ? psb_split_kernel<D, V, KS, false, true, true> : psb_split_kernel<D, V, KS, false, false, true>;
        SK skr = ix.sphere ? psb_split_kernel<D, V, KS, false, true, false> : psb_split_kernel<D, V, KS, false, false, false>;
        int sper = cached_occupancy((const void *)skn, WARPS_PER_CTA * 32, smem);
        if (sper < 1) sper = 1;
        const int64_t tasks = nq * parts;
        const int64_t resident = (int64_t)sper * ix.sm_count * WARPS_PER_CTA;
        const SK sk = tasks >= resident ? skn : skr;
        if (smem > 48 * 1024 && (e = cudaFuncSetAttribute(sk, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) !=
                                    cudaSuccess) {
            if (order) cudaFreeAsync(order, st);
            return report_cuda(e, "cudaFuncSetAttribute");
        }
        // one scratch allocation: [queue u64][gpd nq][ids cnt][dists cnt]
        const size_t cnt = (size_t)nq * parts * k;
        const size_t o_gpd = 16, o_ids = (o_gpd + (size_t)nq * 4 + 15) & ~(size_t)15;
        const size_t o_d = (o_ids + cnt * 4 + 15) & ~(size_t)15;
        unsigned char *scratch = nullptr;
        if ((e = cudaMallocFromPoolAsync((void **)&scratch, o_d + cnt * 4, pool, st)) != cudaSuccess) {
            if (order) cudaFreeAsync(order, st);
            return report_cuda(e, "cudaMallocFromPoolAsync (split scratch)");
        }
        unsigned long long *squeue = reinterpret_cast<unsigned long long *>(scratch);
        float *gpd = reinterpret_cast<float *>(scratch + o_gpd);
        int32_t *pi = reinterpret_cast<int32_t *>(scratch + o_ids);
        float *pdist = reinterpret_cast<float *>(scratch + o_d);
        int64_t sblocks = (tasks + WARPS_PER_CTA - 1) / WARPS_PER_CTA;
        const bool persistent = sblocks * WARPS_PER_CTA > resident;
        if (persistent) sblocks = resident / WARPS_PER_CTA;
        init_shared_pd(gpd, nq, persistent ? squeue : nullptr, st);   // +inf per query, queue 0
        sk<<<(unsigned)sblocks, WARPS_PER_CTA * 32, smem, st>>>(ix, queries, nq, parts, k, pi, pdist, gpd, variant,
                                                                 persistent ? squeue : nullptr, order);
        int rc = report_cuda(cudaGetLastError(), "split kernel launch");
        if (rc == PSB_OK) rc = launch_merge_parts(pi, pdist, gpd, parts, nq, k, oi, od, st);
        cudaFreeAsync(scratch, st);
        if (order) cudaFreeAsync(order, st);
        return rc;
    }
    // More queries than resident warps: persistent grid + atomic query queue.
    const int per_sm = cached_occupancy((const void *)kern, WARPS_PER_CTA * 32, smem);
    unsigned long long *queue = nullptr;
    if (per_sm > 0 && blocks > (int64_t)per_sm * ix.sm_count) {
        if ((e = cudaMallocFromPoolAsync((void **)&queue, sizeof(unsigned long long), pool, st)) != cudaSuccess) {
            if (order) cudaFreeAsync(order, st);
            return report_cuda(e, "cudaMallocFromPoolAsync (query queue)");
        }
        if ((e = cudaMemsetAsync(queue, 0, sizeof(unsigned long long), st)) != cudaSuccess) {
            cudaFreeAsync(queue, st);
            if (order) cudaFreeAsync(order, st);
            return report_cuda(e, "cudaMemsetAsync (query queue)");
        }
        blocks = (int64_t)per_sm * ix.sm_count;
    }
    cudaGetLastError();
    kern<<<(unsigned)blocks, WARPS_PER_CTA * 32, smem, st>>>(ix, queries, nq, k, oi, od, variant, stats, queue,
                                                             order, tr);
    int rc = report_cuda(cudaGetLastError(), "tree kernel launch");
    if (queue) cudaFreeAsync(queue, st);
    if (order) cudaFreeAsync(order, st);
    return rc;
}

template <int D, int V>
int launch_tree_ks(int algo, const DevIndex &ix, const float *queries, int64_t nq, int k,
                          int32_t *oi, float *od, cudaStream_t st, uint32_t variant, int64_t *stats,
                         cudaMemPool_t pool, int parts, const TraceOut &tr)
{
    // the prefetch variants run the runtime-d kernels (see PSB_VAR_PREFETCH_* above)
    if (D > 0 && (variant & (PSB_VAR_GENERIC_D | PSB_VAR_PREFETCH_NEXT | PSB_VAR_PREFETCH_IDS)))
        return PSB_NOT_INSTANTIATED;
    if (k <= 32) return launch_tree_t<D, V, 1>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool, parts, tr);
    if (k <= 64) return launch_tree_t<D, V, 2>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool, parts, tr);
    if constexpr (D == 0) {
        if (k <= 128) return launch_tree_t<D, V, 4>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool, parts, tr);
        return launch_tree_t<D, V, 0>(algo, ix, queries, nq, k, oi, od, st, variant, stats, pool, parts, tr);  // NEXT-3
    }
    return PSB_NOT_INSTANTIATED;   // k > 64: generic-d kernels (keeps compile time down)
}

}  // namespace psb
