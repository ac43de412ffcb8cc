// psb_device.cuh — warp-level building blocks of the sm_100a kNN kernels.
//
// One warp owns one query. For a node (or leaf) of fanout F = 32*V, lane l owns
// the V consecutive children (points) l*V .. l*V+V-1, so each SoA row of F
// floats is read by the warp as one fully coalesced 128-bit (V=4), 64-bit (V=2)
// or 32-bit (V=1) load per lane ("SoA so that memory coalescing can be naturally
// employed", §V-A; "parfor tid <- 1, numChildNodes",
// Alg. 1 l.9-12).
//
// Arithmetic is binary32 with every operation explicitly rounded to nearest
// (__fsub_rn/__fmul_rn/__fadd_rn: never contracted to FMA, never flushed to
// zero), dimensions in order — the distance the oracle defines.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "psb_internal.h"

namespace psb {

typedef unsigned long long u64;
#ifndef PSB_INSERT_MAX
#define PSB_INSERT_MAX 2   // up to this many candidates are inserted one by one, more are merged
#endif
// With a one-segment list (KS = 1, k <= 32) a 32-key merge is cheap enough that
// only a single candidate is inserted (C5 slab 9.63 -> 9.39 ms, C2/C3 unchanged;
// C4's two-segment list is faster with 2: profiles/r01ak/ins.txt).
#ifndef PSB_INSERT_MAX_KS1
#define PSB_INSERT_MAX_KS1 1
#endif
// Sizes of the candidate sorting network in TopK::offer (code size vs work):
// 3 = 8 / 16 / 32 candidates, 2 = 8 / 32, 1 = 32 only.
#ifndef PSB_MERGE_SIZES
#define PSB_MERGE_SIZES 3
#endif
constexpr unsigned FULL = 0xffffffffu;
enum : unsigned { PF_NEXT = 1u, PF_IDS = 2u, PF_P1_INDEX_TIE = 4u, PF_KTH_RULE = 8u };   // per-launch traversal flags
// (dist, id) packed as one u64 key: for dist >= +0 the IEEE bit pattern orders
// like the value, so u64 order == lexicographic (dist, id) order for ids >= 0.
// The pad (+inf, -1) = 0x7F800000FFFFFFFF is larger than every real key.
constexpr u64 PAD_KEY = 0x7F800000FFFFFFFFull;

__device__ __forceinline__ u64 make_key(float d, int32_t id)
{
    return ((u64)__float_as_uint(d) << 32) | (u64)(uint32_t)id;
}
__device__ __forceinline__ float key_dist(u64 k) { return __uint_as_float((uint32_t)(k >> 32)); }
__device__ __forceinline__ int32_t key_id(u64 k) { return (int32_t)(uint32_t)(k & 0xffffffffu); }

// (a - b)^2, each op rounded once.
__device__ __forceinline__ float sq_diff(float a, float b)
{
    float t = __fsub_rn(a, b);
    return __fmul_rn(t, t);
}

// Packed binary32 pairs (sm_100 FADD2 / FFMA2): each half is rounded exactly as
// the scalar op. ptxas 12.9 contracts a mul.rn.f32x2 that feeds an
// add.rn.f32x2 into FFMA2 even with --fmad=false, which would break the RN
// contract. So the square is written as fma.rn.f32x2(x, x, -0) with the -0 pair
// read from constant memory, which ptxas cannot fold: RN(x*x + -0) = RN(x*x)
// bit for bit (x*x >= +0, and +0 + -0 = +0 under RN), and an fma feeding an add
// cannot be contracted further. The running sums are then packed add.rn.f32x2.
// tests/test_abi_host.py checks that the only FFMA2 in the SASS are squares
// (both multiplicands the same register) with a uniform-register (constant) addend.
static __constant__ u64 c_neg_zero2 = 0x8000000080000000ull;
__device__ __forceinline__ u64 f2_pack(float a, float b)
{
    u64 r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
    return r;
}
__device__ __forceinline__ void f2_unpack(u64 r, float &a, float &b)
{
    asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(r));
}
__device__ __forceinline__ u64 f2_sub(u64 a, u64 b)
{
    u64 r;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ u64 f2_add(u64 a, u64 b)
{
    u64 r;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
// x*x per half, rounded once (see above)
__device__ __forceinline__ u64 f2_sq(u64 a)
{
    u64 r;
    asm("fma.rn.f32x2 %0, %1, %1, %2;" : "=l"(r) : "l"(a), "l"(c_neg_zero2));
    return r;
}
__device__ __forceinline__ u64 f2_mul(u64 a, u64 b)
{
    u64 r;
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
// Packed running sums pay off where the kernels are issue bound (d <= 8). At
// d = 16 (C4, bound by the latency of its longest queries) the scalar sums
// measured faster (C4 PSB 17.05 -> 18.2 ms with packed sums, profiles/r01_packed_sums.md).
#ifndef PSB_PACKED_SUM_MAXD
#define PSB_PACKED_SUM_MAXD 8
#endif
template <int D>
struct PackedSum {
    static constexpr bool value = D == 0 || D <= PSB_PACKED_SUM_MAXD;
};
// s = first ? x*x : s + x*x per half (first: fl(+0 + y) = y for y >= +0);
// PS: packed FADD2 sum, else FMUL2 square and scalar sums.
template <bool PS = true>
__device__ __forceinline__ void f2_acc_sq(float &s0, float &s1, u64 x, bool first)
{
    if constexpr (PS) {
        const u64 y = f2_sq(x);
        f2_unpack(first ? y : f2_add(f2_pack(s0, s1), y), s0, s1);
    } else {
        float a, b;
        f2_unpack(f2_mul(x, x), a, b);
        s0 = first ? a : __fadd_rn(s0, a);
        s1 = first ? b : __fadd_rn(s1, b);
    }
}
// dist[t] += (p[t] - q)^2 for V points, pairs packed when V is even.
// first: dimension 0, where fl(+0 + x) = x for the square x >= +0, so the sum
// starts at the square (no FADD; bit-identical).
template <int V, bool PS = true>
__device__ __forceinline__ void acc_sq_diff(float (&dist)[V], const float (&p)[V], float qj, bool first = false)
{
    if constexpr (V % 2 == 0) {
        const u64 qq = f2_pack(qj, qj);
#pragma unroll
        for (int t = 0; t < V; t += 2) {
            f2_acc_sq<PS>(dist[t], dist[t + 1], f2_sub(f2_pack(p[t], p[t + 1]), qq), first);
        }
    } else {
#pragma unroll
        for (int t = 0; t < V; ++t) {
            const float x = sq_diff(p[t], qj);
            dist[t] = first ? x : __fadd_rn(dist[t], x);
        }
    }
}

// Loop over dimensions 0..d-1 in order: fully unrolled for a compile-time D (so
// query coordinates stay in registers), a runtime loop otherwise.
template <int D, typename Body>
__device__ __forceinline__ void for_dims(int d, Body &&body)
{
    if constexpr (D > 0) {
#pragma unroll
        for (int j = 0; j < D; ++j) body(j);
    } else {
#pragma unroll 2
        for (int j = 0; j < d; ++j) body(j);
    }
}

// V consecutive floats, V*4-byte aligned, read-only path.
template <int V>
__device__ __forceinline__ void ldv(const float *__restrict__ p, float (&o)[V])
{
    if constexpr (V == 1) {
        o[0] = __ldg(p);
    } else if constexpr (V == 2) {
        float2 x = __ldg(reinterpret_cast<const float2 *>(p));
        o[0] = x.x; o[1] = x.y;
    } else {
#pragma unroll
        for (int i = 0; i < V; i += 4) {
            float4 x = __ldg(reinterpret_cast<const float4 *>(p + i));
            o[i] = x.x; o[i + 1] = x.y; o[i + 2] = x.z; o[i + 3] = x.w;
        }
    }
}

// Query coordinates: registers for a compile-time D, shared memory otherwise.
template <int D>
struct Query {
    float c[D];
    __device__ __forceinline__ void load(const float *__restrict__ q, int, float *)
    {
#pragma unroll
        for (int j = 0; j < D; ++j) c[j] = __ldg(q + j);
    }
    __device__ __forceinline__ float operator[](int j) const { return c[j]; }
};
template <>
struct Query<0> {
    const float *s;
    __device__ __forceinline__ void load(const float *__restrict__ q, int d, float *smem)
    {
        for (int j = threadIdx.x & 31; j < d; j += 32) smem[j] = __ldg(q + j);
        __syncwarp();
        s = smem;
    }
    __device__ __forceinline__ float operator[](int j) const { return s[j]; }
};

// S4: MINDIST and MAXDIST of the query to this lane's V child
// MBRs of one node block [d][2][F] (Alg. 1 l.9-12, §III).
//   MINDIST term: lo-q if q<lo, q-hi if q>hi, else 0;  MAXDIST term: max(|q-lo|,|q-hi|)
// Empty slots (lo=+inf, hi=-inf) give +inf for both.
//   With a = fl(lo - q) and c = fl(hi - q) (RN keeps the sign of the exact
//   difference, and fl(q - hi) = -c exactly): MINDIST term = max(a, -c, 0),
//   MAXDIST term = max(|a|, |c|), bit for bit the case analysis above. For even
//   V the differences and the squares run as packed FADD2 / FMUL2 pairs over two
//   children, the squares as FFMA2 with a -0 addend and the sums as FADD2 (see f2_sq).
template <int D, int V, bool MAX>
__device__ __forceinline__ void node_bounds(const float *__restrict__ blk, const Query<D> &q, int d,
                                            int lane, float (&md)[V], float (&Md)[V])
{
    constexpr int F = 32 * V;
#pragma unroll
    for (int t = 0; t < V; ++t) { md[t] = 0.f; Md[t] = 0.f; }
    for_dims<D>(d, [&](int j) {
        float lo[V], hi[V];
        ldv<V>(blk + (2 * j) * F + lane * V, lo);
        ldv<V>(blk + (2 * j + 1) * F + lane * V, hi);
        const float qj = q[j];
        if constexpr (V % 2 == 0) {
            const u64 qq = f2_pack(qj, qj);
#pragma unroll
            for (int t = 0; t < V; t += 2) {
                float a0, a1, c0, c1;
                f2_unpack(f2_sub(f2_pack(lo[t], lo[t + 1]), qq), a0, a1);
                f2_unpack(f2_sub(f2_pack(hi[t], hi[t + 1]), qq), c0, c1);
                const float m0 = fmaxf(fmaxf(a0, -c0), 0.f), m1 = fmaxf(fmaxf(a1, -c1), 0.f);
                f2_acc_sq<PackedSum<D>::value>(md[t], md[t + 1], f2_pack(m0, m1), j == 0);
                if (MAX) {
                    const float x0 = fmaxf(fabsf(a0), fabsf(c0)), x1 = fmaxf(fabsf(a1), fabsf(c1));
                    f2_acc_sq<PackedSum<D>::value>(Md[t], Md[t + 1], f2_pack(x0, x1), j == 0);
                }
            }
        } else {
#pragma unroll
            for (int t = 0; t < V; ++t) {
                const float a = __fsub_rn(lo[t], qj);   // lo - q
                const float c = __fsub_rn(hi[t], qj);   // hi - q  (q - hi = -c exactly)
                const float tm = fmaxf(fmaxf(a, -c), 0.f);
                md[t] = __fadd_rn(md[t], __fmul_rn(tm, tm));
                if (MAX) {
                    const float tx = fmaxf(fabsf(a), fabsf(c));
                    Md[t] = __fadd_rn(Md[t], __fmul_rn(tx, tx));
                }
            }
        }
    });
}

// S4 for the SS-tree variant (NEXT-2; §II-C, L499-504 §III):
// child bounding spheres, block [d+1][F] = centroid rows then the radius row.
// A sphere's MINDIST/MAXDIST need a square root, so unlike the MBR bounds they
// cannot ride on monotone RN rounding; they are made safe explicitly:
//   |q_j - c_j| rounded toward zero / away from zero, squares and sums rounded
//   down / up, sqrt down / up, (sqrt - r) down, (sqrt + r) up, squared down / up,
//   then scaled by (1 -/+ (2d+4) 2^-24), which covers the relative error of the
//   RN point distance (recursive sum of d+2 rounded terms; R24).
// So MINDIST <= dist_fl(q, p) <= MAXDIST for every point p inside the sphere,
// which is all the exactness argument of §2 needs. Empty slots (centre +inf,
// radius 0) give +inf for both.
template <int D, int V, bool MAX>
__device__ __forceinline__ void sphere_bounds(const float *__restrict__ blk, const Query<D> &q, int d, int lane,
                                              float (&md)[V], float (&Md)[V])
{
    constexpr int F = 32 * V;
    float lo2[V], hi2[V];
#pragma unroll
    for (int t = 0; t < V; ++t) { lo2[t] = 0.f; hi2[t] = 0.f; }
    for_dims<D>(d, [&](int j) {
        float c[V];
        ldv<V>(blk + j * F + lane * V, c);
        const float qj = q[j];
#pragma unroll
        for (int t = 0; t < V; ++t) {
            const float a = fabsf(__fsub_rz(qj, c[t]));
            lo2[t] = __fadd_rd(lo2[t], __fmul_rd(a, a));
            if (MAX) {
                const float b = fmaxf(__fsub_ru(qj, c[t]), __fsub_ru(c[t], qj));
                hi2[t] = __fadd_ru(hi2[t], __fmul_ru(b, b));
            }
        }
    });
    if (!MAX) {
#pragma unroll
        for (int t = 0; t < V; ++t) Md[t] = 0.f;   // defined for callers that read it (closest_child)
    }
    float r[V];
    ldv<V>(blk + d * F + lane * V, r);
    const float g = __fmul_ru((float)(2 * d + 4), 5.9604644775390625e-8f);   // (2d+4) 2^-24
    const float shrink = __fsub_rd(1.0f, g), grow = __fadd_ru(1.0f, g);
#pragma unroll
    for (int t = 0; t < V; ++t) {
        const float dm = fmaxf(__fsub_rd(__fsqrt_rd(lo2[t]), r[t]), 0.0f);
        md[t] = __fmul_rd(__fmul_rd(dm, dm), shrink);
        if (MAX) {
            const float dx = __fadd_ru(__fsqrt_ru(hi2[t]), r[t]);
            Md[t] = __fmul_ru(__fmul_ru(dx, dx), grow);
        }
    }
}

// S8: distances of the query to this lane's V points of one leaf block [d][F].
template <int D, int V>
__device__ __forceinline__ void leaf_dists(const float *__restrict__ lp, const Query<D> &q, int d,
                                           int lane, float (&dist)[V])
{
    constexpr int F = 32 * V;
#pragma unroll
    for (int t = 0; t < V; ++t) dist[t] = 0.f;
    for_dims<D>(d, [&](int j) {
        float p[V];
        ldv<V>(lp + j * F + lane * V, p);
        acc_sq_diff<V, PackedSum<D>::value>(dist, p, q[j], j == 0);
    });
}

// Warp minimum of a float v >= +0 (or +inf, never NaN or -0): non-negative
// binary32 values order like their bit patterns, so one REDUX.MIN on the bits
// replaces a 5-step shuffle tree.
__device__ __forceinline__ float warp_min_f(float v)
{
    return __uint_as_float(__reduce_min_sync(FULL, __float_as_uint(v)));
}

// Warp minimum of a u64 key: the high words first, then the low words among
// the lanes holding that high word (two REDUX.MIN).
__device__ __forceinline__ u64 warp_min_u64(u64 v)
{
    const uint32_t hi = __reduce_min_sync(FULL, (uint32_t)(v >> 32));
    const uint32_t lo = __reduce_min_sync(FULL, (uint32_t)(v >> 32) == hi ? (uint32_t)v : 0xffffffffu);
    return ((u64)hi << 32) | lo;
}

// S5: k-th smallest of the warp's F MAXDIST values if it is below `pd`, else pd
// (Alg. 1 l.13-15 parReduceFindKthMinMaxDist). The k-th smallest
// MAXDIST over k non-empty disjoint children bounds the k-th NN distance.
// Cheap filter first: fewer than k values below pd cannot lower pd. Otherwise a
// 31-step radix select on the (non-negative) float bit patterns.
template <int V>
__device__ __forceinline__ float kth_bound(const float (&Md)[V], int k, float pd)
{
    int c = 0;
#pragma unroll
    for (int t = 0; t < V; ++t) c += Md[t] < pd;
    c = __reduce_add_sync(FULL, c);
    if (c < k) return pd;
    uint32_t res = 0;
#pragma unroll 1
    for (int bit = 30; bit >= 0; --bit) {
        const uint32_t trial = res | (1u << bit);
        int n = 0;
#pragma unroll
        for (int t = 0; t < V; ++t) n += __float_as_uint(Md[t]) < trial;
        n = __reduce_add_sync(FULL, n);
        if (n < k) res = trial;
    }
    return __uint_as_float(res);
}

// Warp bitonic network on one u64 key per lane: sort ascending by lane, and the
// final merge stage alone (a bitonic sequence -> ascending).
__device__ __forceinline__ u64 cmpx(u64 v, int j, bool take_min)
{
    const u64 o = __shfl_xor_sync(FULL, v, j);
    // one u64 compare and one select (o == v only for equal fillers: either is right)
    return (o < v) == take_min ? o : v;
}
// Sorts each group of G lanes (G = 8, 16 or 32; groups alternate direction).
// With candidates in lanes 0..G-1 and ~0 everywhere else, the whole warp is
// then ascending.
template <int G = 32>
__device__ __forceinline__ u64 warp_sort32(u64 v, int lane)
{
#pragma unroll
    for (int kk = 2; kk <= G; kk <<= 1) {
        const bool asc = (lane & kk) == 0;
#pragma unroll
        for (int j = kk >> 1; j > 0; j >>= 1) v = cmpx(v, j, ((lane & j) == 0) == asc);
    }
    return v;
}
__device__ __forceinline__ u64 warp_merge32(u64 v, int lane)
{
#pragma unroll
    for (int j = 16; j > 0; j >>= 1) v = cmpx(v, j, (lane & j) == 0);
    return v;
}

// Warp-distributed sorted top-k of u64 keys (S9; the paper keeps "the kNN list
// and k pruning distances" in shared memory; here they live in
// registers): position r = s*32 + lane holds the r-th smallest key, KS keys per
// lane, k <= 32*KS. Positions >= k are scratch.
template <int KS>
struct TopK {
    u64 key[KS];

    __device__ __forceinline__ void init()
    {
#pragma unroll
        for (int s = 0; s < KS; ++s) key[s] = PAD_KEY;
    }
    __device__ __forceinline__ void init(u64 *, int) { init(); }
    // key at position k-1 (the current k-th neighbour), warp-uniform
    __device__ __forceinline__ u64 kth(int k) const
    {
        const int s = (k - 1) >> 5;
        u64 v = key[0];
#pragma unroll
        for (int i = 1; i < KS; ++i)
            if (i == s) v = key[i];
        return __shfl_sync(FULL, v, (k - 1) & 31);
    }
    // insert warp-uniform x (x not already present); everything above shifts up
    __device__ __forceinline__ void insert(u64 x, int lane)
    {
        int p = 0;
#pragma unroll
        for (int s = 0; s < KS; ++s) p += __popc(__ballot_sync(FULL, key[s] < x));
        u64 prev[KS];
#pragma unroll
        for (int s = 0; s < KS; ++s) {
            u64 up = __shfl_up_sync(FULL, key[s], 1);
            u64 wrap = s ? __shfl_sync(FULL, key[s > 0 ? s - 1 : 0], 31) : x;
            prev[s] = lane ? up : wrap;
        }
#pragma unroll
        for (int s = 0; s < KS; ++s) {
            const int r = s * 32 + lane;
            key[s] = r > p ? prev[s] : (r == p ? x : key[s]);
        }
    }
    // Merge 32 candidate keys (one per lane, ~0 = none) into the list: sort them
    // with a warp bitonic network, then for each 32-key segment of the list take
    // the elementwise min/max against the reversed candidates (the 32 smallest /
    // largest of the union, each a bitonic sequence) and re-sort both halves;
    // the larger half carries into the next segment, the last one is dropped.
    template <int G = 32>
    __device__ __forceinline__ void merge32(u64 c, int lane)
    {
        c = warp_sort32<G>(c, lane);
#pragma unroll
        for (int s = 0; s < KS; ++s) {
            const u64 rc = __shfl_sync(FULL, c, 31 - lane);
            const u64 lo = rc < key[s] ? rc : key[s];
            const u64 hi = rc < key[s] ? key[s] : rc;
            key[s] = warp_merge32(lo, lane);
            if (s + 1 < KS) c = warp_merge32(hi, lane);
        }
    }
    // Offer this lane's V candidate keys (~0 = none); returns how many were below
    // the k-th key (> 0 iff the first k positions changed). `thr` is the k-th key, kept current. Few candidates
    // are inserted one by one; more are compacted through `scratch` (32 u64 of
    // per-warp shared memory) and merged 32 at a time.
    template <int V>
    __device__ __forceinline__ int offer(const u64 (&cand)[V], int k, int lane, u64 &thr, u64 *scratch)
    {
        // Code size matters here (the kernels are instruction-cache bound at
        // small d, profiles/r01_icache.md): every insertion / merge network below
        // has exactly one inlined copy per call site of offer().
        unsigned bal[V];
        int m = 0;
#pragma unroll
        for (int t = 0; t < V; ++t) {
            bal[t] = __ballot_sync(FULL, cand[t] < thr);
            m += __popc(bal[t]);
        }
        if (m == 0) return 0;
        if (m <= (KS == 1 ? PSB_INSERT_MAX_KS1 : PSB_INSERT_MAX)) {
            for (int i = 0; i < m; ++i) {                // (t, lane) order; warp-uniform
                int t0 = 0;                                  // first t with a pending candidate
                unsigned b = bal[0];
#pragma unroll
                for (int t = V - 1; t >= 0; --t)
                    if (bal[t]) { t0 = t; b = bal[t]; }
                const int src = __ffs(b) - 1;
                u64 v = cand[0];
#pragma unroll
                for (int t = 1; t < V; ++t)
                    if (t == t0) v = cand[t];
#pragma unroll
                for (int t = 0; t < V; ++t)
                    if (t == t0) bal[t] &= bal[t] - 1;
                const u64 x = __shfl_sync(FULL, v, src);
                if (x < thr) {
                    insert(x, lane);
                    thr = kth(k);
                }
            }
            return m;
        }
        // Compact the candidates in (t, lane) order through 32 u64 of scratch and
        // merge them 32 at a time (m <= 32*V). A candidate that is no longer below
        // the k-th key after an earlier round only lands at positions >= k.
        const unsigned lt = (1u << lane) - 1;
        for (int r = 0; r < m; r += 32) {
            int base = -r;
#pragma unroll
            for (int t = 0; t < V; ++t) {
                const int i = base + __popc(bal[t] & lt);
                if ((bal[t] >> lane & 1u) && i >= 0 && i < 32) scratch[i] = cand[t];
                base += __popc(bal[t]);
            }
            __syncwarp();
            const int n = min(m - r, 32);
            const u64 c = lane < n ? scratch[lane] : ~0ull;
            __syncwarp();
#if PSB_MERGE_SIZES == 1
            merge32<32>(c, lane);
#elif PSB_MERGE_SIZES == 2
            if (n <= 8) merge32<8>(c, lane);
            else merge32<32>(c, lane);
#else
            if (n <= 8) merge32<8>(c, lane);
            else if (n <= 16) merge32<16>(c, lane);
            else merge32<32>(c, lane);
#endif
        }
        thr = kth(k);
        return m;
    }
    __device__ __forceinline__ void store(int k, int lane, int32_t *__restrict__ oi,
                                          float *__restrict__ od) const
    {
#pragma unroll
        for (int s = 0; s < KS; ++s) {
            const int r = s * 32 + lane;
            if (r < k) {
                oi[r] = key_id(key[s]);
                od[r] = key_dist(key[s]);
            }
        }
    }
};

// Per-query traversal counters (psb_knn_stats, int64[q][8]). They define the
// algorithmic bytes of a launch without changing the traversal.
// Compiled in only for the psb_knn_stats instantiations (ON = true): the timed
// kernels carry no counting code.
__device__ __forceinline__ int64_t global_ns()
{
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return (int64_t)t;
}
// Traversal trace (psb_knn_trace): one int64 per step of a query's walk, in
// order: node | level << 32 | flags << 40 (include/psb.h PSB_TRACE_*).
enum : unsigned { TR_PASS1 = 1u, TR_CHANGED = 2u, TR_SKIPPED = 4u, TR_FETCHED = 8u };
template <bool ON>
struct Stats {
    uint32_t fetch = 0, hit = 0, leaf = 0, ids = 0, offers = 0, cand = 0;
    int64_t t0 = 0;   // %globaltimer at the query's start (in-batch service time)
    int32_t nstep = 0;
    __device__ __forceinline__ Stats() { if (ON) t0 = global_ns(); }
    __device__ __forceinline__ void node(bool fetched) { if (ON) { fetched ? ++fetch : ++hit; } }
    __device__ __forceinline__ void scan() { if (ON) ++leaf; }
    __device__ __forceinline__ void id_loads(int n) { if (ON) ids += n; }
    __device__ __forceinline__ void merged(int m) { if (ON) { cand += m; offers += m > 0; } }
    // one traversal step: internal node (lvl >= 1) or leaf (lvl = 0)
    __device__ __forceinline__ void step(const TraceOut &tr, int64_t qi, int lane, int lvl, int node, unsigned flags)
    {
        if (ON) {
            if (tr.buf && lane == 0 && nstep < tr.cap)
                tr.buf[qi * tr.cap + nstep] = (int64_t)(uint32_t)node | ((int64_t)lvl << 32) | ((int64_t)flags << 40);
            ++nstep;
        }
    }
    __device__ __forceinline__ void write(int64_t *st, const TraceOut &tr, int64_t qi, int lane) const
    {
        if (ON && lane == 0) {
            if (tr.len) tr.len[qi] = nstep;
            if (!st) return;
            int64_t *o = st + qi * 8;
            o[0] = fetch;   // internal-node blocks fetched from memory
            o[1] = leaf;    // leaf blocks scanned
            o[2] = ids;     // point ids loaded
            o[3] = hit;     // internal visits served by the path cache
            o[4] = offers;  // leaf scans that changed the kNN list
            o[5] = cand;    // keys merged into the kNN list
            o[6] = t0;            // %globaltimer (ns) when the warp took the query
            o[7] = global_ns();   // ... and when it finished it (before the row store)
        }
    }
};


// NEXT-3 (large k, §V-E: "the kNN list grows with k
// ... future work: store large distances in shared memory"): for k > 128 the
// sorted list lives in per-warp shared memory (k u64 keys) instead of registers.
// Candidates below the k-th key are compacted (<= 32 per round), bitonic-sorted,
// and merged in place: list keys at positions >= the first insertion point move
// right by the number of candidates below them (processed in 32-key chunks from
// the end, so every key is read before its slot is overwritten) and candidates
// drop into the gaps; positions >= k fall off.
template <>
struct TopK<0> {
    u64 *list;   // [k] ascending, shared memory

    __device__ __forceinline__ void init(u64 *smem_list, int k)
    {
        list = smem_list;
        for (int i = threadIdx.x & 31; i < k; i += 32) list[i] = PAD_KEY;
        __syncwarp();
    }
    __device__ __forceinline__ u64 kth(int k) const { return list[k - 1]; }

    // number of keys < x in the ascending a[0..n)
    static __device__ __forceinline__ int rank(const u64 *a, int n, u64 x)
    {
        int lo = 0, hi = n;
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            if (a[mid] < x) lo = mid + 1;
            else hi = mid;
        }
        return lo;
    }

    template <int V>
    __device__ __forceinline__ int offer(const u64 (&cand)[V], int k, int lane, u64 &thr, u64 *scratch)
    {
        int total = 0;
        const unsigned lt = (1u << lane) - 1;
#pragma unroll
        for (int t = 0; t < V; ++t) {
            const unsigned b = __ballot_sync(FULL, cand[t] < thr);
            const int m = __popc(b);
            if (m == 0) continue;
            total += m;
            if (b >> lane & 1u) scratch[__popc(b & lt)] = cand[t];
            __syncwarp();
            u64 c = lane < m ? scratch[lane] : ~0ull;
            __syncwarp();
            c = m <= 8 ? warp_sort32<8>(c, lane) : (m <= 16 ? warp_sort32<16>(c, lane) : warp_sort32<32>(c, lane));
            scratch[lane] = c;
            __syncwarp();
            const int rc = lane < m ? rank(list, k, c) : k;       // candidate's rank among the old keys
            const int p0 = __shfl_sync(FULL, rc, 0);               // first insertion point
            for (int base = ((k - 1) >> 5) << 5; base >= 0 && base + 31 >= p0; base -= 32) {
                const int i = base + lane;
                const bool mv = i < k && i >= p0;
                const u64 a = mv ? list[i] : 0ull;
                const int sh = mv ? rank(scratch, m, a) : 0;
                __syncwarp();
                if (mv && i + sh < k) list[i + sh] = a;
                __syncwarp();
            }
            if (lane < m && lane + rc < k) list[lane + rc] = c;
            __syncwarp();
            thr = list[k - 1];
        }
        return total;
    }
    __device__ __forceinline__ void store(int k, int lane, int32_t *__restrict__ oi, float *__restrict__ od) const
    {
        for (int r = lane; r < k; r += 32) {
            oi[r] = key_id(list[r]);
            od[r] = key_dist(list[r]);
        }
    }
};

// S8+S9: scan one leaf, offer its points. Ids are fetched lazily, only for
// points whose distance can enter the list (dist <= current k-th distance).
template <int D, int V, int KS, bool ST>
__device__ __forceinline__ bool scan_leaf(const DevIndex &ix, int leaf, const Query<D> &q,
                                          int lane, TopK<KS> &T, int k, u64 &thr, Stats<ST> &S,
                                          u64 *scratch, unsigned pf)
{
    constexpr int F = 32 * V;
    float dist[V];
    S.scan();
    // Latency hiding (PSB_VAR_PREFETCH_*): the right sibling is the
    // next leaf whenever this scan changes the list (Alg. 1 l.41), and this leaf's
    // ids are needed as soon as a distance passes the filter: start both L2->L1
    // transfers now, without holding registers.
    if constexpr (D == 0) {   // the PSB_VAR_PREFETCH_* variants run the runtime-d kernels only
        if ((pf & PF_NEXT) && leaf + 1 < ix.L) {
            // the whole right-sibling block: d*V lines of 128 B
            for (int o = lane; o < ix.d * V; o += 32)
                asm volatile("prefetch.global.L1 [%0];" ::"l"(ix.pts + ((int64_t)leaf + 1) * ix.d * F + o * 32));
        }
        if ((pf & PF_IDS) && lane < V)
            asm volatile("prefetch.global.L1 [%0];" ::"l"(ix.ids + (int64_t)leaf * F + lane * 32));
    }
    constexpr int DC = D;   // compile-time d (0: runtime)
    leaf_dists<D, V>(ix.pts + (int64_t)leaf * (DC > 0 ? DC : ix.d) * F, q, ix.d, lane, dist);
    const float td = key_dist(thr);
    bool any = false;
#pragma unroll
    for (int t = 0; t < V; ++t) any |= dist[t] <= td;
    if (!__any_sync(FULL, any)) return false;
    const int32_t *__restrict__ lid = ix.ids + (int64_t)leaf * F + lane * V;
    u64 cand[V];
    int loads = 0;
#pragma unroll
    for (int t = 0; t < V; ++t) {
        cand[t] = dist[t] <= td ? make_key(dist[t], __ldg(lid + t)) : ~0ull;
        loads += dist[t] <= td;
    }
    if (ST) S.id_loads(__reduce_add_sync(FULL, loads));
    const int m = T.template offer<V>(cand, k, lane, thr, scratch);
    S.merged(m);
    return m > 0;
}

// Per-warp shared-memory layout for the traversal kernels.
struct WarpSmem {
    static __host__ __device__ __forceinline__ size_t cache_floats(int H, int F) { return (size_t)(H + 1) * F; }
    static __host__ __device__ __forceinline__ size_t bytes(int H, int F, bool qsmem, int kbig = 0)
    {
        size_t b = cache_floats(H, F) * 4;
        b = (b + 15) & ~(size_t)15;
        b += (size_t)(H + 1) * 4;
        b = (b + 15) & ~(size_t)15;
        b += 32 * 8;                        // top-k merge scratch
        b += (size_t)kbig * 8;              // large-k list (TopK<0>)
        if (qsmem) b += PSB_DMAX * 4;
        return b;
    }
};

}  // namespace psb
