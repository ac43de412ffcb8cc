// psb_launch.h — host-side launchers implemented in the .cu files.
#pragma once
#include <cuda_runtime.h>

#include "psb_internal.h"

namespace psb {

// Records a CUDA error in psb_last_error and maps it to PSB_ECUDA.
int report_cuda(cudaError_t e, const char *what);

// PSB_ALGO_PSB or PSB_ALGO_BNB, one warp per query (knn_tree.cu).
// `stats` (nullable, device [nq][4] int64): per query {internal node fetches,
// leaf scans, id loads, path-cache hits}.
// parts > 1 (PSB only): latency mode, each query's leaves split over `parts` warps.
// `tr` (psb_knn_trace): per-query traversal steps; with stats or tr.len set the
// counting instantiation runs (PSB_VAR_GENERIC_D: the generic-d one).
int launch_tree(int algo, const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi,
                float *od, cudaStream_t st, uint32_t variant, int64_t *stats, cudaMemPool_t pool, int parts,
                const TraceOut &tr);

// Exhaustive scan of all points (knn_brute.cu). Splits the point set into
// chunks when there are too few queries to fill the GPU and merges the partial
// lists with launch_merge; scratch is stream-ordered.
int launch_brute(const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi, float *od,
                 cudaStream_t st, int sm_count, cudaMemPool_t pool);

// Per-(d, fanout) launchers, instantiated one translation unit each
// (knn_tree_d<D>_v<V>.cu, knn_brute_d<D>_v<V>.cu; V = fanout/32, D = 0: runtime d).
// They return PSB_NOT_INSTANTIATED when the request needs the generic-d kernels.
constexpr int PSB_NOT_INSTANTIATED = 1;
template <int D, int V>
int launch_tree_ks(int algo, const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi,
                   float *od, cudaStream_t st, uint32_t variant, int64_t *stats, cudaMemPool_t pool, int parts,
                   const TraceOut &tr);
template <int D, int V>
int launch_brute_ks(const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi, float *od,
                    cudaStream_t st, int sm, cudaMemPool_t pool);

// Latency-mode helpers (knn_merge.cu): shared pruning distances to +inf (and the
// task queue, if any, to 0) in one launch, and the filtered merge of [nq][parts][k]
// per-part lists.
void init_shared_pd(float *gpd, int64_t nq, unsigned long long *queue, cudaStream_t st);

// cudaOccupancyMaxActiveBlocksPerMultiprocessor, memoised per (kernel, block size,
// dynamic smem, device): the launchers ask on every call, and a single-query call
// is latency-bound by host work like this (psb_api.cpp).
int cached_occupancy(const void *kern, int threads, size_t smem);
int launch_merge_parts(const int32_t *ids, const float *dists, const float *gpd, int parts, int64_t nq, int k,
                       int32_t *oi, float *od, cudaStream_t st);
template <int D>
int launch_brute_v(const DevIndex &ix, const float *queries, int64_t nq, int k, int32_t *oi, float *od,
                   cudaStream_t st, int sm, cudaMemPool_t pool);

// GPU bulk load (psb_build_gpu.cu) into preallocated pts/ids/nodes; d_points is
// device memory [n][d]. Synchronous on `st`.
int gpu_bulk_load(const float *d_points, const GpuLayoutShape &sh, int64_t id_base, float *pts, int32_t *ids,
                  float *nodes, cudaStream_t st, bool sphere, int kmeans_iters);

// Batch order by Hilbert key for d <= PSB_HILBERT_ORDER_MAX_D (knn_order.cu):
// order[i] = the input row processed i-th, keys over the index box (index_box).
int hilbert_query_order(const float *queries, int64_t nq, int d, const float *box, int32_t *order, cudaMemPool_t pool,
                        cudaStream_t st);
// Bounding box of an index's real points into box[2d] (lo row, hi row). Async.
int index_box(const float *pts, const int32_t *ids, int64_t L, int d, int F, float *box, cudaStream_t st);

// Stable sort of queries by closest-leaf id (knn_order.cu): order[i] = the input
// row processed i-th. leaf_key is [nq] device memory; order is [nq].
int sort_query_order(const uint32_t *leaf_key, int64_t nq, int64_t L, int32_t *order, cudaMemPool_t pool,
                     cudaStream_t st);

// [parts][nq][k] sorted (dist, id) lists -> first k of their union (knn_brute.cu).
int launch_merge(const int32_t *ids, const float *dists, int parts, int64_t nq, int k, int32_t *oi,
                 float *od, cudaStream_t st);

}  // namespace psb
