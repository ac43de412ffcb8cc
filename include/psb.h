/*
 * psb.h — C ABI of libpsb.so: exact k-nearest-neighbour queries by Parallel Scan
 * and Backtrack (PSB) over a bulk-loaded n-ary R-tree, on NVIDIA B200 (sm_100a).
 *
 * Paper: M. Nam, J. Kim, B. Nam, "Parallel Tree Traversal for Nearest Neighbor
 * Query on the GPU", ICPP 2016. Citations "P:Lx-y" are lines of that paper's text
 * with the section / algorithm they fall in.
 *
 * Problem (§I; Alg. 1 "SearchKNN(Point Q, int k)" P:L403-405): given n
 * points in d dimensions and a query point Q, return the k points closest to Q,
 * exactly (§I, §VI).
 *
 * Conventions shared by every entry point (DESIGN.md §2 "Readings"):
 *  - Distances are SQUARED Euclidean in binary32, accumulated over dimensions
 *    0..d-1 in order, each subtraction, product and sum rounded to nearest-even
 *    separately (no FMA, no flush-to-zero):
 *        s = +0; for j: t = p[j] - q[j]; s = s + t*t.
 *  - A result row holds the k smallest (dist, id) pairs under lexicographic order
 *    (distance first, then id), ascending. If k > n the row is padded with
 *    (id -1, dist +inf).
 *  - Ids are 0-based input row numbers plus the index's id_base.
 *  - Layouts: points[n][d], queries[q][d] fp32 row-major; out_ids[q][k] int32,
 *    out_dists[q][k] fp32, row-major.
 *  - Queries and outputs may be CUDA device pointers on the index's device or
 *    host memory. Pinned (page-locked, hence device-mapped) host buffers are
 *    used in place by the kernels (zero-copy): result rows are written row by
 *    row as queries finish, and for batches of up to 16,384 queries the
 *    one-warp-per-query traversals read each query's d floats over the host link
 *    (larger batches, split mode and brute force, where many warps read each
 *    query, stage pinned queries with one copy). Pageable host
 *    queries and outputs are staged through stream-ordered device scratch with
 *    cudaMemcpyAsync on `stream`. Either way
 *    the results are in host memory once the stream reaches the end of the call
 *    (psb_build: points may be host or device memory).
 *  - Query calls are asynchronous on `stream` (a cudaStream_t; NULL = legacy
 *    default stream). Argument errors are returned synchronously without
 *    launching; launch failures return PSB_ECUDA; errors during execution surface
 *    at the caller's next synchronisation. Inputs must stay alive and unmodified
 *    until the stream reaches the work.
 *  - No entry point prints, aborts or throws. psb_last_error() returns a
 *    thread-local message describing the last failure on the calling thread.
 *  - An index is immutable after build: concurrent queries on different streams
 *    are safe. It is bound to the device that was current at build time.
 */
#ifndef PSB_H
#define PSB_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct psb_index psb_index; /* opaque */

enum {
    PSB_OK = 0,
    PSB_EINVAL = -1,          /* bad argument (null pointer, range, non-finite coordinate) */
    PSB_ENOMEM = -2,          /* host or device allocation failed                          */
    PSB_ECUDA = -3,           /* CUDA runtime error (message in psb_last_error)           */
    PSB_EUNSUPPORTED = -4     /* valid but outside this build (e.g. k > PSB_KMAX)         */
};

/* Leaf packing order for psb_build_ex `flags` (§IV-A: sort points by
 * a space-filling-curve key and pack them into full leaves, bottom-up). */
enum { PSB_PACK_HILBERT = 0, PSB_PACK_STR = 1, PSB_PACK_KMEANS = 2 };
/* PSB_PACK_KMEANS (NEXT-4, §IV-B): k-means with k = number of leaves
 * (P:L586-587), initialised from the Hilbert leaves, 4 Lloyd iterations whose
 * assignment step is this library's own exact 1-NN search over the centroids;
 * leaves are then packed cluster by cluster in the Hilbert order of the
 * centroids. GPU loader only. Deterministic. */
/* Build-location flag (OR into psb_build_ex `flags`). Hilbert packing runs on
 * the GPU by default (keys, CUB radix sort, permutation and MBR levels in CUDA
 * kernels; NEXT-1); PSB_BUILD_HOST forces the host (OpenMP) loader. STR always
 * runs on the host. Both loaders produce the same index. */
#define PSB_BUILD_HOST 0x100u
/* Node-shape flag (OR into psb_build_ex `flags`): SS-tree bounding spheres
 * instead of MBRs (the paper's own index, §II-C; NEXT-2). Each internal
 * node stores its children's spheres as rows centre[d][fanout] then
 * radius[fanout], built bottom-up by parallel Ritter (Alg. 2) on the
 * GPU with radii rounded up so every point is contained. Query bounds use
 * directed rounding plus a relative margin, so results stay exact. GPU Hilbert
 * loader only (not with PSB_BUILD_HOST / PSB_PACK_STR). */
#define PSB_NODE_SPHERE 0x200u

#define PSB_KMAX 2048         /* largest k: <= 128 in registers (4 keys per lane), up to
                                 2048 in a per-warp shared-memory list (NEXT-3) */
#define PSB_DMAX 64           /* largest dimensionality                               */

/* Bulk-load an R-tree over points[n][d] (§IV, bottom-up construction,
 * with minimum bounding rectangles as the bounding shape, §I):
 *  - points are ordered by a Hilbert key and packed left to right
 *    into leaves of exactly `fanout` points (100% utilisation, P:L162-163,
 *    P:L678-684); only the last leaf may be partial;
 *  - every internal node has up to `fanout` children; each node stores its
 *    children's MBRs as structure-of-arrays rows lo[d][fanout], hi[d][fanout]
 *    (§V-A: "stored in SoA so that memory coalescing can be employed");
 *  - leaves are contiguous in left-to-right order with sequence ids 0..L-1; the
 *    parent of node i is i/fanout one level up and the right sibling of leaf j
 *    is j+1 (the parent links and rightSibling of Alg. 1).
 * `points` may be host or device memory; it is copied (the caller may free it
 * afterwards). n >= 1, 1 <= d <= PSB_DMAX, fanout in {32,64,128,256,512}, all
 * coordinates finite. Synchronous. Returns NULL on error (see psb_last_error). */
psb_index *psb_build(const float *points, int64_t n, int32_t d, int32_t fanout);

/* As psb_build, plus: returned ids are id_base + input row (data-sharded use:
 * a shard over rows [r0, r1) of a global set passes id_base = r0;
 * id_base >= 0 and id_base + n <= 2^31 - 1), and `flags` selects the packing
 * (PSB_PACK_HILBERT or PSB_PACK_STR, optionally | PSB_BUILD_HOST). On success
 * *out receives the index. */
int psb_build_ex(const float *points, int64_t n, int32_t d, int32_t fanout, int64_t id_base,
                 uint32_t flags, psb_index **out);

/* PSB kNN (Alg. 1, §III, with the readings of DESIGN.md §2): for each
 * of the q queries, one warp descends greedily to the closest leaf to obtain an
 * initial pruning distance (Alg. 1 l.3), then restarts at the root, descends to
 * the leftmost child within the pruning distance whose leaves are not yet
 * visited (l.16-26), scans leaves left to right while they improve the kNN set
 * (l.32-41) and backtracks through parent links otherwise (l.27-30, l.42-45).
 * 1 <= k <= PSB_KMAX (else PSB_EUNSUPPORTED), q >= 0 (q = 0 is a no-op).
 * For k > 128 the kNN list lives in shared memory (§V-E future
 * work: large k) and psb_knn_split runs as psb_knn. */
int psb_knn(const psb_index *idx, const float *queries, int64_t q, int32_t k,
            int32_t *out_ids, float *out_dists, void *stream);

/* Split mode of psb_knn (SURVEY.md §8(e) "intra-GPU split"): `parts` warps share
 * each query, each running PSB (Alg. 1) over the leaves it owns; the warps of a
 * query share their pruning distance through atomicMin and their per-part
 * lists are merged on the device. Same results as psb_knn.
 *  - When the (query, part) tasks do not fill the GPU (single queries: latency),
 *    part p owns the p-th of `parts` contiguous leaf ranges.
 *  - When they do (batches), part p owns the level-1 nodes n with n % parts == p,
 *    so the eligible leaves of a query, which cluster in neighbouring nodes, are
 *    spread over all parts: this shortens the long queries that end a batch.
 * parts = 0 picks, with W = (1 + (min(k,F)/F)^(1/d))^d the classic uniform-data
 * estimate of the leaves a query touches: ~16 warps per SM in total (at least 16
 * leaves per part) for q <= 8 x SMs when W >= 16; 2-8 parts (14 x resident warps / q)
 * for batches of fewer
 * than 128 x SMs queries when W >= 64; else 1.
 * parts = 1 is psb_knn. For k > 128 psb_knn_split runs as psb_knn. */
int psb_knn_split(const psb_index *idx, const float *queries, int64_t q, int32_t k, int32_t parts,
                  int32_t *out_ids, float *out_dists, void *stream);

/* The paper's comparison algorithm: classic branch-and-bound kNN (Roussopoulos
 * et al. [17], §III) run data-parallel on the GPU with parent links
 * instead of a stack (§IV-D): children in (MINDIST, index) order,
 * each leaf followed by a return to its parent. Same arguments and results as
 * psb_knn. */
int psb_knn_branch_and_bound(const psb_index *idx, const float *queries, int64_t q, int32_t k,
                             int32_t *out_ids, float *out_dists, void *stream);

/* GPU brute-force exhaustive kNN (the paper's other baseline, §I,
 * P:L936-947 §V-D): every point against every query, same distance formula and
 * order. Same arguments and results as psb_knn. May allocate stream-ordered
 * scratch on `stream`. */
int psb_knn_bruteforce(const psb_index *idx, const float *queries, int64_t q, int32_t k,
                       int32_t *out_ids, float *out_dists, void *stream);

/* Variant selector for the two tree traversals (measurement and ablations):
 * bit 0 PSB_VAR_NOCACHE  — re-fetch every node on return instead of reusing the
 *                          per-level MINDIST path cache (the paper's parent-link
 *                          behaviour);
 * bit 1 PSB_VAR_NOMAXDIST — skip the k-th-MAXDIST bound (Alg. 1 l.13-15);
 * bit 2 PSB_VAR_INPUT_ORDER — process the queries in input order;
 * bit 3 PSB_VAR_LEAF_ORDER — process them in the order of their ClosestLeaf: the
 *                          batch is first sorted (stably) by the sequence id of
 *                          the leaf PSB's pass 1 descends to (Alg. 1 l.3),
 *                          so warps running together walk neighbouring leaves and
 *                          share them in L1/L2. Rows are still written in input
 *                          order. With neither bit, the batch is ordered when
 *                          q >= 1024 and the leaves (points + ids) exceed 64 MiB:
 *                          by ClosestLeaf for d > 4, by the queries' Hilbert key
 *                          over the data's bounding box for d <= 4 (no node reads;
 *                          C5 slab 9.74 -> 9.24 ms).
 * bit 4 PSB_VAR_PREFETCH_NEXT — with every leaf scan, prefetch the right
 *                          sibling's coordinates into L1 (the next leaf whenever
 *                          the scan changes the kNN list, Alg. 1 l.41);
 * bit 5 PSB_VAR_PREFETCH_IDS — with every leaf scan, prefetch the leaf's point
 *                          ids into L1 (they are loaded lazily, only for points
 *                          that pass the distance filter). Bits 4 and 5 run the
 *                          runtime-d kernels (measured slower in batches,
 *                          DESIGN.md §6; the compile-time-d kernels carry no
 *                          prefetch code).
 * bit 6 PSB_VAR_P1_INDEX_TIE — pass 1's ClosestLeaf descent (R4) breaks
 *                          MINDIST ties by child index alone. By default a tie
 *                          goes to the child with the smaller MAXDIST first (a
 *                          query inside several overlapping boxes descends into
 *                          the one that hugs it), which tightens the initial
 *                          pruning distance (R4).
 * bit 7 PSB_VAR_KTH_MAXDIST — bound the k-th neighbour distance at each fetched
 *                          node by the k-th smallest child MAXDIST, as Alg. 1
 *                          l.13-15 prints it (every child counted as one point).
 *                          By default, when k <= fanout, the bound is the
 *                          smallest MAXDIST over children whose subtrees hold
 *                          >= k points (R3): tighter, and a warp min
 *                          instead of a radix select.
 * bit 8 PSB_VAR_NO_AUTO_PREFETCH — accepted, no effect: round 1 turned bits 4
 *                          and 5 on by default at d = 16 and this bit turned them
 *                          off; no build does so any more.
 * bit 9 PSB_VAR_GENERIC_D — run the runtime-d instantiation of the kernels even
 *                          where a compile-time-d one exists (d, fanout) in
 *                          {(2,32), (3,64), (3,128), (8,128), (16,128)}: the two
 *                          traverse identically (tests compare their traces).
 * Results are identical for every variant. */
enum { PSB_VAR_NOCACHE = 1, PSB_VAR_NOMAXDIST = 2, PSB_VAR_INPUT_ORDER = 4,
       PSB_VAR_LEAF_ORDER = 8, PSB_VAR_PREFETCH_NEXT = 16, PSB_VAR_PREFETCH_IDS = 32,
       PSB_VAR_P1_INDEX_TIE = 64, PSB_VAR_KTH_MAXDIST = 128, PSB_VAR_NO_AUTO_PREFETCH = 256,
       PSB_VAR_GENERIC_D = 512 };
int psb_knn_ex(const psb_index *idx, const float *queries, int64_t q, int32_t k,
               int32_t *out_ids, float *out_dists, void *stream, int32_t algo, uint32_t variant);
enum { PSB_ALGO_PSB = 0, PSB_ALGO_BNB = 1, PSB_ALGO_BRUTE = 2 };

/* psb_knn_ex (algo PSB_ALGO_PSB or PSB_ALGO_BNB) that also writes per-query
 * traversal counters to `stats`, a DEVICE array int64[q][8]:
 *   {internal-node fetches from memory, leaf scans, point ids loaded,
 *    internal-node visits served by the path cache, leaf scans that changed the
 *    kNN list, keys merged into the list, t_start, t_end}
 * where t_start/t_end are the device %globaltimer (ns) when the warp took the
 * query and when it finished it: the in-batch service time.
 * The counters define the algorithmic bytes of a launch:
 *   fetches*fanout*2*d*4 + leaf_scans*fanout*d*4 + ids*4 + q*(4*d + 8*k).
 * The traversal (and hence every counter) is deterministic: a counting run and
 * a timing run do the same work. Results are identical to psb_knn_ex. */
int psb_knn_stats(const psb_index *idx, const float *queries, int64_t q, int32_t k,
                  int32_t *out_ids, float *out_dists, void *stream, int32_t algo, uint32_t variant,
                  int64_t *stats);

/* psb_knn_stats plus the traversal trace of every query (tests and
 * diagnostics: the visit order of Alg. 1, and of the B&B
 * comparator). trace is a DEVICE int64[q][cap]: step i of query r's walk is
 * trace[r][i] = node | level << 32 | flags << 40, where level 0 is a leaf (node =
 * its sequence id) and level >= 1 an internal node visit (node = its index in
 * the level), in the order the warp took them; flags:
 *   PSB_TRACE_PASS1   (1)  the step belongs to pass 1 (getInitialPruningDistance);
 *   PSB_TRACE_CHANGED (2)  leaf scan that changed the kNN list;
 *   PSB_TRACE_SKIPPED (4)  pass-2 visit of a leaf already scanned in pass 1
 *                          (not scanned again);
 *   PSB_TRACE_FETCHED (8)  internal node fetched from memory (else served by
 *                          the path cache).
 * trace_len (DEVICE int32[q]) receives each query's number of steps; steps past
 * cap are counted but not stored. stats may be NULL. 1 <= cap. The counting
 * kernels run (compile-time-d ones where they exist, PSB_VAR_GENERIC_D for the
 * generic ones); the traversal and results are those of psb_knn_ex. */
enum { PSB_TRACE_PASS1 = 1, PSB_TRACE_CHANGED = 2, PSB_TRACE_SKIPPED = 4, PSB_TRACE_FETCHED = 8 };
int psb_knn_trace(const psb_index *idx, const float *queries, int64_t q, int32_t k,
                  int32_t *out_ids, float *out_dists, void *stream, int32_t algo, uint32_t variant,
                  int64_t *stats, int64_t *trace, int32_t cap, int32_t *trace_len);

/* Merge `parts` per-shard result sets ids/dists[parts][q][k] (each row ascending
 * by (dist, id), ids global) into the first k of their union, out[q][k]
 * (data-sharded mode: the step after the all-gather). Device pointers,
 * asynchronous on `stream`. 1 <= parts, 1 <= k <= PSB_KMAX. */
int psb_merge_topk(const int32_t *ids, const float *dists, int32_t parts, int64_t q, int32_t k,
                   int32_t *out_ids, float *out_dists, void *stream);

/* ---- Data-sharded exchange over peer memory (north_star) ----
 * The NCCL route (all-gather of every shard's [q][k] lists + psb_merge_topk) is
 * replaced by kernels that pull only the rows a rank owns directly out of the
 * peers' result buffers (CUDA IPC mappings over NVLink/NVSwitch) and merge them,
 * after a device-side flag barrier: no collective launch, no staging buffer,
 * P-fold less traffic into each rank than an all-gather. (The paper itself is
 * single-GPU, §V-A; the merge is exact because (dist, id) is a total
 * order and every global id lives in one slab.)
 *
 * Protocol, one object per rank (all ranks: same parts, q, k):
 *   psb_exchange_create(parts, rank, q, k, &x)   allocates on the current device
 *     two [q][k] result buffers (alternating by epoch parity), parts 64-bit flag
 *     slots and a status word; 1 <= parts <= PSB_MAX_PARTS, 1 <= q < 2^32,
 *     1 <= k <= 128;
 *   psb_exchange_handle(x, blob, cap, &used)     blob (IPC handles + a random
 *     per-process nonce) to share with every rank (e.g. torch.distributed
 *     all_gather_object); blob == NULL: only *used is written;
 *   psb_exchange_connect(x, blobs)               maps all ranks' buffers (blobs in
 *     rank order). A blob from the calling process (same nonce) is used without
 *     IPC; if it lives on another device, peer access is enabled;
 *   each step, with epoch = 1, 2, 3 ... (< 2^31):
 *     psb_exchange_buffers(x, epoch, &ids, &dists)  this rank's [q][k] result
 *       buffers for the step: run the local psb_knn* into them (global ids);
 *     psb_exchange_signal(x, epoch, rows_done, stream)  stream-ordered after the
 *       local search of rows [0, rows_done): publishes (epoch, rows_done) to
 *       every peer (release, system scope). Rows may be searched and signalled
 *       in increasing chunks (rows_done increasing within an epoch) so that the
 *       merge of one chunk overlaps the search of the next;
 *     psb_exchange_merge(x, epoch, row0, rows, out_ids, out_dists, stream)
 *       one single-thread wait kernel until every rank (this one included) has
 *       signalled (epoch, >= max(row0 + rows, 1)), then one warp per row writes
 *       the merged first k of rows [row0, row0+rows) of all parts' lists to
 *       out[rows][k] (device pointers). rows may be 0: the wait still runs (it
 *       is what makes the double buffering safe), nothing is written;
 *     psb_exchange_step(x, epoch, row0, rows, out...)  = signal(epoch, q) + merge.
 *   Every rank must signal each epoch (rows_done = q at the latest) and call
 *   merge at least once per epoch, after its signals. Within one process, issue
 *   every rank's signal for a chunk before any rank's merge that waits on it
 *   (a merge's wait must not be queued ahead of a signal it needs: kernels on
 *   different streams are not guaranteed to run concurrently).
 * Failure: the wait gives up after the timeout (10 s by default,
 * psb_exchange_set_timeout) or at once if an earlier wait gave up. The merge
 * then writes pad rows (-1, +inf), and from the moment the host can see it
 * (mapped status word, no synchronisation needed) every psb_exchange_* call on
 * x except psb_exchange_status / psb_exchange_free returns PSB_ECUDA: the
 * exchange must be freed and recreated. psb_exchange_status reports it
 * (1 = timed out) for work the device has completed.
 * Synchronous except psb_exchange_signal / merge / step. */
#define PSB_MAX_PARTS 16
typedef struct psb_exchange psb_exchange; /* opaque */
int psb_exchange_create(int32_t parts, int32_t rank, int64_t q, int32_t k, psb_exchange **out);
int psb_exchange_set_timeout(psb_exchange *x, int64_t timeout_ns);
int psb_exchange_handle(const psb_exchange *x, void *blob, int64_t cap, int64_t *used);
int psb_exchange_connect(psb_exchange *x, const void *const *blobs);
int psb_exchange_buffers(const psb_exchange *x, int64_t epoch, int32_t **ids, float **dists);
int psb_exchange_signal(psb_exchange *x, int64_t epoch, int64_t rows_done, void *stream);
int psb_exchange_merge(psb_exchange *x, int64_t epoch, int64_t row0, int64_t rows, int32_t *out_ids,
                       float *out_dists, void *stream);
int psb_exchange_step(psb_exchange *x, int64_t epoch, int64_t row0, int64_t rows, int32_t *out_ids,
                      float *out_dists, void *stream);
int psb_exchange_status(const psb_exchange *x, int32_t *timed_out);
void psb_exchange_free(psb_exchange *x);

/* Shape of an index. Any output pointer may be NULL. `levels` counts internal
 * levels (root at level `levels`, leaves at level 0); device_bytes is the index's
 * device footprint. */
int psb_index_info(const psb_index *idx, int64_t *n, int32_t *d, int32_t *fanout, int64_t *leaves,
                   int32_t *levels, int64_t *device_bytes);

/* Copy the index's flat arrays to host memory (tests, replicas). Layout of the
 * exported blob (all little-endian):
 *   int64 header[8] = {n, d, fanout, leaves L, levels H, id_base, total_nodes, sphere}
 *   int64 nodes_per_level[H+1]            (level 0 = L leaves)
 *   float pts[L][d][fanout]               (leaf-blocked SoA; pad slots +inf)
 *   int32 ids[L][fanout]                  (pad slots -1)
 *   float nodes: for level 1..H, nodes_per_level[l] blocks of [d][2][fanout]
 *                (row 2j = lo of dim j, row 2j+1 = hi; empty slots lo=+inf, hi=-inf),
 *                or for sphere indexes blocks of [d+1][fanout] (centre rows, then
 *                the radius row; empty slots centre +inf, radius 0)
 * If host_buf is NULL or cap is too small, only *used is written (required size)
 * and PSB_EINVAL is returned when host_buf is non-NULL. Synchronous. */
int psb_index_export(const psb_index *idx, void *host_buf, int64_t cap, int64_t *used);

/* Create an index on the current device from a psb_index_export blob (same
 * layout): replicas (query-sharded mode: build once, broadcast
 * the flat buffers, import on every rank) and hand-built trees (tests: the
 * Fig. 2 tree). The blob is validated before anything is uploaded:
 * level geometry of a packed tree (nodes_per_level[l] = ceil(previous / fanout)
 * up to a single root), finite coordinates with id >= 0 for points and +inf
 * with id -1 for pad slots, header n = the number of points, and every box
 * bounding its leaf's points or its node's child boxes (empty content: lo =
 * +inf, hi = -inf) — what exactness needs (MINDIST <= dist <= MAXDIST under RN
 * rounding). Pad slots may sit anywhere; if a leaf other than the
 * last holds fewer than `fanout` points, the traversals bound the k-th distance
 * with the printed k-th-MAXDIST rule (Alg. 1 l.13-15) instead of the
 * count-aware one (R3). Sphere indexes: PSB_EUNSUPPORTED. The blob is copied
 * (the caller keeps ownership). Synchronous. */
int psb_index_import(const void *blob, int64_t size, psb_index **out);

/* Host-only bulk load (no CUDA call, no device needed): runs the same packing as
 * psb_build_ex and writes the psb_index_export blob for it into host_buf
 * (same size protocol as psb_index_export). For layout tests on machines without
 * a GPU; a device index built from the same arguments exports identical bytes. */
int psb_build_host_blob(const float *points, int64_t n, int32_t d, int32_t fanout, int64_t id_base,
                        uint32_t flags, void *host_buf, int64_t cap, int64_t *used);

/* Measurement probe (not part of the query path): the L2 read bandwidth of the
 * current device, in GB/s, for the roofline bench.py reports (SURVEY.md §8(d):
 * the traversal's node and leaf blocks are served mostly from L2, so that is the
 * memory ceiling their algorithmic bytes are compared with). A `bytes` buffer
 * (>= 1 MiB; 64 MiB fits B200's L2) is read once to make it L2-resident, then
 * `passes` times per timed launch with L2-only (ld.global.cg) loads by 4 x 512
 * threads per SM, in four shapes (one or four 16-byte loads in flight per thread,
 * one or two 32-byte loads); *gbs = the best of `reps` CUDA-event-timed launches
 * over all shapes (one 16-byte load per thread under-reads the L2 by ~20 %).
 * Synchronous; allocates and frees its own buffer. */
int psb_probe_l2_read(int64_t bytes, int32_t passes, int32_t reps, double *gbs);

/* Release the index and its device memory. NULL is a no-op. */
void psb_free(psb_index *idx);

/* Thread-local message for the last failing call on this thread ("" if none). */
const char *psb_last_error(void);

/* Library version string ("psb-b200 <version> sm_100a"). */
const char *psb_version(void);

#ifdef __cplusplus
}
#endif
#endif /* PSB_H */
