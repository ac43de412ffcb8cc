// psb_api.cpp — the C ABI of libpsb.so (declared and documented in include/psb.h):
// argument validation, index upload, kernel dispatch, error reporting.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <new>
#include <tuple>

#include "psb_internal.h"
#include "psb_launch.h"

#ifndef PSB_VERSION
#define PSB_VERSION "0.1.0"
#endif

static thread_local char g_err[512];

void psb_set_error(const char *fmt, ...)
{
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof g_err, fmt, ap);
    va_end(ap);
}

namespace psb {
int cached_occupancy(const void *kern, int threads, size_t smem)
{
    static std::mutex mu;
    static std::map<std::tuple<const void *, int, size_t, int>, int> memo;
    int dev = 0;
    cudaGetDevice(&dev);
    const auto key = std::make_tuple(kern, threads, smem, dev);
    {
        std::lock_guard<std::mutex> g(mu);
        auto it = memo.find(key);
        if (it != memo.end()) return it->second;
    }
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, threads, smem) != cudaSuccess) {
        cudaGetLastError();
        return 0;                      // not memoised: a later call may succeed
    }
    std::lock_guard<std::mutex> g(mu);
    memo[key] = n;
    return n;
}

int report_cuda(cudaError_t e, const char *what)
{
    if (e == cudaSuccess) return PSB_OK;
    psb_set_error("%s: %s (%s)", what, cudaGetErrorString(e), cudaGetErrorName(e));
    return e == cudaErrorMemoryAllocation ? PSB_ENOMEM : PSB_ECUDA;
}
}  // namespace psb
using psb::report_cuda;

struct psb_index {
    int device = -1;
    int sm_count = 0;
    int64_t n = 0, L = 0, id_base = 0;
    int32_t d = 0, F = 0, H = 0;
    int64_t nlev[PSB_MAXLVL + 1] = {};
    int64_t level_off[PSB_MAXLVL + 1] = {};
    int64_t node_floats = 0;
    float *pts = nullptr;
    int32_t *ids = nullptr;
    float *nodes = nullptr;
    float *box = nullptr;           // bounding box of the real points [2][d] (batch ordering)
    int64_t device_bytes = 0;
    int32_t sphere = 0, blk_floats = 0;
    int32_t irregular = 0;          // imported with non-full leaves (DevIndex::irregular)
    cudaMemPool_t pool = nullptr;   // stream-ordered scratch (host-buffer staging, brute-force partials)
};

static void index_release(psb_index *ix)
{
    if (!ix) return;
    int prev = -1;
    cudaGetDevice(&prev);
    if (ix->device >= 0) cudaSetDevice(ix->device);
    cudaFree(ix->pts);
    cudaFree(ix->ids);
    cudaFree(ix->nodes);
    cudaFree(ix->box);
    if (ix->pool) cudaMemPoolDestroy(ix->pool);
    if (prev >= 0) cudaSetDevice(prev);
    delete ix;
}

static DevIndex dev_view(const psb_index *ix)
{
    DevIndex v;
    memset(&v, 0, sizeof v);
    v.pts = ix->pts;
    v.ids = ix->ids;
    v.nodes = ix->nodes;
    v.box = ix->box;
    for (int l = 0; l <= PSB_MAXLVL; ++l) {
        v.level_off[l] = ix->level_off[l];
        v.nlev[l] = ix->nlev[l];
    }
    int64_t s = 1;
    for (int l = 0; l <= PSB_MAXLVL; ++l) {
        v.span[l] = s < ix->L ? s : ix->L;   // F^l clamped at L (only the root reaches it)
        if (s < ix->L) s *= ix->F;
    }
    v.n = ix->n;
    v.L = ix->L;
    v.H = ix->H;
    v.d = ix->d;
    v.F = ix->F;
    v.sm_count = ix->sm_count;
    v.sphere = ix->sphere;
    v.blk_floats = ix->blk_floats;
    v.irregular = ix->irregular;
    return v;
}

// Own pool for per-call scratch; memory stays mapped between calls (a zero
// release threshold would unmap and remap it at every synchronisation).
static int make_pool(psb_index *ix, const char *fn)
{
    cudaMemPoolProps props;
    memset(&props, 0, sizeof props);
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = ix->device;
    cudaError_t e = cudaMemPoolCreate(&ix->pool, &props);
    if (e != cudaSuccess) {
        ix->pool = nullptr;
        return report_cuda(e, fn);
    }
    uint64_t keep = UINT64_MAX;
    cudaMemPoolSetAttribute(ix->pool, cudaMemPoolAttrReleaseThreshold, &keep);
    return PSB_OK;
}

// The bounding box of the index's points (the Hilbert batch order, knn_order.cu).
static int attach_box(psb_index *ix, const char *fn)
{
    cudaError_t e = cudaMalloc((void **)&ix->box, sizeof(float) * 2 * (size_t)ix->d);
    if (e != cudaSuccess) return report_cuda(e, fn);
    int rc = psb::index_box(ix->pts, ix->ids, ix->L, ix->d, ix->F, ix->box, 0);
    if (rc == PSB_OK) rc = report_cuda(cudaStreamSynchronize(0), fn);
    ix->device_bytes += (int64_t)(sizeof(float) * 2 * ix->d);
    return rc;
}

extern "C" {

const char *psb_last_error(void) { return g_err; }

const char *psb_version(void) { return "psb-b200 " PSB_VERSION " sm_100a"; }

int psb_build_ex(const float *points, int64_t n, int32_t d, int32_t fanout, int64_t id_base,
                 uint32_t flags, psb_index **out)
{
    g_err[0] = 0;
    if (!out) { psb_set_error("psb_build_ex: out is NULL"); return PSB_EINVAL; }
    *out = nullptr;
    if (!points) { psb_set_error("psb_build_ex: points is NULL"); return PSB_EINVAL; }
    if (n < 1 || d < 1 || d > PSB_DMAX) {
        psb_set_error("psb_build_ex: n=%lld d=%d out of range", (long long)n, d);
        return PSB_EINVAL;
    }
    int dev = -1;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return report_cuda(e, "psb_build_ex: cudaGetDevice");
    GpuLayoutShape shape;
    int rc = psb_layout_shape(n, d, fanout, id_base, flags, &shape);
    if (rc != PSB_OK) return rc;
    const bool sphere = (flags & PSB_NODE_SPHERE) != 0;
    const uint32_t pack = flags & ~(uint32_t)(PSB_BUILD_HOST | PSB_NODE_SPHERE);
    const bool kmeans = pack == PSB_PACK_KMEANS;
    const bool on_gpu = (pack == PSB_PACK_HILBERT || kmeans) && !(flags & PSB_BUILD_HOST);
    if ((sphere || kmeans) && !on_gpu) {
        psb_set_error("psb_build_ex: PSB_NODE_SPHERE / PSB_PACK_KMEANS need the GPU loader");
        return PSB_EUNSUPPORTED;
    }
    cudaPointerAttributes attr;
    e = cudaPointerGetAttributes(&attr, points);
    if (e != cudaSuccess) {
        cudaGetLastError();
        attr.type = cudaMemoryTypeUnregistered;
    }
    const bool dev_in = attr.type == cudaMemoryTypeDevice;

    psb_index *ix = new (std::nothrow) psb_index;
    if (!ix) { psb_set_error("psb_build_ex: host allocation failed"); return PSB_ENOMEM; }
    ix->device = dev;
    cudaDeviceGetAttribute(&ix->sm_count, cudaDevAttrMultiProcessorCount, dev);
    ix->n = n; ix->L = shape.L; ix->id_base = id_base;
    ix->d = d; ix->F = fanout; ix->H = shape.H;
    for (int l = 0; l <= PSB_MAXLVL; ++l) { ix->nlev[l] = shape.nlev[l]; ix->level_off[l] = shape.level_off[l]; }
    ix->node_floats = shape.total_node_floats;
    ix->sphere = shape.sphere;
    ix->blk_floats = shape.blk_floats;
    const size_t bp = sizeof(float) * (size_t)(shape.L * d * fanout);
    const size_t bi = sizeof(int32_t) * (size_t)(shape.L * fanout);
    const size_t bn = sizeof(float) * (size_t)shape.total_node_floats;
    if ((e = cudaMalloc((void **)&ix->pts, bp)) != cudaSuccess ||
        (e = cudaMalloc((void **)&ix->ids, bi)) != cudaSuccess ||
        (e = cudaMalloc((void **)&ix->nodes, bn)) != cudaSuccess) {
        rc = report_cuda(e, "psb_build_ex: device allocation");
        index_release(ix);
        return rc;
    }
    if (on_gpu) {
        // NEXT-1: the whole bulk load in CUDA kernels on a private stream
        cudaStream_t st;
        if ((e = cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking)) != cudaSuccess) {
            rc = report_cuda(e, "psb_build_ex: stream");
            index_release(ix);
            return rc;
        }
        const float *dpts = points;
        float *staged = nullptr;
        if (!dev_in) {
            const size_t bytes = sizeof(float) * (size_t)(n * d);
            if ((e = cudaMalloc((void **)&staged, bytes)) != cudaSuccess ||
                (e = cudaMemcpy(staged, points, bytes, cudaMemcpyHostToDevice)) != cudaSuccess) {
                rc = report_cuda(e, "psb_build_ex: stage points");
                cudaFree(staged);
                cudaStreamDestroy(st);
                index_release(ix);
                return rc;
            }
            dpts = staged;
        }
        rc = psb::gpu_bulk_load(dpts, shape, id_base, ix->pts, ix->ids, ix->nodes, st, sphere, kmeans ? 4 : 0);
        cudaStreamSynchronize(st);
        cudaFree(staged);
        cudaStreamDestroy(st);
        if (rc != PSB_OK) {
            index_release(ix);
            return rc;
        }
    } else {
        const float *host_pts = points;
        float *staged = nullptr;
        if (dev_in) {
            staged = (float *)malloc(sizeof(float) * (size_t)(n * d));
            if (!staged) { psb_set_error("psb_build_ex: host staging allocation failed"); index_release(ix); return PSB_ENOMEM; }
            e = cudaMemcpy(staged, points, sizeof(float) * (size_t)(n * d), cudaMemcpyDeviceToHost);
            if (e != cudaSuccess) { free(staged); rc = report_cuda(e, "psb_build_ex: copy points to host"); index_release(ix); return rc; }
            host_pts = staged;
        }
        HostLayout h;
        rc = psb_host_build(host_pts, n, d, fanout, id_base, flags, &h);
        free(staged);
        if (rc != PSB_OK) { index_release(ix); return rc; }
        if ((e = cudaMemcpy(ix->pts, h.pts, bp, cudaMemcpyHostToDevice)) != cudaSuccess ||
            (e = cudaMemcpy(ix->ids, h.ids, bi, cudaMemcpyHostToDevice)) != cudaSuccess ||
            (e = cudaMemcpy(ix->nodes, h.nodes, bn, cudaMemcpyHostToDevice)) != cudaSuccess) {
            rc = report_cuda(e, "psb_build_ex: upload");
            index_release(ix);
            return rc;
        }
    }
    ix->device_bytes = (int64_t)(bp + bi + bn);
    if ((rc = attach_box(ix, "psb_build_ex: bounding box")) != PSB_OK || (rc = make_pool(ix, "psb_build_ex")) != PSB_OK) {
        index_release(ix);
        return rc;
    }
    *out = ix;
    return PSB_OK;
}

psb_index *psb_build(const float *points, int64_t n, int32_t d, int32_t fanout)
{
    psb_index *ix = nullptr;
    return psb_build_ex(points, n, d, fanout, 0, PSB_PACK_HILBERT, &ix) == PSB_OK ? ix : nullptr;
}

void psb_free(psb_index *ix) { index_release(ix); }

static int check_query_args(const char *fn, const psb_index *ix, const float *queries, int64_t q,
                            int32_t k, const void *oi, const void *od)
{
    if (!ix) { psb_set_error("%s: index is NULL", fn); return PSB_EINVAL; }
    if (q < 0) { psb_set_error("%s: q=%lld < 0", fn, (long long)q); return PSB_EINVAL; }
    if (k < 1) { psb_set_error("%s: k=%d < 1", fn, k); return PSB_EINVAL; }
    if (k > PSB_KMAX) { psb_set_error("%s: k=%d > PSB_KMAX=%d", fn, k, PSB_KMAX); return PSB_EUNSUPPORTED; }
    if (q > 0 && (!queries || !oi || !od)) { psb_set_error("%s: NULL buffer", fn); return PSB_EINVAL; }
    if (q > ((int64_t)1 << 40)) { psb_set_error("%s: q=%lld too large", fn, (long long)q); return PSB_EINVAL; }
    int dev = -1;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return report_cuda(e, fn);
    if (dev != ix->device) {
        psb_set_error("%s: index lives on device %d but device %d is current", fn, ix->device, dev);
        return PSB_EINVAL;
    }
    return PSB_OK;
}

static bool is_device_ptr(const void *p)
{
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// true for device (or managed) memory; otherwise *mapped = the device address of
// page-locked (pinned or registered) host memory registered by device `dev`'s
// context, nullptr for pageable memory (or memory pinned by another device's
// context, which is then staged like pageable memory).
static bool ptr_info(const void *p, int dev, void **mapped)
{
    *mapped = nullptr;
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) return true;
    if (a.type == cudaMemoryTypeHost && a.device == dev) *mapped = a.devicePointer;
    return false;
}

// Largest batch whose pinned host queries the kernels read in place (knn_impl).
constexpr int64_t ZERO_COPY_MAX_QUERIES = 16384;

// Launch one algorithm on device buffers. Host buffers: pinned ones are used in
// place by the kernels (zero-copy queries and result rows), pageable ones are
// staged through stream-ordered device scratch with copies on the same stream.
static int knn_impl(const char *fn, const psb_index *ix, const float *queries, int64_t q, int32_t k,
                    int32_t *out_ids, float *out_dists, void *stream, int32_t algo, uint32_t variant,
                    int64_t *stats, int parts = 1, TraceOut tr = TraceOut{nullptr, nullptr, 0})
{
    g_err[0] = 0;
    int rc = check_query_args(fn, ix, queries, q, k, out_ids, out_dists);
    if (rc != PSB_OK) return rc;
    if (variant & ~(uint32_t)(PSB_VAR_NOCACHE | PSB_VAR_NOMAXDIST | PSB_VAR_INPUT_ORDER | PSB_VAR_LEAF_ORDER |
                              PSB_VAR_PREFETCH_NEXT | PSB_VAR_PREFETCH_IDS | PSB_VAR_P1_INDEX_TIE |
                              PSB_VAR_KTH_MAXDIST | PSB_VAR_NO_AUTO_PREFETCH | PSB_VAR_GENERIC_D)) {
        psb_set_error("%s: unknown variant bits 0x%x", fn, variant);
        return PSB_EINVAL;
    }
    if (algo != PSB_ALGO_PSB && algo != PSB_ALGO_BNB && algo != PSB_ALGO_BRUTE) {
        psb_set_error("%s: unknown algo %d", fn, algo);
        return PSB_EINVAL;
    }
    if ((stats || tr.len) && algo == PSB_ALGO_BRUTE) {
        psb_set_error("%s: stats are defined for the tree traversals only", fn);
        return PSB_EINVAL;
    }
    if (q == 0) return PSB_OK;
    cudaStream_t st = (cudaStream_t)stream;
    // one attribute query per pointer: device memory, or the device address of
    // page-locked host memory (nullptr for pageable memory)
    void *mq_dev = nullptr, *mi_dev = nullptr, *md_dev = nullptr;
    const bool hq = !ptr_info(queries, ix->device, &mq_dev);
    const bool hi = !ptr_info(out_ids, ix->device, &mi_dev), hd = !ptr_info(out_dists, ix->device, &md_dev);
    bool hq_mapped = false;
    const bool ho = hi || hd;
    const float *dq = queries;
    int32_t *di = out_ids;
    float *dd = out_dists;
    cudaError_t e = cudaSuccess;
    const size_t bq = sizeof(float) * (size_t)(q * ix->d), bo = sizeof(float) * (size_t)(q * k);
    // Pinned host queries of a small batch are read by the tree kernels in place
    // (zero-copy: each warp loads its query's d floats over the host link), so
    // nothing is staged and no copy precedes the first kernel: C2's e2e
    // 47.7 -> 50.5 M q/s, single-query p50 -10 us. They are staged (one bulk copy
    // on the stream) when many warps read each query (split mode: a query per
    // part; brute force: a query per chunk CTA; host-link reads of one address by
    // thousands of warps cost C3's latency mode 15 us, r02bn) and for large
    // batches, where 10^6 small host-link reads (the closest-leaf pre-pass and the
    // traversal each read every query) cost more than one copy (C5 slab e2e
    // 97.8 -> 92.4 M q/s, r02bv). Pageable queries are always staged.
    bool staged_q = false;
    if (hq && mq_dev && parts <= 1 && algo != PSB_ALGO_BRUTE && q <= ZERO_COPY_MAX_QUERIES) {
        dq = static_cast<const float *>(mq_dev);
        hq_mapped = true;
    }
    if (hq && !hq_mapped) {
        staged_q = true;
        float *tmp = nullptr;
        if ((e = cudaMallocFromPoolAsync((void **)&tmp, bq, ix->pool, st)) != cudaSuccess) return report_cuda(e, fn);
        if ((e = cudaMemcpyAsync(tmp, queries, bq, cudaMemcpyHostToDevice, st)) != cudaSuccess) {
            cudaFreeAsync(tmp, st);
            return report_cuda(e, fn);
        }
        dq = tmp;
    }
    // Pinned host outputs: the kernels store each finished row straight into host
    // memory (zero-copy, over PCIe/C2C while the batch runs) instead of staging
    // the whole result for a copy after the last query; pageable ones are staged.
    bool staged = ho;
    if (ho) {
        int32_t *mi = !hi ? out_ids : static_cast<int32_t *>(mi_dev);
        float *md = !hd ? out_dists : static_cast<float *>(md_dev);
        if (mi && md) {
            di = mi;
            dd = md;
            staged = false;
        }
    }
    if (staged) {
        if ((e = cudaMallocFromPoolAsync((void **)&di, bo, ix->pool, st)) != cudaSuccess ||
            (e = cudaMallocFromPoolAsync((void **)&dd, bo, ix->pool, st)) != cudaSuccess)
            rc = report_cuda(e, fn);
    }
    if (rc == PSB_OK) {
        const DevIndex v = dev_view(ix);
        rc = algo == PSB_ALGO_BRUTE ? psb::launch_brute(v, dq, q, k, di, dd, st, ix->sm_count, ix->pool)
                                    : psb::launch_tree(algo, v, dq, q, k, di, dd, st, variant, stats, ix->pool, parts, tr);
    }
    if (staged) {
        if (rc == PSB_OK && ((e = cudaMemcpyAsync(out_ids, di, bo, cudaMemcpyDeviceToHost, st)) != cudaSuccess ||
                             (e = cudaMemcpyAsync(out_dists, dd, bo, cudaMemcpyDeviceToHost, st)) != cudaSuccess))
            rc = report_cuda(e, fn);
        if (di != out_ids) cudaFreeAsync(di, st);
        if (dd != out_dists) cudaFreeAsync(dd, st);
    }
    if (staged_q) cudaFreeAsync((void *)dq, st);
    return rc;
}

int psb_knn_ex(const psb_index *ix, const float *queries, int64_t q, int32_t k, int32_t *out_ids,
               float *out_dists, void *stream, int32_t algo, uint32_t variant)
{
    return knn_impl("psb_knn_ex", ix, queries, q, k, out_ids, out_dists, stream, algo, variant, nullptr);
}

int psb_knn_stats(const psb_index *ix, const float *queries, int64_t q, int32_t k, int32_t *out_ids,
                  float *out_dists, void *stream, int32_t algo, uint32_t variant, int64_t *stats)
{
    if (!stats && q > 0) { psb_set_error("psb_knn_stats: stats is NULL"); return PSB_EINVAL; }
    if (stats && q > 0 && !is_device_ptr(stats)) {
        psb_set_error("psb_knn_stats: stats must be device memory");
        return PSB_EINVAL;
    }
    return knn_impl("psb_knn_stats", ix, queries, q, k, out_ids, out_dists, stream, algo, variant, stats);
}

int psb_knn_trace(const psb_index *ix, const float *queries, int64_t q, int32_t k, int32_t *out_ids,
                  float *out_dists, void *stream, int32_t algo, uint32_t variant, int64_t *stats, int64_t *trace,
                  int32_t cap, int32_t *trace_len)
{
    if (q > 0 && (!trace || !trace_len || cap < 1)) {
        psb_set_error("psb_knn_trace: trace / trace_len NULL or cap < 1");
        return PSB_EINVAL;
    }
    if (q > 0 && (!is_device_ptr(trace) || !is_device_ptr(trace_len) || (stats && !is_device_ptr(stats)))) {
        psb_set_error("psb_knn_trace: trace, trace_len and stats must be device memory");
        return PSB_EINVAL;
    }
    return knn_impl("psb_knn_trace", ix, queries, q, k, out_ids, out_dists, stream, algo, variant, stats, 1,
                    TraceOut{trace, trace_len, cap});
}

int psb_knn_split(const psb_index *ix, const float *queries, int64_t q, int32_t k, int32_t parts,
                  int32_t *out_ids, float *out_dists, void *stream)
{
    if (parts < 0) { psb_set_error("psb_knn_split: parts=%d < 0", parts); return PSB_EINVAL; }
    if (ix && parts == 0) {
        // auto (DESIGN.md §6 "split mode"):
        //  - few queries (<= 1/4 of the resident warps): latency mode, about 16
        //    warps per SM in total, at least 16 leaves per part, when the
        //    estimated leaves per query (below) reach 16;
        //  - a batch that fills the GPU less than 4 times over, of queries that
        //    touch many leaves: 2-8 parts per query against the batch's tail. The
        //    work per query is estimated by the classic uniform-data cost model
        //    (1 + (k'/F)^(1/d))^d leaves (k' = min(k, F)): >= 64 splits;
        //  - otherwise 1 (plain psb_knn).
        const int64_t resident = (int64_t)ix->sm_count * 32;
        const double kf = (double)(k < ix->F ? k : ix->F) / ix->F;
        const double work = std::pow(1.0 + std::pow(kf, 1.0 / ix->d), (double)ix->d);
        int64_t p = 1;
        if (q * 4 <= resident) {
            if (work >= 16.0) {                   // else one warp is faster than the split's overhead
                p = q > 0 ? (int64_t)ix->sm_count * 16 / q : 1;
                const int64_t pmax = ix->L / 16;     // C3: 1,953 parts, p50 72 us (976: 79; r02de)
                if (p > pmax) p = pmax;
            }
        } else if (q < 4 * resident) {
            if (work >= 64.0) {
                p = 14 * resident / q;             // C4: 6 parts (8.11 ms; 5: 8.33, 7: 8.13, 8: 8.45; r02by)
                p = p < 2 ? 2 : (p > 8 ? 8 : p);
            }
        }
        parts = (int32_t)(p < 1 ? 1 : p);
    }
    if (ix && parts > ix->L) parts = (int32_t)ix->L;
    return knn_impl("psb_knn_split", ix, queries, q, k, out_ids, out_dists, stream, PSB_ALGO_PSB, 0, nullptr,
                    parts < 1 ? 1 : parts);
}

int psb_knn(const psb_index *ix, const float *queries, int64_t q, int32_t k, int32_t *out_ids,
            float *out_dists, void *stream)
{
    return knn_impl("psb_knn", ix, queries, q, k, out_ids, out_dists, stream, PSB_ALGO_PSB, 0, nullptr);
}

int psb_knn_branch_and_bound(const psb_index *ix, const float *queries, int64_t q, int32_t k,
                             int32_t *out_ids, float *out_dists, void *stream)
{
    return knn_impl("psb_knn_branch_and_bound", ix, queries, q, k, out_ids, out_dists, stream, PSB_ALGO_BNB,
                    0, nullptr);
}

int psb_knn_bruteforce(const psb_index *ix, const float *queries, int64_t q, int32_t k,
                       int32_t *out_ids, float *out_dists, void *stream)
{
    return knn_impl("psb_knn_bruteforce", ix, queries, q, k, out_ids, out_dists, stream, PSB_ALGO_BRUTE,
                    0, nullptr);
}

int psb_merge_topk(const int32_t *ids, const float *dists, int32_t parts, int64_t q, int32_t k,
                   int32_t *out_ids, float *out_dists, void *stream)
{
    g_err[0] = 0;
    if (parts < 1 || q < 0 || k < 1) {
        psb_set_error("psb_merge_topk: parts=%d q=%lld k=%d out of range", parts, (long long)q, k);
        return PSB_EINVAL;
    }
    if (k > PSB_KMAX) { psb_set_error("psb_merge_topk: k=%d > PSB_KMAX", k); return PSB_EUNSUPPORTED; }
    if (q == 0) return PSB_OK;
    if (!ids || !dists || !out_ids || !out_dists) { psb_set_error("psb_merge_topk: NULL buffer"); return PSB_EINVAL; }
    return psb::launch_merge(ids, dists, parts, q, k, out_ids, out_dists, (cudaStream_t)stream);
}

int psb_index_info(const psb_index *ix, int64_t *n, int32_t *d, int32_t *fanout, int64_t *leaves,
                   int32_t *levels, int64_t *device_bytes)
{
    if (!ix) { psb_set_error("psb_index_info: index is NULL"); return PSB_EINVAL; }
    if (n) *n = ix->n;
    if (d) *d = ix->d;
    if (fanout) *fanout = ix->F;
    if (leaves) *leaves = ix->L;
    if (levels) *levels = ix->H;
    if (device_bytes) *device_bytes = ix->device_bytes;
    return PSB_OK;
}

static int64_t blob_size(int64_t L, int32_t d, int32_t F, int32_t H, int64_t node_floats)
{
    return 8 * 8 + 8 * (int64_t)(H + 1) + 4 * L * d * F + 4 * L * F + 4 * node_floats;
}

static void blob_header(char *buf, int64_t n, int32_t d, int32_t F, int64_t L, int32_t H, int64_t id_base,
                        const int64_t *nlev, int32_t sphere = 0)
{
    int64_t total = 0;
    for (int l = 1; l <= H; ++l) total += nlev[l];
    int64_t hdr[8] = {n, d, F, L, H, id_base, total, sphere};
    memcpy(buf, hdr, sizeof hdr);
    memcpy(buf + sizeof hdr, nlev, 8 * (size_t)(H + 1));
}

int psb_index_export(const psb_index *ix, void *host_buf, int64_t cap, int64_t *used)
{
    if (!ix || !used) { psb_set_error("psb_index_export: NULL argument"); return PSB_EINVAL; }
    const int64_t need = blob_size(ix->L, ix->d, ix->F, ix->H, ix->node_floats);
    *used = need;
    if (!host_buf) return PSB_OK;
    if (cap < need) { psb_set_error("psb_index_export: cap %lld < %lld", (long long)cap, (long long)need); return PSB_EINVAL; }
    char *b = (char *)host_buf;
    blob_header(b, ix->n, ix->d, ix->F, ix->L, ix->H, ix->id_base, ix->nlev, ix->sphere);
    char *p = b + 64 + 8 * (ix->H + 1);
    const size_t bp = 4 * (size_t)(ix->L * ix->d * ix->F), bi = 4 * (size_t)(ix->L * ix->F);
    cudaError_t e;
    if ((e = cudaMemcpy(p, ix->pts, bp, cudaMemcpyDeviceToHost)) != cudaSuccess ||
        (e = cudaMemcpy(p + bp, ix->ids, bi, cudaMemcpyDeviceToHost)) != cudaSuccess ||
        (e = cudaMemcpy(p + bp + bi, ix->nodes, 4 * (size_t)ix->node_floats, cudaMemcpyDeviceToHost)) != cudaSuccess)
        return report_cuda(e, "psb_index_export");
    return PSB_OK;
}

// Upload an export blob as an index (replicas: build once, broadcast the blob;
// tests: hand-built trees). Everything the exactness argument rests on is
// checked first: the level geometry of a packed tree, finite coordinates for
// real points and +inf for pad slots (id -1), and every box containing what is
// below it (App. C of SURVEY.md: then MINDIST <= dist <= MAXDIST holds under
// RN rounding for every point beneath).
int psb_index_import(const void *blob, int64_t size, psb_index **out)
{
    g_err[0] = 0;
    if (!out || !blob) { psb_set_error("psb_index_import: NULL argument"); return PSB_EINVAL; }
    *out = nullptr;
    if (size < 64) { psb_set_error("psb_index_import: blob too small"); return PSB_EINVAL; }
    const char *b = (const char *)blob;
    int64_t hdr[8];
    memcpy(hdr, b, sizeof hdr);
    const int64_t n_hdr = hdr[0], L = hdr[3], id_base = hdr[5], total = hdr[6];
    const int64_t d64 = hdr[1], F64 = hdr[2], H64 = hdr[4];
    if (hdr[7] != 0) { psb_set_error("psb_index_import: sphere indexes cannot be imported"); return PSB_EUNSUPPORTED; }
    if (d64 < 1 || d64 > PSB_DMAX || H64 < 1 || H64 > PSB_MAXLVL || L < 1 || L > ((int64_t)1 << 31) / 32) {
        psb_set_error("psb_index_import: header out of range");
        return PSB_EINVAL;
    }
    const int32_t d = (int32_t)d64, F = (int32_t)F64, H = (int32_t)H64;
    GpuLayoutShape shape;
    int rc = psb_layout_shape(L * F64, d, F, 0, 0, &shape);   // validates d and F
    if (rc != PSB_OK) return rc;
    if (size < 64 + 8 * (H64 + 1)) { psb_set_error("psb_index_import: blob too small"); return PSB_EINVAL; }
    int64_t nlev[PSB_MAXLVL + 1] = {};
    memcpy(nlev, b + 64, 8 * (size_t)(H + 1));
    if (shape.H != H || shape.L != L || shape.total_node_floats / (2 * d64 * F64) != total) {
        psb_set_error("psb_index_import: level geometry is not that of a packed tree with %lld leaves", (long long)L);
        return PSB_EINVAL;
    }
    for (int l = 0; l <= H; ++l)
        if (nlev[l] != shape.nlev[l]) { psb_set_error("psb_index_import: nodes_per_level[%d] wrong", l); return PSB_EINVAL; }
    if (size != blob_size(L, d, F, H, shape.total_node_floats)) {
        psb_set_error("psb_index_import: size %lld does not match the header", (long long)size);
        return PSB_EINVAL;
    }
    const float *pts = (const float *)(b + 64 + 8 * (H + 1));
    const int32_t *ids = (const int32_t *)(pts + L * d64 * F64);
    const float *nodes = (const float *)(ids + L * F64);
    // points: real slots finite with an id >= 0, pad slots +inf with id -1
    int64_t n_real = 0;
    bool irregular = false;
    for (int64_t j = 0; j < L; ++j) {
        int64_t cnt = 0;
        for (int s = 0; s < F; ++s) {
            const int32_t id = ids[j * F + s];
            if (id < -1) { psb_set_error("psb_index_import: id %d < -1", id); return PSB_EINVAL; }
            for (int c = 0; c < d; ++c) {
                const float v = pts[(j * d + c) * F + s];
                if (id >= 0 ? !std::isfinite(v) : !(std::isinf(v) && v > 0)) {
                    psb_set_error("psb_index_import: leaf %lld slot %d: coordinates must be finite for a point "
                                  "and +inf for a pad slot", (long long)j, s);
                    return PSB_EINVAL;
                }
            }
            cnt += id >= 0;
        }
        n_real += cnt;
        if (j + 1 < L && cnt < F) irregular = true;
    }
    if (n_real != n_hdr || n_real < 1) {
        psb_set_error("psb_index_import: header n=%lld but %lld real points", (long long)n_hdr, (long long)n_real);
        return PSB_EINVAL;
    }
    // boxes: child c of node (l, i) is (l-1, i*F + c); its box must contain the
    // points of leaf i*F + c (l = 1) or the boxes of that node's children (l >= 2)
    const int64_t blk = 2 * d64 * F64;
    for (int l = 1; l <= H; ++l) {
        const float *cur = nodes + shape.level_off[l];
        for (int64_t i = 0; i < nlev[l]; ++i) {
            for (int c = 0; c < F; ++c) {
                const int64_t g = i * F + c;
                for (int dd = 0; dd < d; ++dd) {
                    const float lo = cur[i * blk + (2 * dd) * F + c], hi = cur[i * blk + (2 * dd + 1) * F + c];
                    if (std::isnan(lo) || std::isnan(hi)) { psb_set_error("psb_index_import: NaN box"); return PSB_EINVAL; }
                    float mn = INFINITY, mx = -INFINITY;
                    if (g < nlev[l - 1]) {
                        if (l == 1) {
                            for (int s = 0; s < F; ++s)
                                if (ids[g * F + s] >= 0) {
                                    mn = std::min(mn, pts[(g * d + dd) * F + s]);
                                    mx = std::max(mx, pts[(g * d + dd) * F + s]);
                                }
                        } else {
                            const float *cb = nodes + shape.level_off[l - 1] + g * blk;
                            for (int s = 0; s < F; ++s) {
                                mn = std::min(mn, cb[(2 * dd) * F + s]);
                                mx = std::max(mx, cb[(2 * dd + 1) * F + s]);
                            }
                        }
                    }
                    const bool empty = mn > mx;
                    if (empty ? !(std::isinf(lo) && lo > 0 && std::isinf(hi) && hi < 0) : (lo > mn || hi < mx)) {
                        psb_set_error("psb_index_import: box of child %d of node %lld at level %d does not bound "
                                      "its content (dim %d)", c, (long long)i, l, dd);
                        return PSB_EINVAL;
                    }
                }
            }
        }
    }
    int dev = -1;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return report_cuda(e, "psb_index_import: cudaGetDevice");
    psb_index *ix = new (std::nothrow) psb_index;
    if (!ix) { psb_set_error("psb_index_import: host allocation failed"); return PSB_ENOMEM; }
    ix->device = dev;
    cudaDeviceGetAttribute(&ix->sm_count, cudaDevAttrMultiProcessorCount, dev);
    ix->n = n_real; ix->L = L; ix->id_base = id_base;
    ix->d = d; ix->F = F; ix->H = H;
    for (int l = 0; l <= PSB_MAXLVL; ++l) { ix->nlev[l] = shape.nlev[l]; ix->level_off[l] = shape.level_off[l]; }
    ix->node_floats = shape.total_node_floats;
    ix->blk_floats = (int32_t)blk;
    ix->irregular = irregular ? 1 : 0;
    const size_t bp = 4 * (size_t)(L * d64 * F64), bi = 4 * (size_t)(L * F64), bn = 4 * (size_t)shape.total_node_floats;
    if ((e = cudaMalloc((void **)&ix->pts, bp)) != cudaSuccess || (e = cudaMalloc((void **)&ix->ids, bi)) != cudaSuccess ||
        (e = cudaMalloc((void **)&ix->nodes, bn)) != cudaSuccess ||
        (e = cudaMemcpy(ix->pts, pts, bp, cudaMemcpyHostToDevice)) != cudaSuccess ||
        (e = cudaMemcpy(ix->ids, ids, bi, cudaMemcpyHostToDevice)) != cudaSuccess ||
        (e = cudaMemcpy(ix->nodes, nodes, bn, cudaMemcpyHostToDevice)) != cudaSuccess) {
        rc = report_cuda(e, "psb_index_import: upload");
        index_release(ix);
        return rc;
    }
    ix->device_bytes = (int64_t)(bp + bi + bn);
    if ((rc = attach_box(ix, "psb_index_import: bounding box")) != PSB_OK ||
        (rc = make_pool(ix, "psb_index_import")) != PSB_OK) {
        index_release(ix);
        return rc;
    }
    *out = ix;
    return PSB_OK;
}

// Host-only bulk load into the export blob layout (no CUDA calls): lets the CPU
// test suite check the layout logic; the GPU tests check psb_index_export of a
// real index against it.
int psb_build_host_blob(const float *points, int64_t n, int32_t d, int32_t fanout, int64_t id_base,
                        uint32_t flags, void *host_buf, int64_t cap, int64_t *used)
{
    g_err[0] = 0;
    if (!used) { psb_set_error("psb_build_host_blob: used is NULL"); return PSB_EINVAL; }
    HostLayout h;
    int rc = psb_host_build(points, n, d, fanout, id_base, flags, &h);
    if (rc != PSB_OK) return rc;
    const int64_t need = blob_size(h.L, h.d, h.F, h.H, h.total_node_floats);
    *used = need;
    if (!host_buf) return PSB_OK;
    if (cap < need) { psb_set_error("psb_build_host_blob: cap too small"); return PSB_EINVAL; }
    char *b = (char *)host_buf;
    blob_header(b, h.n, h.d, h.F, h.L, h.H, h.id_base, h.nlev);
    char *p = b + 64 + 8 * (h.H + 1);
    const size_t bp = 4 * (size_t)(h.L * h.d * h.F), bi = 4 * (size_t)(h.L * h.F);
    memcpy(p, h.pts, bp);
    memcpy(p + bp, h.ids, bi);
    memcpy(p + bp + bi, h.nodes, 4 * (size_t)h.total_node_floats);
    return PSB_OK;
}

}  // extern "C"
