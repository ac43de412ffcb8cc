// knn_exchange.cu — data-sharded exchange fused into the merge, over peer memory.
//
// North_star / SURVEY.md §8(e): in data-sharded mode every GPU answers all q
// queries over its own slab, and each GPU then needs, for the queries it owns,
// the P per-shard top-k lists merged into one. The NCCL route gathers all q
// rows of every shard onto every rank (P*q*k*8 bytes in per rank) and merges.
// Here the merge kernel itself pulls only the rows it owns straight out of the
// peers' result buffers through CUDA IPC mappings (NVLink/NVSwitch loads,
// q*k*8 bytes in per rank, no staging copy, no collective launch).
//
// Protocol (include/psb.h): a rank's progress is one 64-bit flag value
// (epoch << 32 | rows done), stored with release semantics (system scope) into
// its slot of every peer's flag array by psb_exchange_signal, stream-ordered
// after the local search of a chunk of rows. psb_exchange_merge launches
//   1. wait_kernel: ONE thread polls the P slots of this rank's flags until all
//      reach (epoch << 32 | row_end) (acquire), with a single deadline per
//      launch; on timeout (or if an earlier launch already timed out) it sets
//      the exchange's status word, on the device and in mapped host memory;
//   2. merge_peers_kernel (stream-ordered after it): one warp per owned row
//      reads the P lists from peer memory and merges them; when the status is
//      set it writes (-1, +inf) pad rows instead and reads no peer memory.
// The host checks the mapped status word at every call: once a wait has timed
// out, every later psb_exchange_* call returns PSB_ECUDA (sticky).
// Result buffers alternate by epoch parity. A rank overwrites parity p at epoch
// e+2 only after its merge of epoch e+1 saw every peer signal e+1, which each
// peer does only after its merges of epoch e (stream order), i.e. after it
// stopped reading the epoch-e buffers. The wait runs even when a rank owns no
// rows (rows == 0), so the argument holds for every rank.
#include <cuda_runtime.h>

#include <chrono>
#include <cstring>
#include <new>
#include <random>
#include <unistd.h>

#include "psb_device.cuh"
#include "psb_launch.h"

namespace psb {

struct ExBlob {                    // what a rank publishes (psb_exchange_handle)
    uint64_t magic;
    uint64_t nonce[2];             // identifies the publishing process (not its pid)
    int32_t device, rank, parts, k;
    int64_t q;
    uint64_t raw[5];               // ids0, ids1, d0, d1, flags (valid in the owning process)
    cudaIpcMemHandle_t h[5];
};
constexpr uint64_t EX_MAGIC = 0x5053424558434832ull;   // "PSBEXCH2"
constexpr int64_t EX_DEFAULT_TIMEOUT_NS = 10ll * 1000 * 1000 * 1000;

// Random per-process identity: two processes in different PID namespaces can
// share a pid, so the pid alone cannot tell that a blob's raw pointers are ours.
static const uint64_t *process_nonce()
{
    static uint64_t n[2] = {0, 0};
    static bool init = false;
    if (!init) {
        std::random_device rd;
        const uint64_t t = (uint64_t)std::chrono::high_resolution_clock::now().time_since_epoch().count();
        n[0] = ((uint64_t)rd() << 32 | rd()) ^ t;
        n[1] = ((uint64_t)rd() << 32 | rd()) ^ ((uint64_t)getpid() << 17) ^ (uint64_t)(uintptr_t)&n;
        init = true;
    }
    return n;
}

struct PeerLists {
    const int32_t *ids[PSB_MAX_PARTS];
    const float *dists[PSB_MAX_PARTS];
};

struct FlagPtrs {
    unsigned long long *p[PSB_MAX_PARTS];
};

__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v)
{
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Stream-ordered after this rank's local search of a chunk: publish progress to every peer.
__global__ void signal_kernel(FlagPtrs fl, int parts, int self, unsigned long long value)
{
    __threadfence_system();
    for (int p = threadIdx.x; p < parts; p += blockDim.x) st_release_sys(fl.p[p] + self, value);
}

// One thread waits for every part's flag to reach `target`, with one deadline
// for the whole launch. A status already set by an earlier launch ends the wait
// at once (a dead peer costs one timeout, not one per step).
__global__ void wait_kernel(const unsigned long long *flags, int parts, unsigned long long target,
                            int64_t timeout_ns, int32_t *status_dev, volatile int32_t *status_host)
{
    if (threadIdx.x != 0) return;
    if (*(volatile int32_t *)status_dev) return;
    const int64_t t0 = global_ns();
    for (int p = 0; p < parts; ++p) {
        while (ld_acquire_sys(flags + p) < target) {
            if (global_ns() - t0 > timeout_ns || *(volatile int32_t *)status_dev) {
                *(volatile int32_t *)status_dev = 1;
                *status_host = 1;
                __threadfence_system();
                return;
            }
            __nanosleep(200);
        }
    }
}

// Gather + merge, one warp per owned row, stream-ordered after wait_kernel.
template <int KS>
__global__ void __launch_bounds__(128)
merge_peers_kernel(PeerLists src, int parts, int64_t row0, int64_t rows, int k, const int32_t *__restrict__ status,
                   int32_t *__restrict__ out_ids, float *__restrict__ out_dists)
{
    __shared__ u64 scratch_all[4][32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t r = (int64_t)blockIdx.x * 4 + w;
    if (r >= rows) return;
    TopK<KS> T;
    T.init();
    if (!*(volatile const int32_t *)status) {
        const int64_t row = row0 + r;
        u64 thr = PAD_KEY;
        for (int p = 0; p < parts; ++p) {
            const int32_t *pi = src.ids[p] + row * k;
            const float *pd = src.dists[p] + row * k;
            u64 cand[KS];
#pragma unroll
            for (int s = 0; s < KS; ++s) {
                const int c = s * 32 + lane;
                // peer memory: plain (coherent) loads, not the read-only path
                cand[s] = c < k ? make_key(__ldcv(pd + c), __ldcv(pi + c)) : ~0ull;
            }
            T.template offer<KS>(cand, k, lane, thr, scratch_all[w]);
        }
    }
    T.store(k, lane, out_ids + r * k, out_dists + r * k);   // pad rows (-1, +inf) after a timeout
}

}  // namespace psb

using namespace psb;

struct psb_exchange {
    int device = -1;
    int parts = 0, rank = 0;
    int64_t q = 0;
    int k = 0;
    int64_t timeout_ns = EX_DEFAULT_TIMEOUT_NS;
    int32_t *ids[2] = {nullptr, nullptr};     // own [q][k] result lists, by epoch parity
    float *dists[2] = {nullptr, nullptr};
    unsigned long long *flags = nullptr;      // own [parts] flag slots (peer r writes slot r)
    int32_t *status = nullptr;                // device word: 1 = a wait timed out
    int32_t *status_host = nullptr;           // mapped pinned host copy (read by the host, no sync)
    int32_t *status_host_dev = nullptr;       // its device address
    // peers' buffers as mapped into this process (own entries for self)
    int32_t *peer_ids[PSB_MAX_PARTS][2] = {};
    float *peer_dists[PSB_MAX_PARTS][2] = {};
    unsigned long long *peer_flags[PSB_MAX_PARTS] = {};
    bool opened[PSB_MAX_PARTS] = {};          // mapped with cudaIpcOpenMemHandle (closed on free)
};

static void ex_release(psb_exchange *x)
{
    if (!x) return;
    int prev = -1;
    cudaGetDevice(&prev);
    if (x->device >= 0) cudaSetDevice(x->device);
    for (int p = 0; p < x->parts; ++p) {
        if (!x->opened[p]) continue;
        for (int e = 0; e < 2; ++e) {
            cudaIpcCloseMemHandle(x->peer_ids[p][e]);
            cudaIpcCloseMemHandle(x->peer_dists[p][e]);
        }
        cudaIpcCloseMemHandle(x->peer_flags[p]);
    }
    for (int e = 0; e < 2; ++e) {
        cudaFree(x->ids[e]);
        cudaFree(x->dists[e]);
    }
    cudaFree(x->flags);
    cudaFree(x->status);
    if (x->status_host) cudaFreeHost(x->status_host);
    if (prev >= 0) cudaSetDevice(prev);
    delete x;
}

// Sticky failure: a wait that timed out leaves the exchange unusable.
static int ex_check(const psb_exchange *x, const char *fn)
{
    if (x->status_host && *(volatile int32_t *)x->status_host) {
        psb_set_error("%s: an earlier exchange wait timed out (a peer never signalled); "
                      "the exchange is unusable, free and recreate it", fn);
        return PSB_ECUDA;
    }
    return PSB_OK;
}

static int ex_connected(const psb_exchange *x, const char *fn)
{
    for (int p = 0; p < x->parts; ++p)
        if (!x->peer_flags[p]) { psb_set_error("%s: not connected", fn); return PSB_EINVAL; }
    return PSB_OK;
}

extern "C" {

int psb_exchange_create(int32_t parts, int32_t rank, int64_t q, int32_t k, psb_exchange **out)
{
    if (!out) { psb_set_error("psb_exchange_create: out is NULL"); return PSB_EINVAL; }
    *out = nullptr;
    if (parts < 1 || parts > PSB_MAX_PARTS || rank < 0 || rank >= parts || q < 1 || q >= (1ll << 32) || k < 1 ||
        k > 128) {
        psb_set_error("psb_exchange_create: parts=%d rank=%d q=%lld k=%d out of range", parts, rank, (long long)q, k);
        return PSB_EINVAL;
    }
    psb_exchange *x = new (std::nothrow) psb_exchange;
    if (!x) { psb_set_error("psb_exchange_create: host allocation failed"); return PSB_ENOMEM; }
    cudaGetDevice(&x->device);
    x->parts = parts; x->rank = rank; x->q = q; x->k = k;
    const size_t b = (size_t)q * k * 4;
    cudaError_t e = cudaSuccess;
    for (int i = 0; i < 2 && e == cudaSuccess; ++i) {
        if ((e = cudaMalloc((void **)&x->ids[i], b)) == cudaSuccess) e = cudaMalloc((void **)&x->dists[i], b);
    }
    if (e == cudaSuccess) e = cudaMalloc((void **)&x->flags, 8 * (size_t)parts);
    if (e == cudaSuccess) e = cudaMalloc((void **)&x->status, 4);
    if (e == cudaSuccess) e = cudaHostAlloc((void **)&x->status_host, 4, cudaHostAllocMapped);
    if (e == cudaSuccess) e = cudaHostGetDevicePointer((void **)&x->status_host_dev, x->status_host, 0);
    if (e == cudaSuccess) e = cudaMemset(x->flags, 0, 8 * (size_t)parts);
    if (e == cudaSuccess) e = cudaMemset(x->status, 0, 4);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
        int rc = report_cuda(e, "psb_exchange_create");
        ex_release(x);
        return rc;
    }
    *x->status_host = 0;
    *out = x;
    return PSB_OK;
}

int psb_exchange_set_timeout(psb_exchange *x, int64_t timeout_ns)
{
    if (!x || timeout_ns < 1) { psb_set_error("psb_exchange_set_timeout: bad argument"); return PSB_EINVAL; }
    x->timeout_ns = timeout_ns;
    return PSB_OK;
}

int psb_exchange_handle(const psb_exchange *x, void *buf, int64_t cap, int64_t *used)
{
    if (!x || !used) { psb_set_error("psb_exchange_handle: NULL argument"); return PSB_EINVAL; }
    *used = sizeof(ExBlob);
    if (!buf) return PSB_OK;
    if (cap < (int64_t)sizeof(ExBlob)) { psb_set_error("psb_exchange_handle: cap too small"); return PSB_EINVAL; }
    ExBlob bl;
    memset(&bl, 0, sizeof bl);
    bl.magic = EX_MAGIC;
    const uint64_t *nn = process_nonce();
    bl.nonce[0] = nn[0];
    bl.nonce[1] = nn[1];
    bl.device = x->device; bl.rank = x->rank; bl.parts = x->parts; bl.k = x->k; bl.q = x->q;
    void *ptrs[5] = {x->ids[0], x->ids[1], x->dists[0], x->dists[1], x->flags};
    for (int i = 0; i < 5; ++i) {
        bl.raw[i] = (uint64_t)(uintptr_t)ptrs[i];
        cudaError_t e = cudaIpcGetMemHandle(&bl.h[i], ptrs[i]);
        if (e != cudaSuccess) return report_cuda(e, "psb_exchange_handle: cudaIpcGetMemHandle");
    }
    memcpy(buf, &bl, sizeof bl);
    return PSB_OK;
}

int psb_exchange_connect(psb_exchange *x, const void *const *blobs)
{
    if (!x || !blobs) { psb_set_error("psb_exchange_connect: NULL argument"); return PSB_EINVAL; }
    const uint64_t *me = process_nonce();
    for (int p = 0; p < x->parts; ++p) {
        if (!blobs[p]) { psb_set_error("psb_exchange_connect: blob %d is NULL", p); return PSB_EINVAL; }
        ExBlob bl;
        memcpy(&bl, blobs[p], sizeof bl);
        if (bl.magic != EX_MAGIC || bl.rank != p || bl.parts != x->parts || bl.k != x->k || bl.q != x->q) {
            psb_set_error("psb_exchange_connect: blob %d does not match (rank/parts/q/k)", p);
            return PSB_EINVAL;
        }
        void *ptrs[5];
        if (bl.nonce[0] == me[0] && bl.nonce[1] == me[1]) {
            // same process: the raw pointers are valid; a buffer on another device
            // of this process needs peer access from ours
            if (bl.device != x->device) {
                cudaError_t e = cudaDeviceEnablePeerAccess(bl.device, 0);
                if (e == cudaErrorPeerAccessAlreadyEnabled) {
                    cudaGetLastError();
                } else if (e != cudaSuccess) {
                    return report_cuda(e, "psb_exchange_connect: cudaDeviceEnablePeerAccess");
                }
            }
            for (int i = 0; i < 5; ++i) ptrs[i] = (void *)(uintptr_t)bl.raw[i];
        } else {
            for (int i = 0; i < 5; ++i) {
                cudaError_t e = cudaIpcOpenMemHandle(&ptrs[i], bl.h[i], cudaIpcMemLazyEnablePeerAccess);
                if (e != cudaSuccess) {
                    for (int j = 0; j < i; ++j) cudaIpcCloseMemHandle(ptrs[j]);
                    return report_cuda(e, "psb_exchange_connect: cudaIpcOpenMemHandle");
                }
            }
            x->opened[p] = true;
        }
        x->peer_ids[p][0] = (int32_t *)ptrs[0];
        x->peer_ids[p][1] = (int32_t *)ptrs[1];
        x->peer_dists[p][0] = (float *)ptrs[2];
        x->peer_dists[p][1] = (float *)ptrs[3];
        x->peer_flags[p] = (unsigned long long *)ptrs[4];
    }
    return PSB_OK;
}

int psb_exchange_buffers(const psb_exchange *x, int64_t epoch, int32_t **ids, float **dists)
{
    if (!x || !ids || !dists || epoch < 1) { psb_set_error("psb_exchange_buffers: bad argument"); return PSB_EINVAL; }
    int rc = ex_check(x, "psb_exchange_buffers");
    if (rc != PSB_OK) return rc;
    *ids = x->ids[epoch & 1];
    *dists = x->dists[epoch & 1];
    return PSB_OK;
}

int psb_exchange_signal(psb_exchange *x, int64_t epoch, int64_t rows_done, void *stream)
{
    if (!x || epoch < 1 || epoch > 0x7fffffffll || rows_done < 1 || rows_done > x->q) {
        psb_set_error("psb_exchange_signal: bad argument");
        return PSB_EINVAL;
    }
    int rc = ex_check(x, "psb_exchange_signal");
    if (rc == PSB_OK) rc = ex_connected(x, "psb_exchange_signal");
    if (rc != PSB_OK) return rc;
    FlagPtrs fl;
    memset(&fl, 0, sizeof fl);
    for (int p = 0; p < x->parts; ++p) fl.p[p] = x->peer_flags[p];
    const unsigned long long v = ((unsigned long long)epoch << 32) | (unsigned long long)rows_done;
    signal_kernel<<<1, 32, 0, (cudaStream_t)stream>>>(fl, x->parts, x->rank, v);
    return report_cuda(cudaGetLastError(), "psb_exchange_signal");
}

int psb_exchange_merge(psb_exchange *x, int64_t epoch, int64_t row0, int64_t rows, int32_t *out_ids,
                       float *out_dists, void *stream)
{
    if (!x || epoch < 1 || epoch > 0x7fffffffll || row0 < 0 || rows < 0 || row0 + rows > x->q ||
        (rows > 0 && (!out_ids || !out_dists))) {
        psb_set_error("psb_exchange_merge: bad argument");
        return PSB_EINVAL;
    }
    int rc = ex_check(x, "psb_exchange_merge");
    if (rc == PSB_OK) rc = ex_connected(x, "psb_exchange_merge");
    if (rc != PSB_OK) return rc;
    cudaStream_t st = (cudaStream_t)stream;
    // every peer must have finished rows [0, row0+rows) of this epoch (>= 1 row:
    // even a rank with no rows waits for the epoch, see the header comment)
    const int64_t need = row0 + rows > 0 ? row0 + rows : 1;
    const unsigned long long target = ((unsigned long long)epoch << 32) | (unsigned long long)need;
    wait_kernel<<<1, 32, 0, st>>>(x->flags, x->parts, target, x->timeout_ns, x->status, x->status_host_dev);
    rc = report_cuda(cudaGetLastError(), "psb_exchange_merge: wait");
    if (rc != PSB_OK || rows == 0) return rc;
    PeerLists src;
    memset(&src, 0, sizeof src);
    for (int p = 0; p < x->parts; ++p) {
        src.ids[p] = x->peer_ids[p][epoch & 1];
        src.dists[p] = x->peer_dists[p][epoch & 1];
    }
    const unsigned blocks = (unsigned)((rows + 3) / 4);
    if (x->k <= 32)
        merge_peers_kernel<1><<<blocks, 128, 0, st>>>(src, x->parts, row0, rows, x->k, x->status, out_ids, out_dists);
    else if (x->k <= 64)
        merge_peers_kernel<2><<<blocks, 128, 0, st>>>(src, x->parts, row0, rows, x->k, x->status, out_ids, out_dists);
    else
        merge_peers_kernel<4><<<blocks, 128, 0, st>>>(src, x->parts, row0, rows, x->k, x->status, out_ids, out_dists);
    return report_cuda(cudaGetLastError(), "psb_exchange_merge: merge");
}

int psb_exchange_step(psb_exchange *x, int64_t epoch, int64_t row0, int64_t rows, int32_t *out_ids,
                      float *out_dists, void *stream)
{
    if (!x) { psb_set_error("psb_exchange_step: NULL exchange"); return PSB_EINVAL; }
    int rc = psb_exchange_signal(x, epoch, x->q, stream);
    if (rc != PSB_OK) return rc;
    return psb_exchange_merge(x, epoch, row0, rows, out_ids, out_dists, stream);
}

int psb_exchange_status(const psb_exchange *x, int32_t *timed_out)
{
    if (!x || !timed_out) { psb_set_error("psb_exchange_status: NULL argument"); return PSB_EINVAL; }
    *timed_out = *(volatile int32_t *)x->status_host;
    return PSB_OK;
}

void psb_exchange_free(psb_exchange *x) { ex_release(x); }

}  // extern "C"
