// knn_exchange.cu — data-sharded exchange fused into the merge, over peer memory.
//
// North_star / SURVEY.md §8(e): in data-sharded mode every GPU answers all q
// queries over its own slab, and each GPU then needs, for the q/P queries it
// owns, the P per-shard top-k lists merged into one. The NCCL route gathers all
// q rows of every shard onto every rank (P*q*k*8 bytes in per rank) and merges.
// Here the merge kernel itself pulls only the rows it owns straight out of the
// peers' result buffers through CUDA IPC mappings (NVLink/NVSwitch loads,
// q*k*8 bytes in per rank, no staging copy, no collective launch), after a
// device-side flag barrier: each rank, stream-ordered after its local search,
// stores the step's epoch into a flag slot on every peer (release, system
// scope); the merge kernel waits until all P slots of its own flag array reach
// the epoch (acquire) before it reads. Result buffers alternate by epoch parity,
// so a rank can start step e+1 while a slower peer is still reading step e
// (it cannot reach e+2 before that peer has signalled e+1, i.e. finished e).
#include <cuda_runtime.h>

#include <cstring>
#include <new>
#include <unistd.h>

#include "psb_device.cuh"
#include "psb_launch.h"

struct psb_exchange {
    int device = -1;
    int parts = 0, rank = 0;
    int64_t q = 0;
    int k = 0;
    int32_t *ids[2] = {nullptr, nullptr};     // own [q][k] result lists, by epoch parity
    float *dists[2] = {nullptr, nullptr};
    uint32_t *flags = nullptr;                // own [parts] flag slots (peer r writes slot r)
    int32_t *status = nullptr;                // device word: 1 = a wait timed out
    // peers' buffers as mapped into this process (own entries for self)
    int32_t *peer_ids[PSB_MAX_PARTS][2] = {};
    float *peer_dists[PSB_MAX_PARTS][2] = {};
    uint32_t *peer_flags[PSB_MAX_PARTS] = {};
    bool opened[PSB_MAX_PARTS] = {};          // mapped with cudaIpcOpenMemHandle (closed on free)
};

namespace psb {

struct ExBlob {                    // what a rank publishes (psb_exchange_handle)
    uint64_t magic;
    int64_t pid;
    int32_t device, rank, parts, k;
    int64_t q;
    uint64_t raw[5];               // ids0, ids1, d0, d1, flags (valid in the owning process)
    cudaIpcMemHandle_t h[5];
};
constexpr uint64_t EX_MAGIC = 0x5053424558434831ull;   // "PSBEXCH1"

struct PeerLists {
    const int32_t *ids[PSB_MAX_PARTS];
    const float *dists[PSB_MAX_PARTS];
};

__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(uint32_t *p, uint32_t v)
{
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

struct FlagPtrs {
    uint32_t *p[PSB_MAX_PARTS];
};

// Stream-ordered after this rank's local search: publish the epoch to every peer.
__global__ void signal_kernel(FlagPtrs fl, int parts, int self, uint32_t epoch)
{
    __threadfence_system();
    for (int p = threadIdx.x; p < parts; p += blockDim.x) st_release_sys(fl.p[p] + self, epoch);
}

// Gather + merge: one warp per owned row. Every CTA first waits (thread 0, with
// a 10 s bound so a missing peer cannot hang the GPU) for all parts' flags.
template <int KS>
__global__ void __launch_bounds__(128)
merge_peers_kernel(PeerLists src, int parts, int64_t row0, int64_t rows, int k, const uint32_t *__restrict__ flags,
                   uint32_t epoch, int32_t *__restrict__ status, int32_t *__restrict__ out_ids,
                   float *__restrict__ out_dists)
{
    __shared__ u64 scratch_all[4][32];
    __shared__ int ok;
    if (threadIdx.x == 0) {
        uint64_t t0;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        int good = 1;
        for (int p = 0; p < parts && good; ++p) {
            while (ld_acquire_sys(flags + p) < epoch) {
                uint64_t t;
                asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
                if (t - t0 > 10000000000ull) { good = 0; break; }
                __nanosleep(256);
            }
        }
        if (!good) atomicExch(status, 1);
        ok = good;
    }
    __syncthreads();
    if (!ok) return;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t r = (int64_t)blockIdx.x * 4 + w;
    if (r >= rows) return;
    const int64_t row = row0 + r;
    TopK<KS> T;
    T.init();
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
    T.store(k, lane, out_ids + r * k, out_dists + r * k);
}

}  // namespace psb

using namespace psb;

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
    if (prev >= 0) cudaSetDevice(prev);
    delete x;
}

extern "C" {

int psb_exchange_create(int32_t parts, int32_t rank, int64_t q, int32_t k, psb_exchange **out)
{
    if (!out) { psb_set_error("psb_exchange_create: out is NULL"); return PSB_EINVAL; }
    *out = nullptr;
    if (parts < 1 || parts > PSB_MAX_PARTS || rank < 0 || rank >= parts || q < 1 || k < 1 || k > 128) {
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
    if (e == cudaSuccess) e = cudaMalloc((void **)&x->flags, 4 * (size_t)parts);
    if (e == cudaSuccess) e = cudaMalloc((void **)&x->status, 4);
    if (e == cudaSuccess) e = cudaMemset(x->flags, 0, 4 * (size_t)parts);
    if (e == cudaSuccess) e = cudaMemset(x->status, 0, 4);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
        int rc = report_cuda(e, "psb_exchange_create");
        ex_release(x);
        return rc;
    }
    *out = x;
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
    bl.pid = (int64_t)getpid();
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
    const int64_t me = (int64_t)getpid();
    for (int p = 0; p < x->parts; ++p) {
        ExBlob bl;
        memcpy(&bl, blobs[p], sizeof bl);
        if (bl.magic != EX_MAGIC || bl.rank != p || bl.parts != x->parts || bl.k != x->k || bl.q != x->q) {
            psb_set_error("psb_exchange_connect: blob %d does not match (rank/parts/q/k)", p);
            return PSB_EINVAL;
        }
        void *ptrs[5];
        if (bl.pid == me) {                          // same process: the raw pointers are valid
            for (int i = 0; i < 5; ++i) ptrs[i] = (void *)(uintptr_t)bl.raw[i];
        } else {
            for (int i = 0; i < 5; ++i) {
                cudaError_t e = cudaIpcOpenMemHandle(&ptrs[i], bl.h[i], cudaIpcMemLazyEnablePeerAccess);
                if (e != cudaSuccess) return report_cuda(e, "psb_exchange_connect: cudaIpcOpenMemHandle");
            }
            x->opened[p] = true;
        }
        x->peer_ids[p][0] = (int32_t *)ptrs[0];
        x->peer_ids[p][1] = (int32_t *)ptrs[1];
        x->peer_dists[p][0] = (float *)ptrs[2];
        x->peer_dists[p][1] = (float *)ptrs[3];
        x->peer_flags[p] = (uint32_t *)ptrs[4];
    }
    return PSB_OK;
}

int psb_exchange_buffers(const psb_exchange *x, int64_t epoch, int32_t **ids, float **dists)
{
    if (!x || !ids || !dists || epoch < 1) { psb_set_error("psb_exchange_buffers: bad argument"); return PSB_EINVAL; }
    *ids = x->ids[epoch & 1];
    *dists = x->dists[epoch & 1];
    return PSB_OK;
}

int psb_exchange_step(psb_exchange *x, int64_t epoch, int64_t row0, int64_t rows, int32_t *out_ids,
                      float *out_dists, void *stream)
{
    if (!x || epoch < 1 || epoch > 0xffffffffll || row0 < 0 || rows < 0 || row0 + rows > x->q ||
        (rows > 0 && (!out_ids || !out_dists))) {
        psb_set_error("psb_exchange_step: bad argument");
        return PSB_EINVAL;
    }
    for (int p = 0; p < x->parts; ++p)
        if (!x->peer_flags[p]) { psb_set_error("psb_exchange_step: not connected"); return PSB_EINVAL; }
    cudaStream_t st = (cudaStream_t)stream;
    FlagPtrs fl;
    PeerLists src;
    memset(&fl, 0, sizeof fl);
    memset(&src, 0, sizeof src);
    for (int p = 0; p < x->parts; ++p) {
        fl.p[p] = x->peer_flags[p];
        src.ids[p] = x->peer_ids[p][epoch & 1];
        src.dists[p] = x->peer_dists[p][epoch & 1];
    }
    signal_kernel<<<1, 32, 0, st>>>(fl, x->parts, x->rank, (uint32_t)epoch);
    int rc = report_cuda(cudaGetLastError(), "psb_exchange_step: signal");
    if (rc != PSB_OK || rows == 0) return rc;
    const unsigned blocks = (unsigned)((rows + 3) / 4);
    const uint32_t ep = (uint32_t)epoch;
    if (x->k <= 32)
        merge_peers_kernel<1><<<blocks, 128, 0, st>>>(src, x->parts, row0, rows, x->k, x->flags, ep, x->status, out_ids, out_dists);
    else if (x->k <= 64)
        merge_peers_kernel<2><<<blocks, 128, 0, st>>>(src, x->parts, row0, rows, x->k, x->flags, ep, x->status, out_ids, out_dists);
    else
        merge_peers_kernel<4><<<blocks, 128, 0, st>>>(src, x->parts, row0, rows, x->k, x->flags, ep, x->status, out_ids, out_dists);
    return report_cuda(cudaGetLastError(), "psb_exchange_step: merge");
}

int psb_exchange_status(const psb_exchange *x, int32_t *timed_out)
{
    if (!x || !timed_out) { psb_set_error("psb_exchange_status: NULL argument"); return PSB_EINVAL; }
    cudaError_t e = cudaMemcpy(timed_out, x->status, 4, cudaMemcpyDeviceToHost);
    return report_cuda(e, "psb_exchange_status");
}

void psb_exchange_free(psb_exchange *x) { ex_release(x); }

}  // extern "C"
