"""psb-b200 — exact kNN by Parallel Scan and Backtrack on NVIDIA B200 (sm_100a).

Thin Python binding over ``libpsb.so`` (C ABI in ``include/psb.h``). Every step
of the query path runs in the library's CUDA kernels; this module only marshals
arguments: torch tensors provide device memory and streams. There is no CPU
fallback: importing the package fails if ``libpsb.so`` has not been built
(``python -c "import __graft_entry__ as g; g.build()"``).

Names mirror the C ABI: ``psb_build``, ``psb_build_ex``, ``psb_knn``,
``psb_knn_branch_and_bound``, ``psb_knn_bruteforce``, ``psb_knn_ex``,
``psb_merge_topk``, ``psb_index_info``, ``psb_index_export``,
``psb_build_host_blob``, ``psb_free``, ``psb_last_error``, ``psb_version``.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("PSB_LIB_PATH") or os.path.join(_HERE, "libpsb.so")   # override: A/B builds

PSB_OK, PSB_EINVAL, PSB_ENOMEM, PSB_ECUDA, PSB_EUNSUPPORTED = 0, -1, -2, -3, -4
PSB_PACK_HILBERT, PSB_PACK_STR, PSB_PACK_KMEANS = 0, 1, 2
PSB_BUILD_HOST = 0x100
PSB_NODE_SPHERE = 0x200
PSB_ALGO_PSB, PSB_ALGO_BNB, PSB_ALGO_BRUTE = 0, 1, 2
PSB_VAR_NOCACHE, PSB_VAR_NOMAXDIST, PSB_VAR_INPUT_ORDER, PSB_VAR_LEAF_ORDER = 1, 2, 4, 8
PSB_VAR_PREFETCH_NEXT, PSB_VAR_PREFETCH_IDS, PSB_VAR_P1_INDEX_TIE = 16, 32, 64
PSB_VAR_KTH_MAXDIST = 128
PSB_VAR_NO_AUTO_PREFETCH = 256
PSB_VAR_GENERIC_D = 512
PSB_TRACE_PASS1, PSB_TRACE_CHANGED, PSB_TRACE_SKIPPED, PSB_TRACE_FETCHED = 1, 2, 4, 8
PSB_KMAX, PSB_DMAX, PSB_MAX_PARTS = 2048, 64, 16
FANOUTS = (32, 64, 128, 256, 512)

# every symbol include/psb.h declares (tests check the .so exports all of them)
EXPORTS = ("psb_build", "psb_build_ex", "psb_knn", "psb_knn_branch_and_bound", "psb_knn_bruteforce",
           "psb_knn_ex", "psb_knn_stats", "psb_knn_trace", "psb_knn_split", "psb_merge_topk", "psb_index_info", "psb_index_export", "psb_index_import", "psb_build_host_blob",
           "psb_free", "psb_last_error", "psb_version", "psb_exchange_create", "psb_exchange_handle",
           "psb_exchange_connect", "psb_exchange_buffers", "psb_exchange_signal", "psb_exchange_merge",
           "psb_exchange_step", "psb_exchange_status", "psb_exchange_set_timeout", "psb_exchange_free",
           "psb_probe_l2_read")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libpsb.so not built at {LIB_PATH}: run __graft_entry__.build() "
                      "(there is no CPU fallback)")

_lib = ctypes.CDLL(LIB_PATH)
_vp, _i64, _i32, _u32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint32
_P = ctypes.POINTER
_sig = {
    "psb_build": (_vp, [_vp, _i64, _i32, _i32]),
    "psb_build_ex": (ctypes.c_int, [_vp, _i64, _i32, _i32, _i64, _u32, _P(_vp)]),
    "psb_knn": (ctypes.c_int, [_vp, _vp, _i64, _i32, _vp, _vp, _vp]),
    "psb_knn_branch_and_bound": (ctypes.c_int, [_vp, _vp, _i64, _i32, _vp, _vp, _vp]),
    "psb_knn_bruteforce": (ctypes.c_int, [_vp, _vp, _i64, _i32, _vp, _vp, _vp]),
    "psb_knn_ex": (ctypes.c_int, [_vp, _vp, _i64, _i32, _vp, _vp, _vp, _i32, _u32]),
    "psb_knn_split": (ctypes.c_int, [_vp, _vp, _i64, _i32, _i32, _vp, _vp, _vp]),
    "psb_knn_stats": (ctypes.c_int, [_vp, _vp, _i64, _i32, _vp, _vp, _vp, _i32, _u32, _vp]),
    "psb_knn_trace": (ctypes.c_int, [_vp, _vp, _i64, _i32, _vp, _vp, _vp, _i32, _u32, _vp, _vp, _i32, _vp]),
    "psb_merge_topk": (ctypes.c_int, [_vp, _vp, _i32, _i64, _i32, _vp, _vp, _vp]),
    "psb_index_info": (ctypes.c_int, [_vp, _P(_i64), _P(_i32), _P(_i32), _P(_i64), _P(_i32), _P(_i64)]),
    "psb_index_export": (ctypes.c_int, [_vp, _vp, _i64, _P(_i64)]),
    "psb_index_import": (ctypes.c_int, [_vp, _i64, _P(_vp)]),
    "psb_build_host_blob": (ctypes.c_int, [_vp, _i64, _i32, _i32, _i64, _u32, _vp, _i64, _P(_i64)]),
    "psb_free": (None, [_vp]),
    "psb_exchange_create": (ctypes.c_int, [_i32, _i32, _i64, _i32, _P(_vp)]),
    "psb_exchange_handle": (ctypes.c_int, [_vp, _vp, _i64, _P(_i64)]),
    "psb_exchange_connect": (ctypes.c_int, [_vp, _P(_vp)]),
    "psb_exchange_buffers": (ctypes.c_int, [_vp, _i64, _P(_vp), _P(_vp)]),
    "psb_exchange_signal": (ctypes.c_int, [_vp, _i64, _i64, _vp]),
    "psb_exchange_merge": (ctypes.c_int, [_vp, _i64, _i64, _i64, _vp, _vp, _vp]),
    "psb_exchange_step": (ctypes.c_int, [_vp, _i64, _i64, _i64, _vp, _vp, _vp]),
    "psb_exchange_set_timeout": (ctypes.c_int, [_vp, _i64]),
    "psb_exchange_status": (ctypes.c_int, [_vp, _P(_i32)]),
    "psb_exchange_free": (None, [_vp]),
    "psb_probe_l2_read": (ctypes.c_int, [_i64, _i32, _i32, _P(ctypes.c_double)]),
    "psb_last_error": (ctypes.c_char_p, []),
    "psb_version": (ctypes.c_char_p, []),
}
for _name, (_res, _args) in _sig.items():
    _f = getattr(_lib, _name)
    _f.restype, _f.argtypes = _res, _args


class PSBError(RuntimeError):
    def __init__(self, code: int, where: str):
        self.code = code
        super().__init__(f"{where} failed ({code}): {psb_last_error()}")


def _check(rc: int, where: str):
    if rc != PSB_OK:
        raise PSBError(rc, where)


def psb_last_error() -> str:
    return _lib.psb_last_error().decode()


def psb_version() -> str:
    return _lib.psb_version().decode()


_TORCH = None


def _torch():
    global _TORCH
    if _TORCH is None:
        import torch
        _TORCH = torch
    return _TORCH


def _stream_handle(stream, device: int | None = None) -> int:
    """cudaStream_t of `stream` (None: torch's current stream on `device`). The raw
    getter avoids building a Stream object: a one-query call is host-latency bound."""
    if stream is None:
        torch = _torch()
        raw = getattr(torch._C, "_cuda_getCurrentRawStream", None)
        if raw is not None:
            return int(raw(torch.cuda.current_device() if device is None else device))
        stream = torch.cuda.current_stream()
    return int(stream.cuda_stream) if hasattr(stream, "cuda_stream") else int(stream)


class Index:
    """Owns a psb_index* (device memory on the device current at build time)."""

    def __init__(self, handle: int):
        self._h = ctypes.c_void_p(handle)
        n, d, f, L, H, b = _i64(), _i32(), _i32(), _i64(), _i32(), _i64()
        _check(_lib.psb_index_info(self._h, ctypes.byref(n), ctypes.byref(d), ctypes.byref(f),
                                   ctypes.byref(L), ctypes.byref(H), ctypes.byref(b)), "psb_index_info")
        self.n, self.d, self.fanout = n.value, d.value, f.value
        self.leaves, self.levels, self.device_bytes = L.value, H.value, b.value
        self.device = _torch().cuda.current_device()

    @property
    def handle(self):
        return self._h

    def free(self):
        if self._h is not None and self._h.value:
            _lib.psb_free(self._h)
        self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass

    def info(self) -> dict:
        return {"n": self.n, "d": self.d, "fanout": self.fanout, "leaves": self.leaves,
                "levels": self.levels, "device_bytes": self.device_bytes}


def _as_points(points):
    """Host numpy / CPU tensor / CUDA tensor -> (pointer, keepalive, n, d)."""
    torch = _torch()
    if isinstance(points, np.ndarray):
        a = np.ascontiguousarray(points, dtype=np.float32)
        return a.ctypes.data, a, a.shape[0], a.shape[1]
    t = points.contiguous()
    if t.dtype != torch.float32:
        raise TypeError("points must be float32")
    return t.data_ptr(), t, t.shape[0], t.shape[1]


def psb_build_ex(points, fanout: int, id_base: int = 0, packing: int = PSB_PACK_HILBERT) -> Index:
    """Bulk-load the R-tree (include/psb.h psb_build_ex) on the current CUDA device."""
    ptr, keep, n, d = _as_points(points)
    out = ctypes.c_void_p()
    _check(_lib.psb_build_ex(ptr, n, d, fanout, id_base, packing, ctypes.byref(out)), "psb_build_ex")
    del keep
    return Index(out.value)


def psb_build(points, fanout: int) -> Index:
    ptr, keep, n, d = _as_points(points)
    h = _lib.psb_build(ptr, n, d, fanout)
    if not h:
        raise PSBError(PSB_EINVAL, "psb_build")
    return Index(h)


def _check_out(out, q: int, k: int, device: int):
    """out = (ids, dists): int32 / float32 [q, k] C-contiguous tensors, on CUDA
    device `device` or in host memory."""
    torch = _torch()
    ids, dists = out
    for t, dt, name in ((ids, torch.int32, "ids"), (dists, torch.float32, "dists")):
        if t.dtype is not dt or t.shape != (q, k) or not t.is_contiguous():
            raise ValueError(f"out {name} must be a contiguous {dt} [{q}, {k}] tensor")
        if t.is_cuda and t.get_device() != device:
            raise ValueError(f"out {name} is on {t.device}, the index on cuda:{device}")


def _query_buffers(index: Index, queries, k: int, out):
    """Queries: float32 [q, d] tensor on the index's device, or a CPU tensor
    (pinned: read in place by the kernels; pageable: staged by the library).
    Outputs default to the queries' device (CPU outputs are pinned)."""
    torch = _torch()
    if queries.dtype is not torch.float32 or queries.dim() != 2 or queries.shape[1] != index.d:
        raise ValueError(f"queries must be a float32 [q, {index.d}] tensor")
    if not queries.is_contiguous():
        queries = queries.contiguous()
    q = queries.shape[0]
    if queries.is_cuda and queries.get_device() != index.device:
        raise ValueError(f"queries are on {queries.device}, the index on cuda:{index.device}")
    if out is None:
        pin = not queries.is_cuda
        ids = torch.empty((q, k), dtype=torch.int32, device=queries.device, pin_memory=pin)
        dists = torch.empty((q, k), dtype=torch.float32, device=queries.device, pin_memory=pin)
    else:
        _check_out(out, q, k, index.device)
        ids, dists = out
    return queries, q, ids, dists


def _host_sync(stream, *tensors):
    """The C ABI is asynchronous and keeps no reference to its buffers. Host
    tensors (queries read in place or by a stream-ordered copy, outputs written by
    the kernels) would otherwise be returned while the device still uses them, and
    a temporary pinned input could be recycled by torch's caching host allocator:
    with any host tensor, the call waits for its stream before returning."""
    for t in tensors:
        if not t.is_cuda:
            break
    else:
        return
    torch = _torch()
    s = stream if stream is not None else torch.cuda.current_stream()
    if hasattr(s, "synchronize"):
        s.synchronize()
    else:
        torch.cuda.ExternalStream(int(s)).synchronize()


def psb_knn_ex(index: Index, queries, k: int, algo: int = PSB_ALGO_PSB, variant: int = 0,
               stream=None, out=None):
    """Asynchronous on `stream` (default: torch's current stream) for device
    tensors; waits for the stream when a tensor is in host memory. Returns (ids, dists)."""
    queries, q, ids, dists = _query_buffers(index, queries, k, out)
    _check(_lib.psb_knn_ex(index.handle, queries.data_ptr(), q, k, ids.data_ptr(), dists.data_ptr(),
                           _stream_handle(stream, index.device), algo, variant), "psb_knn_ex")
    _host_sync(stream, queries, ids, dists)
    return ids, dists


def psb_knn_stats(index: Index, queries, k: int, algo: int = PSB_ALGO_PSB, variant: int = 0,
                  stream=None, out=None):
    """psb_knn_ex plus per-query counters: returns (ids, dists, stats int64 [q, 8] on device)
    with stats = {node fetches, leaf scans, id loads, path-cache hits, changing leaf scans,
    keys merged, t_start ns, t_end ns} (include/psb.h; the last two are the device
    %globaltimer when the warp took / finished the query)."""
    torch = _torch()
    queries, q, ids, dists = _query_buffers(index, queries, k, out)
    stats = torch.zeros((q, 8), dtype=torch.int64, device=f"cuda:{index.device}")
    _check(_lib.psb_knn_stats(index.handle, queries.data_ptr(), q, k, ids.data_ptr(), dists.data_ptr(),
                              _stream_handle(stream), algo, variant, stats.data_ptr()), "psb_knn_stats")
    _host_sync(stream, queries, ids, dists)
    return ids, dists, stats


def psb_knn_trace(index: Index, queries, k: int, cap: int = 4096, algo: int = PSB_ALGO_PSB, variant: int = 0,
                  stream=None, out=None):
    """psb_knn_stats plus each query's traversal steps (include/psb.h psb_knn_trace).
    Returns (ids, dists, stats [q, 8], trace int64 [q, cap], trace_len int32 [q]), all
    on the device; decode with trace_steps()."""
    torch = _torch()
    queries, q, ids, dists = _query_buffers(index, queries, k, out)
    dev = f"cuda:{index.device}"
    stats = torch.zeros((q, 8), dtype=torch.int64, device=dev)
    trace = torch.full((q, cap), -1, dtype=torch.int64, device=dev)
    tlen = torch.zeros((q,), dtype=torch.int32, device=dev)
    _check(_lib.psb_knn_trace(index.handle, queries.data_ptr(), q, k, ids.data_ptr(), dists.data_ptr(),
                              _stream_handle(stream), algo, variant, stats.data_ptr(), trace.data_ptr(), cap,
                              tlen.data_ptr()), "psb_knn_trace")
    _host_sync(stream, queries, ids, dists)
    return ids, dists, stats, trace, tlen


def trace_steps(row, n: int) -> list[tuple[int, int, int]]:
    """Decode one query's trace row (first n steps) into (level, node, flags)."""
    out = []
    for v in [int(x) for x in row[:n]]:
        out.append(((v >> 32) & 0xFF, v & 0xFFFFFFFF, (v >> 40) & 0xFF))
    return out


def algorithmic_bytes(index: Index, stats, q: int, k: int) -> int:
    """Bytes a launch must move: node blocks fetched, leaf blocks
    scanned, ids loaded, queries read, results written."""
    s = stats.sum(0).tolist() if hasattr(stats, "sum") else stats
    F, d = index.fanout, index.d
    return int(s[0] * F * 2 * d * 4 + s[1] * F * d * 4 + s[2] * 4 + q * (4 * d + 8 * k))


def psb_knn(index: Index, queries, k: int, stream=None, out=None):
    queries, q, ids, dists = _query_buffers(index, queries, k, out)
    _check(_lib.psb_knn(index.handle, queries.data_ptr(), q, k, ids.data_ptr(), dists.data_ptr(),
                        _stream_handle(stream)), "psb_knn")
    _host_sync(stream, queries, ids, dists)
    return ids, dists


def psb_knn_split(index: Index, queries, k: int, parts: int = 0, stream=None, out=None):
    """Latency mode: each query split over `parts` warps (0 = auto)."""
    queries, q, ids, dists = _query_buffers(index, queries, k, out)
    _check(_lib.psb_knn_split(index.handle, queries.data_ptr(), q, k, parts, ids.data_ptr(), dists.data_ptr(),
                              _stream_handle(stream)), "psb_knn_split")
    _host_sync(stream, queries, ids, dists)
    return ids, dists


def psb_knn_branch_and_bound(index: Index, queries, k: int, stream=None, out=None):
    queries, q, ids, dists = _query_buffers(index, queries, k, out)
    _check(_lib.psb_knn_branch_and_bound(index.handle, queries.data_ptr(), q, k, ids.data_ptr(),
                                         dists.data_ptr(), _stream_handle(stream)),
           "psb_knn_branch_and_bound")
    _host_sync(stream, queries, ids, dists)
    return ids, dists


def psb_knn_bruteforce(index: Index, queries, k: int, stream=None, out=None):
    queries, q, ids, dists = _query_buffers(index, queries, k, out)
    _check(_lib.psb_knn_bruteforce(index.handle, queries.data_ptr(), q, k, ids.data_ptr(),
                                   dists.data_ptr(), _stream_handle(stream)), "psb_knn_bruteforce")
    _host_sync(stream, queries, ids, dists)
    return ids, dists


def psb_merge_topk(ids, dists, k: int, stream=None, out=None):
    """ids/dists: CUDA [parts, q, k] -> (out_ids, out_dists) [q, k]."""
    torch = _torch()
    parts, q, kk = ids.shape
    assert kk == k and dists.shape == ids.shape
    ids, dists = ids.contiguous(), dists.contiguous()
    if out is None:
        out = (torch.empty((q, k), dtype=torch.int32, device=ids.device),
               torch.empty((q, k), dtype=torch.float32, device=ids.device))
    _check(_lib.psb_merge_topk(ids.data_ptr(), dists.data_ptr(), parts, q, k, out[0].data_ptr(),
                               out[1].data_ptr(), _stream_handle(stream)), "psb_merge_topk")
    return out


class Exchange:
    """Data-sharded exchange over peer memory (include/psb.h psb_exchange_*): this
    rank's double-buffered [q, k] result lists and flag slots, mapped by every
    rank; `step` merges the rows this rank owns straight out of all ranks' lists."""

    def __init__(self, parts: int, rank: int, q: int, k: int):
        h = ctypes.c_void_p()
        _check(_lib.psb_exchange_create(parts, rank, q, k, ctypes.byref(h)), "psb_exchange_create")
        self._h, self.parts, self.rank, self.q, self.k = h, parts, rank, q, k
        self.epoch = 0

    def handle(self) -> bytes:
        used = _i64()
        _check(_lib.psb_exchange_handle(self._h, None, 0, ctypes.byref(used)), "psb_exchange_handle")
        buf = ctypes.create_string_buffer(used.value)
        _check(_lib.psb_exchange_handle(self._h, buf, used.value, ctypes.byref(used)), "psb_exchange_handle")
        return buf.raw

    def connect(self, blobs):
        """blobs: every rank's handle() in rank order."""
        keep = [ctypes.create_string_buffer(b, len(b)) for b in blobs]
        arr = (_vp * len(keep))(*[ctypes.cast(b, _vp) for b in keep])
        _check(_lib.psb_exchange_connect(self._h, arr), "psb_exchange_connect")

    def begin(self):
        """Next epoch; returns (ids_ptr, dists_ptr) of this rank's [q, k] result buffers for it."""
        self.epoch += 1
        pi, pd = _vp(), _vp()
        _check(_lib.psb_exchange_buffers(self._h, self.epoch, ctypes.byref(pi), ctypes.byref(pd)),
               "psb_exchange_buffers")
        return pi.value, pd.value

    def local_knn(self, index: "Index", queries, algo: int = PSB_ALGO_PSB, variant: int = 0, stream=None,
                  rows: slice | None = None):
        """Local search into this rank's buffers. Without `rows`: begin() (next
        epoch) + all q queries. With `rows` (a slice of the current epoch's rows,
        chunked mode): only those queries, written to the same rows."""
        assert queries.is_cuda and queries.shape[0] == self.q
        if rows is None:
            pi, pd = self.begin()
            r0, r1 = 0, self.q
        else:
            pi, pd = _vp(), _vp()
            _check(_lib.psb_exchange_buffers(self._h, self.epoch, ctypes.byref(pi), ctypes.byref(pd)),
                   "psb_exchange_buffers")
            pi, pd = pi.value, pd.value
            r0, r1 = rows.start, rows.stop
        if r1 > r0:
            _check(_lib.psb_knn_ex(index.handle, queries[r0:r1].data_ptr(), r1 - r0, self.k, pi + 4 * r0 * self.k,
                                   pd + 4 * r0 * self.k, _stream_handle(stream), algo, variant),
                   "psb_knn_ex (exchange)")

    def signal(self, rows_done: int | None = None, stream=None):
        """Publish that rows [0, rows_done) of this epoch are final (default: all q)."""
        _check(_lib.psb_exchange_signal(self._h, self.epoch, self.q if rows_done is None else rows_done,
                                        _stream_handle(stream)), "psb_exchange_signal")

    def _out(self, rows, out):
        torch = _torch()
        if out is None:
            return (torch.empty((rows, self.k), dtype=torch.int32, device="cuda"),
                    torch.empty((rows, self.k), dtype=torch.float32, device="cuda"))
        _check_out(out, rows, self.k, torch.cuda.current_device())
        return out

    def merge(self, row0: int, rows: int, stream=None, out=None):
        """Wait (on the device) for every rank's signal, merge rows [row0, row0+rows)."""
        out = self._out(rows, out)
        _check(_lib.psb_exchange_merge(self._h, self.epoch, row0, rows, out[0].data_ptr(), out[1].data_ptr(),
                                       _stream_handle(stream)), "psb_exchange_merge")
        return out

    def step(self, row0: int, rows: int, stream=None, out=None):
        """signal() for all q rows, then merge(row0, rows) (one call per rank and epoch)."""
        out = self._out(rows, out)
        _check(_lib.psb_exchange_step(self._h, self.epoch, row0, rows, out[0].data_ptr(), out[1].data_ptr(),
                                      _stream_handle(stream)), "psb_exchange_step")
        return out

    def set_timeout(self, seconds: float):
        _check(_lib.psb_exchange_set_timeout(self._h, int(seconds * 1e9)), "psb_exchange_set_timeout")

    def timed_out(self) -> bool:
        v = _i32()
        _check(_lib.psb_exchange_status(self._h, ctypes.byref(v)), "psb_exchange_status")
        return bool(v.value)

    def free(self):
        if self._h is not None and self._h.value:
            _lib.psb_exchange_free(self._h)
        self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def _parse_blob(buf: np.ndarray) -> dict:
    hdr = buf[:64].view(np.int64)
    n, d, F, L, H, id_base, total, sphere = (int(x) for x in hdr[:8])
    o = 64
    nlev = buf[o:o + 8 * (H + 1)].view(np.int64).copy()
    o += 8 * (H + 1)
    pts = buf[o:o + 4 * L * d * F].view(np.float32).reshape(L, d, F)
    o += 4 * L * d * F
    ids = buf[o:o + 4 * L * F].view(np.int32).reshape(L, F)
    o += 4 * L * F
    levels = {}
    for lv in range(1, H + 1):
        cnt = int(nlev[lv])
        if sphere:
            levels[lv] = buf[o:o + 4 * cnt * (d + 1) * F].view(np.float32).reshape(cnt, d + 1, F)
            o += 4 * cnt * (d + 1) * F
        else:
            levels[lv] = buf[o:o + 4 * cnt * 2 * d * F].view(np.float32).reshape(cnt, d, 2, F)
            o += 4 * cnt * 2 * d * F
    return {"n": n, "d": d, "fanout": F, "leaves": L, "levels": H, "id_base": id_base, "sphere": bool(sphere),
            "total_nodes": total, "nlev": nlev, "pts": pts, "ids": ids, "nodes": levels}


def psb_index_export(index: Index) -> dict:
    used = _i64()
    _check(_lib.psb_index_export(index.handle, None, 0, ctypes.byref(used)), "psb_index_export")
    buf = np.empty(used.value, dtype=np.uint8)
    _check(_lib.psb_index_export(index.handle, buf.ctypes.data, used.value, ctypes.byref(used)),
           "psb_index_export")
    return _parse_blob(buf)


def psb_index_export_raw(index: Index) -> np.ndarray:
    """The export blob as raw bytes (uint8)."""
    used = _i64()
    _check(_lib.psb_index_export(index.handle, None, 0, ctypes.byref(used)), "psb_index_export")
    buf = np.empty(used.value, dtype=np.uint8)
    _check(_lib.psb_index_export(index.handle, buf.ctypes.data, used.value, ctypes.byref(used)),
           "psb_index_export")
    return buf


def psb_index_import(blob) -> Index:
    """Index on the current device from an export blob (uint8 array / bytes)."""
    a = np.ascontiguousarray(np.frombuffer(blob, dtype=np.uint8) if isinstance(blob, (bytes, bytearray)) else blob,
                             dtype=np.uint8)
    out = ctypes.c_void_p()
    _check(_lib.psb_index_import(a.ctypes.data, a.size, ctypes.byref(out)), "psb_index_import")
    return Index(out.value)


def make_blob(pts, ids, nodes: dict, n: int, id_base: int = 0) -> np.ndarray:
    """Assemble an export blob from arrays: pts [L, d, F] float32, ids [L, F] int32,
    nodes {level: [count, d, 2, F] float32} (psb_index_export layout)."""
    pts = np.ascontiguousarray(pts, np.float32)
    ids = np.ascontiguousarray(ids, np.int32)
    L, d, F = pts.shape
    H = max(nodes)
    nlev = np.array([L] + [nodes[l].shape[0] for l in range(1, H + 1)], np.int64)
    hdr = np.array([n, d, F, L, H, id_base, int(nlev[1:].sum()), 0], np.int64)
    parts = [hdr.view(np.uint8), nlev.view(np.uint8), pts.reshape(-1).view(np.uint8), ids.reshape(-1).view(np.uint8)]
    parts += [np.ascontiguousarray(nodes[l], np.float32).reshape(-1).view(np.uint8) for l in range(1, H + 1)]
    return np.concatenate(parts)


def psb_build_host_blob(points, fanout: int, id_base: int = 0, packing: int = PSB_PACK_HILBERT,
                        raw: bool = False):
    """Host-only bulk load (no CUDA): the export blob of the index psb_build_ex would build."""
    a = np.ascontiguousarray(points, dtype=np.float32)
    used = _i64()
    _check(_lib.psb_build_host_blob(a.ctypes.data, a.shape[0], a.shape[1], fanout, id_base, packing,
                                    None, 0, ctypes.byref(used)), "psb_build_host_blob")
    buf = np.empty(used.value, dtype=np.uint8)
    _check(_lib.psb_build_host_blob(a.ctypes.data, a.shape[0], a.shape[1], fanout, id_base, packing,
                                    buf.ctypes.data, used.value, ctypes.byref(used)), "psb_build_host_blob")
    return buf if raw else _parse_blob(buf)


def psb_probe_l2_read(nbytes: int = 64 << 20, passes: int = 50, reps: int = 5) -> float:
    """Measured L2 read bandwidth of the current device, GB/s (include/psb.h)."""
    g = ctypes.c_double()
    _check(_lib.psb_probe_l2_read(nbytes, passes, reps, ctypes.byref(g)), "psb_probe_l2_read")
    return g.value


def psb_free(index: Index):
    index.free()


def symbols_exported() -> dict:
    """{symbol: bool} for every declared entry point (no compute calls)."""
    out = {}
    for s in EXPORTS:
        try:
            getattr(_lib, s)
            out[s] = True
        except AttributeError:
            out[s] = False
    return out
