"""Multi-GPU modes over torch.distributed (one process per GPU; NCCL over NVLink).

North_star (BASELINE.json): "In query-sharded mode the index is replicated and
the query batch is split, with no collective. In data-sharded mode each GPU
holds a sub-tree over a slab of the points, and per-shard top-k lists are
combined with an NCCL all-gather over NVLink plus an on-device k-way merge."
(SURVEY.md §8(e).) The paper itself is single-GPU (§V-A).

Everything here is plumbing: the local search and the merge are the library's
CUDA kernels (``psb_knn`` / ``psb_merge_topk``); the collective is NCCL via
``torch.distributed``. ``data_sharded_knn_p2p`` is the collective-free route:
the library's exchange kernel pulls each rank's rows from its peers' result
buffers over NVLink (CUDA IPC), torch.distributed only swaps the handles once. The orchestration functions take the local-search and
merge steps as callables so their host logic can be tested on CPU with gloo.
"""
from __future__ import annotations

from typing import Callable, Sequence

import torch
import torch.distributed as dist


def shard_bounds(n: int, world: int) -> list[int]:
    """Slab r of a data-sharded index holds global rows [b[r], b[r+1])."""
    return [n * r // world for r in range(world + 1)]


def query_slice(q: int, world: int, rank: int) -> slice:
    """Contiguous slice of a query batch owned by `rank` (query-sharded mode)."""
    b = shard_bounds(q, world)
    return slice(b[rank], b[rank + 1])


def allgather_topk(ids: torch.Tensor, dists: torch.Tensor, group=None):
    """[q, k] local lists on every rank -> [world, q, k] on every rank."""
    world = dist.get_world_size(group)
    gi = torch.empty((world, *ids.shape), dtype=ids.dtype, device=ids.device)
    gd = torch.empty((world, *dists.shape), dtype=dists.dtype, device=dists.device)
    if ids.is_cuda:
        dist.all_gather_into_tensor(gi, ids.contiguous(), group=group)
        dist.all_gather_into_tensor(gd, dists.contiguous(), group=group)
    else:                              # gloo (CPU tests): list form
        dist.all_gather(list(gi.unbind(0)), ids.contiguous(), group=group)
        dist.all_gather(list(gd.unbind(0)), dists.contiguous(), group=group)
    return gi, gd


def data_sharded_knn(local_knn: Callable, merge: Callable, queries: torch.Tensor, k: int,
                     group=None, merge_all: bool = False):
    """One data-sharded step (the NCCL route): local kNN over this rank's slab(s)
    (ids already global via id_base), all-gather of the lists, exact merge.

    `local_knn(queries, k)` returns this rank's lists as [q, k] (one slab) or
    [s, q, k] (s slabs held by this rank); the all-gather stacks every rank's
    lists into [world*s, q, k] and `merge` (psb_merge_topk) combines them.
    Returns (ids, dists) for this rank's query slice (or for all queries when
    merge_all). Exact because (dist, id) is a total order and every global id
    lives in exactly one slab."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    ids, dists = local_knn(queries, k)
    if ids.dim() == 2:
        if world == 1:
            return ids, dists
        ids, dists = ids.unsqueeze(0), dists.unsqueeze(0)
    s, q = ids.shape[0], ids.shape[1]
    gi, gd = allgather_topk(ids, dists, group)                 # [world, s, q, k]
    gi, gd = gi.reshape(world * s, q, k), gd.reshape(world * s, q, k)
    if merge_all:
        return merge(gi, gd, k)
    sl = query_slice(q, world, rank)
    return merge(gi[:, sl].contiguous(), gd[:, sl].contiguous(), k)


def query_sharded_knn(local_knn: Callable, queries: torch.Tensor, k: int, group=None,
                      gather: bool = False):
    """Query-sharded step: this rank answers its slice of `queries` on its
    replica; no collective unless `gather` (results collected on every rank)."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    sl = query_slice(queries.shape[0], world, rank)
    ids, dists = local_knn(queries[sl].contiguous(), k)
    if not gather or world == 1:
        return ids, dists
    b = shard_bounds(queries.shape[0], world)
    sizes = [b[r + 1] - b[r] for r in range(world)]
    mx = max(sizes)
    pad_i = torch.full((mx, k), -1, dtype=ids.dtype, device=ids.device)
    pad_d = torch.full((mx, k), float("inf"), dtype=dists.dtype, device=dists.device)
    pad_i[: ids.shape[0]] = ids
    pad_d[: dists.shape[0]] = dists
    gi, gd = allgather_topk(pad_i, pad_d, group)
    return (torch.cat([gi[r, : sizes[r]] for r in range(world)]),
            torch.cat([gd[r, : sizes[r]] for r in range(world)]))


def peer_exchange(q: int, k: int, group=None):
    """Set up this rank's psb_exchange (include/psb.h): create it, share its IPC
    handle blob with every rank (all_gather_object: host bytes, once), map the
    peers' buffers. Collective over `group`."""
    from . import Exchange
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    ex = Exchange(world, rank, q, k)
    blobs = [None] * world
    dist.all_gather_object(blobs, ex.handle(), group=group)
    ex.connect(blobs)
    return ex


def chunk_rows(q: int, parts: int, rank: int, chunks: int) -> list[slice]:
    """Rows a rank merges in chunked data-sharded mode: its 1/parts slice of each
    of `chunks` contiguous chunks of the batch, in chunk order (chunks = 1: the
    plain query_slice)."""
    cb = shard_bounds(q, max(1, chunks))
    out = []
    for c in range(max(1, chunks)):
        sl = query_slice(cb[c + 1] - cb[c], parts, rank)
        out.append(slice(cb[c] + sl.start, cb[c] + sl.stop))
    return out


_side_streams: dict = {}


def _side_stream():
    dev = torch.cuda.current_device()
    if dev not in _side_streams:
        _side_streams[dev] = torch.cuda.Stream()
    return _side_streams[dev]


def data_sharded_knn_p2p(ex, index, queries: torch.Tensor, algo: int = 0, variant: int = 0, stream=None,
                         chunks: int = 1, side=None, out=None):
    """One data-sharded step without a collective: local search into this rank's
    exchange buffers, then kernels that wait for every peer's flag and merge this
    rank's rows straight out of all ranks' buffers over NVLink.

    chunks = 1: search all q queries, then merge query_slice(q, world, rank).
    chunks > 1: the batch is cut into `chunks` pieces; chunk c is searched and
    signalled on `stream` while the merge of chunk c-1 runs on a second stream
    (`side`), so the exchange overlaps the search; this rank merges its slice of
    every chunk (chunk_rows). Returns (ids, dists) of those rows, in order."""
    main = stream if stream is not None else torch.cuda.current_stream()
    rows = chunk_rows(ex.q, ex.parts, ex.rank, chunks)
    total = sum(r.stop - r.start for r in rows)
    if out is None:
        out = (torch.empty((total, ex.k), dtype=torch.int32, device=queries.device),
               torch.empty((total, ex.k), dtype=torch.float32, device=queries.device))
    if chunks <= 1:
        ex.local_knn(index, queries, algo=algo, variant=variant, stream=main)
        return ex.step(rows[0].start, total, stream=main, out=out)
    side = side if side is not None else _side_stream()
    ex.begin()
    side.wait_stream(main)                     # out buffers / previous epoch in stream order
    cb = shard_bounds(ex.q, chunks)
    o = 0
    for c in range(chunks):
        ex.local_knn(index, queries, algo=algo, variant=variant, stream=main, rows=slice(cb[c], cb[c + 1]))
        ex.signal(cb[c + 1], stream=main)
        n = rows[c].stop - rows[c].start
        ex.merge(rows[c].start, n, stream=side, out=(out[0][o:o + n], out[1][o:o + n]))
        o += n
    main.wait_stream(side)                     # results (and the next epoch) after every merge
    return out


def build_shard(points, fanout: int, world: int, rank: int, packing: int = 0):
    """Build this rank's sub-tree over slab `rank` of `points` with global ids."""
    from . import psb_build_ex
    b = shard_bounds(points.shape[0], world)
    return psb_build_ex(points[b[rank]:b[rank + 1]], fanout, id_base=b[rank], packing=packing)


def device_merge(ids: torch.Tensor, dists: torch.Tensor, k: int):
    """The on-device k-way merge (psb_merge_topk kernel)."""
    from . import psb_merge_topk
    return psb_merge_topk(ids, dists, k)


def ranks_in(group=None) -> Sequence[int]:
    return list(range(dist.get_world_size(group)))
