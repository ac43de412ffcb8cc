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
    """One data-sharded step: local kNN over this rank's slab (ids already
    global via id_base), all-gather of the [q, k] lists, exact merge.

    Returns (ids, dists) for this rank's query slice (or for all queries when
    merge_all). Exact because (dist, id) is a total order and every global id
    lives in exactly one slab."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    ids, dists = local_knn(queries, k)
    if world == 1:
        return ids, dists
    gi, gd = allgather_topk(ids, dists, group)
    if merge_all:
        return merge(gi, gd, k)
    sl = query_slice(queries.shape[0], world, rank)
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


def data_sharded_knn_p2p(ex, index, queries: torch.Tensor, algo: int = 0, variant: int = 0, stream=None):
    """One data-sharded step without a collective: local search into this rank's
    exchange buffers, then one kernel that waits for every peer's flag and merges
    this rank's query slice straight out of all ranks' buffers over NVLink.
    Returns (ids, dists) for the slice query_slice(q, world, rank)."""
    ex.local_knn(index, queries, algo=algo, variant=variant, stream=stream)
    sl = query_slice(ex.q, ex.parts, ex.rank)
    return ex.step(sl.start, sl.stop - sl.start, stream=stream)


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
