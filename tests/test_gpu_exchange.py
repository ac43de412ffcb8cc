"""GPU tests of the data-sharded exchange over peer memory (include/psb.h
psb_exchange_*; csrc/knn_exchange.cu): every rank's owned rows, merged by the
exchange kernel straight out of all ranks' result buffers, equal the oracle on
the unsharded point set, bit for bit.

Only one GPU is available to the tests, so "ranks" share it: (a) P ranks in one
process on separate streams (the raw-pointer path), (b) two processes on the
same GPU exchanging real CUDA IPC handles (gloo only carries the handle bytes)."""
import os
import socket

import numpy as np
import pytest

import oracle
import workloads as W

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _psb():
    import paper_conf_icpp_namkn16_b200 as psb
    return psb


def _slices(q, P):
    b = [q * r // P for r in range(P + 1)]
    return [slice(b[r], b[r + 1]) for r in range(P)]


def _setup(P, k, n=150_000, q=1003, timeout=None):
    psb = _psb()
    cfg = W.config("C2")
    pts = cfg.points(n=n)
    qs = cfg.queries(q=q)
    qd = torch.from_numpy(qs).cuda()
    bounds = [len(pts) * r // P for r in range(P + 1)]
    subs = [psb.psb_build_ex(pts[bounds[r]:bounds[r + 1]], 64, id_base=bounds[r]) for r in range(P)]
    exs = [psb.Exchange(P, r, len(qs), k) for r in range(P)]
    if timeout is not None:
        for e in exs:
            e.set_timeout(timeout)
    blobs = [e.handle() for e in exs]
    for e in exs:
        e.connect(blobs)
    return pts, qs, qd, subs, exs


def _free_all(*objs):
    for o in objs:
        for x in o:
            x.free()


@pytest.mark.parametrize("P,k", [(3, 32), (2, 7), (5, 64), (1, 16)])
def test_exchange_in_process(P, k):
    pts, qs, qd, subs, exs = _setup(P, k)
    exp = oracle.Tree(pts).knn(qs, k)
    streams = [torch.cuda.Stream() for _ in range(P)]
    sl = _slices(len(qs), P)
    for step in range(3):                                  # epochs 1..3: buffer parity alternates
        for r in range(P):                                 # every signal before any merge
            exs[r].local_knn(subs[r], qd, algo=step % 2, stream=streams[r])
            exs[r].signal(stream=streams[r])
        outs = [exs[r].merge(sl[r].start, sl[r].stop - sl[r].start, stream=streams[r]) for r in range(P)]
        torch.cuda.synchronize()
        for r in range(P):
            assert not exs[r].timed_out()
            gi, gd = outs[r][0].cpu().numpy(), outs[r][1].cpu().numpy()
            assert np.array_equal(gi, exp[0][sl[r]]), f"P={P} rank {r} step {step} ids"
            assert np.array_equal(gd.view(np.uint32), exp[1][sl[r]].view(np.uint32)), f"P={P} rank {r} dists"
    _free_all(exs, subs)


@pytest.mark.parametrize("P,chunks", [(2, 3), (3, 4), (4, 1)])
def test_exchange_chunked_overlap(P, chunks):
    """Chunked mode (dist.data_sharded_knn_p2p): chunk c is searched and signalled
    on each rank's main stream while chunk c's merge runs on its side stream; the
    rows each rank merged (dist.chunk_rows) equal the oracle. Host issue order:
    all ranks' search+signal of a chunk, then all ranks' merges of it."""
    from paper_conf_icpp_namkn16_b200 import dist as pdist
    k = 32
    pts, qs, qd, subs, exs = _setup(P, k, q=2000)
    exp = oracle.Tree(pts).knn(qs, k)
    mains = [torch.cuda.Stream() for _ in range(P)]
    sides = [torch.cuda.Stream() for _ in range(P)]
    cb = pdist.shard_bounds(len(qs), chunks)
    rows = [pdist.chunk_rows(len(qs), P, r, chunks) for r in range(P)]
    for step in range(2):
        outs = []
        for r in range(P):
            exs[r].begin()
            n = sum(s.stop - s.start for s in rows[r])
            outs.append((torch.empty((n, k), dtype=torch.int32, device="cuda"),
                         torch.empty((n, k), dtype=torch.float32, device="cuda")))
            sides[r].wait_stream(torch.cuda.current_stream())
            mains[r].wait_stream(torch.cuda.current_stream())
        off = [0] * P
        for c in range(chunks):
            for r in range(P):
                exs[r].local_knn(subs[r], qd, stream=mains[r], rows=slice(cb[c], cb[c + 1]))
                exs[r].signal(cb[c + 1], stream=mains[r])
            for r in range(P):
                s = rows[r][c]
                n = s.stop - s.start
                exs[r].merge(s.start, n, stream=sides[r], out=(outs[r][0][off[r]:off[r] + n],
                                                               outs[r][1][off[r]:off[r] + n]))
                off[r] += n
        torch.cuda.synchronize()
        seen = np.zeros(len(qs), bool)
        for r in range(P):
            assert not exs[r].timed_out()
            idx = np.concatenate([np.arange(s.start, s.stop) for s in rows[r]])
            seen[idx] = True
            assert np.array_equal(outs[r][0].cpu().numpy(), exp[0][idx]), f"rank {r} step {step}"
            assert np.array_equal(outs[r][1].cpu().numpy().view(np.uint32), exp[1][idx].view(np.uint32))
        assert seen.all()
    _free_all(exs, subs)


def test_exchange_fewer_queries_than_parts_back_to_back():
    """q < parts: some ranks own no rows, yet every merge still waits for its
    epoch (psb.h), so epochs can run back to back without host synchronisation
    and the double-buffered lists are never overwritten while a peer reads them."""
    P, k = 5, 8
    pts, qs, qd, subs, exs = _setup(P, k, n=20_000, q=3)
    exp = oracle.knn_bruteforce(pts, qs, k)
    streams = [torch.cuda.Stream() for _ in range(P)]
    sl = _slices(len(qs), P)
    results = []
    for step in range(6):
        for r in range(P):
            exs[r].local_knn(subs[r], qd, algo=step % 2, stream=streams[r])
            exs[r].signal(stream=streams[r])
        results.append([exs[r].merge(sl[r].start, sl[r].stop - sl[r].start, stream=streams[r]) for r in range(P)])
    torch.cuda.synchronize()
    for outs in results:
        for r in range(P):
            assert np.array_equal(outs[r][0].cpu().numpy(), exp[0][sl[r]])
            assert np.array_equal(outs[r][1].cpu().numpy().view(np.uint32), exp[1][sl[r]].view(np.uint32))
    assert not any(e.timed_out() for e in exs)
    _free_all(exs, subs)


def test_exchange_timeout_pads_rows_and_is_sticky():
    """A peer that never signals: the wait gives up after the timeout, the merge
    writes (-1, +inf) pad rows (never stale or partial rows), and every later
    call on the exchange fails with PSB_ECUDA."""
    psb = _psb()
    P, k = 2, 16
    pts, qs, qd, subs, exs = _setup(P, k, n=20_000, q=100, timeout=0.2)
    exs[0].local_knn(subs[0], qd)
    exs[0].signal()                                        # rank 1 never signals
    oi, od = exs[0].merge(0, 50)
    torch.cuda.synchronize()
    assert exs[0].timed_out()
    assert (oi.cpu().numpy() == -1).all() and np.isinf(od.cpu().numpy()).all()
    with pytest.raises(psb.PSBError) as ei:
        exs[0].local_knn(subs[0], qd)
    assert ei.value.code == psb.PSB_ECUDA
    with pytest.raises(psb.PSBError):
        exs[0].merge(0, 50)
    assert not exs[1].timed_out()
    _free_all(exs, subs)


_LAUNCH_BLOCKING_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import oracle, workloads as W, paper_conf_icpp_namkn16_b200 as psb
cfg = W.config("C2"); pts = cfg.points(n=40_000); qs = cfg.queries(q=301); k = 32; P = 3
exp = oracle.knn_bruteforce(pts, qs, k)
qd = torch.from_numpy(qs).cuda()
b = [len(pts) * r // P for r in range(P + 1)]
subs = [psb.psb_build_ex(pts[b[r]:b[r + 1]], 64, id_base=b[r]) for r in range(P)]
exs = [psb.Exchange(P, r, len(qs), k) for r in range(P)]
for e in exs: e.set_timeout(2.0)
bl = [e.handle() for e in exs]
for e in exs: e.connect(bl)
st = [torch.cuda.Stream() for _ in range(P)]
sl = [slice(len(qs) * r // P, len(qs) * (r + 1) // P) for r in range(P)]
for step in range(2):
    for r in range(P):
        exs[r].local_knn(subs[r], qd, stream=st[r]); exs[r].signal(stream=st[r])
    outs = [exs[r].merge(sl[r].start, sl[r].stop - sl[r].start, stream=st[r]) for r in range(P)]
    torch.cuda.synchronize()
    for r in range(P):
        ok = np.array_equal(outs[r][0].cpu().numpy(), exp[0][sl[r]]) and not exs[r].timed_out()
        if not ok: print("WRONG", step, r); sys.exit(1)
print("OK")
"""


def test_exchange_under_cuda_launch_blocking(tmp_path):
    """With every kernel serialised (CUDA_LAUNCH_BLOCKING=1, as under ncu) the
    in-process exchange still returns the oracle's rows: no merge is queued
    ahead of a signal it waits for."""
    import subprocess
    import sys
    f = tmp_path / "lb.py"
    f.write_text(_LAUNCH_BLOCKING_SCRIPT)
    env = dict(os.environ, CUDA_LAUNCH_BLOCKING="1")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, str(f), root], env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "OK" in r.stdout, r.stdout + r.stderr


def test_nccl_route_single_rank_group_with_merge():
    """The north_star's NCCL route end to end on one GPU: a one-rank NCCL group,
    dist.data_sharded_knn whose local step searches P in-process sub-trees
    ([P, q, k]), a real NCCL all_gather_into_tensor, then psb_merge_topk. Equal to
    the oracle on the unsharded set."""
    import torch.distributed as dist
    from paper_conf_icpp_namkn16_b200 import dist as pdist
    psb = _psb()
    P, k = 4, 32
    cfg = W.config("C2")
    pts = cfg.points(n=100_000)
    qs = cfg.queries(q=1500)
    exp = oracle.Tree(pts).knn(qs, k)
    b = pdist.shard_bounds(len(pts), P)
    subs = [psb.psb_build_ex(pts[b[r]:b[r + 1]], 64, id_base=b[r]) for r in range(P)]
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(_free_port()))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        def local(qq, kk):
            oi = torch.empty((P, qq.shape[0], kk), dtype=torch.int32, device="cuda")
            od = torch.empty((P, qq.shape[0], kk), dtype=torch.float32, device="cuda")
            for r in range(P):
                psb.psb_knn(subs[r], qq, kk, out=(oi[r], od[r]))
            return oi, od
        gi, gd = pdist.data_sharded_knn(local, pdist.device_merge, torch.from_numpy(qs).cuda(), k)
        torch.cuda.synchronize()
        assert np.array_equal(gi.cpu().numpy(), exp[0])
        assert np.array_equal(gd.cpu().numpy().view(np.uint32), exp[1].view(np.uint32))
    finally:
        dist.destroy_process_group()
        for s in subs:
            s.free()


def test_exchange_argument_errors():
    psb = _psb()
    with pytest.raises(psb.PSBError):
        psb.Exchange(0, 0, 10, 8)
    with pytest.raises(psb.PSBError):
        psb.Exchange(2, 2, 10, 8)
    with pytest.raises(psb.PSBError):
        psb.Exchange(2, 0, 10, 129)
    a = psb.Exchange(2, 0, 10, 8)
    with pytest.raises(psb.PSBError):                      # not connected yet
        a.begin(); a.step(0, 5)
    with pytest.raises(psb.PSBError):
        a.signal()
    b = psb.Exchange(2, 1, 11, 8)
    with pytest.raises(psb.PSBError):                      # q differs
        a.connect([a.handle(), b.handle()])
    a.free(); b.free()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _ipc_worker(rank, world, port, q_out, chunks=1):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    psb = _psb()
    from paper_conf_icpp_namkn16_b200 import dist as pdist
    cfg = W.config("C2")
    pts = cfg.points(n=120_000)
    qs = cfg.queries(q=777)
    k = 32
    b = pdist.shard_bounds(len(pts), world)
    idx = psb.psb_build_ex(pts[b[rank]:b[rank + 1]], 64, id_base=b[rank])
    qd = torch.from_numpy(qs).cuda()
    ex = pdist.peer_exchange(len(qs), k)
    rows = np.concatenate([np.arange(s.start, s.stop) for s in pdist.chunk_rows(len(qs), world, rank, chunks)])
    exp = oracle.knn_bruteforce(pts, qs[rows], k)
    ok = True
    for _ in range(3):
        gi, gd = pdist.data_sharded_knn_p2p(ex, idx, qd, chunks=chunks)
        torch.cuda.synchronize()
        ok &= np.array_equal(gi.cpu().numpy(), exp[0])
        ok &= np.array_equal(gd.cpu().numpy().view(np.uint32), exp[1].view(np.uint32))
        ok &= not ex.timed_out()
        dist.barrier()
    q_out.put((rank, bool(ok)))
    dist.barrier()
    ex.free()
    idx.free()
    dist.destroy_process_group()


@pytest.mark.parametrize("chunks", [1, 3])
def test_exchange_two_processes_cuda_ipc(chunks):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    qo = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, qo, chunks)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(qo.get(timeout=600) for _ in procs)
    for p in procs:
        p.join(timeout=120)
    assert res == {0: True, 1: True}
