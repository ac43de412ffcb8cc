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


@pytest.mark.parametrize("P,k", [(3, 32), (2, 7), (5, 64), (1, 16)])
def test_exchange_in_process(P, k):
    psb = _psb()
    cfg = W.config("C2")
    pts = cfg.points(n=150_000)
    qs = cfg.queries(q=1003)
    exp = oracle.Tree(pts).knn(qs, k)
    qd = torch.from_numpy(qs).cuda()
    bounds = [len(pts) * r // P for r in range(P + 1)]
    subs = [psb.psb_build_ex(pts[bounds[r]:bounds[r + 1]], 64, id_base=bounds[r]) for r in range(P)]
    exs = [psb.Exchange(P, r, len(qs), k) for r in range(P)]
    blobs = [e.handle() for e in exs]
    for e in exs:
        e.connect(blobs)
    streams = [torch.cuda.Stream() for _ in range(P)]
    sl = _slices(len(qs), P)
    for step in range(3):                                  # epochs 1..3: buffer parity alternates
        for r in range(P):
            exs[r].local_knn(subs[r], qd, algo=step % 2, stream=streams[r])
        torch.cuda.synchronize()
        outs = [exs[r].step(sl[r].start, sl[r].stop - sl[r].start, stream=streams[r]) for r in range(P)]
        torch.cuda.synchronize()
        for r in range(P):
            assert not exs[r].timed_out()
            gi, gd = outs[r][0].cpu().numpy(), outs[r][1].cpu().numpy()
            assert np.array_equal(gi, exp[0][sl[r]]), f"P={P} rank {r} step {step} ids"
            assert np.array_equal(gd.view(np.uint32), exp[1][sl[r]].view(np.uint32)), f"P={P} rank {r} dists"
    for e in exs:
        e.free()
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


def _ipc_worker(rank, world, port, q_out):
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
    exp = oracle.knn_bruteforce(pts, qs[pdist.query_slice(len(qs), world, rank)], k)
    ok = True
    for _ in range(3):
        gi, gd = pdist.data_sharded_knn_p2p(ex, idx, qd)
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


def test_exchange_two_processes_cuda_ipc():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    qo = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, qo)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(qo.get(timeout=600) for _ in procs)
    for p in procs:
        p.join(timeout=120)
    assert res == {0: True, 1: True}
