"""Packing A/B (dev aid): PSB and B&B batch ms and per-query counters for Hilbert, STR and
k-means leaf packing. usage: pack_ab.py CONFIG [CONFIG ...]"""
import os, sys, statistics, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
from paper_conf_icpp_namkn16_b200 import dist as pdist
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
def t(fn, reps=10):
    ts = []
    for i in range(reps + 2):
        flush.fill_(i & 0xFF)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(); fn(); e.record(); torch.cuda.synchronize()
        if i >= 2: ts.append(s.elapsed_time(e))
    return statistics.median(ts)
for name in sys.argv[1:]:
    cfg = W.config(name)
    if name == "C5":
        b = pdist.shard_bounds(cfg.n, 8); pts = cfg.points(n=b[1] - b[0], row0=0)
    else:
        pts = cfg.points()
    qd = torch.from_numpy(cfg.queries()).cuda()
    ref = None
    for pname, pk in (("hilbert", psb.PSB_PACK_HILBERT), ("str", psb.PSB_PACK_STR), ("kmeans", psb.PSB_PACK_KMEANS)):
        t0 = time.time(); idx = psb.psb_build_ex(pts, cfg.fanout, packing=pk); torch.cuda.synchronize(); tb = time.time() - t0
        for an, a in (("psb", 0), ("bnb", 1)):
            out = psb.psb_knn_ex(idx, qd, cfg.k, algo=a)
            same = True if ref is None else all(torch.equal(x, y) for x, y in zip(out, ref))
            ref = ref or out
            ms = t(lambda: psb.psb_knn_ex(idx, qd, cfg.k, algo=a))
            _, _, st = psb.psb_knn_stats(idx, qd, cfg.k, algo=a)
            m = st[:, :6].double().mean(0).tolist()
            print(f"{name} {pname:7s} {an}: build {tb:6.2f}s {ms:8.3f} ms same={same} fetches {m[0]:.1f} leaves {m[1]:.1f} "
                  f"keys {m[5]:.1f}", flush=True)
        idx.free()
