"""Batch time of psb_knn_split at several part counts (tail balancing check). Dev aid.
usage: split_ab.py CONFIG P [P ...]"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
name = sys.argv[1]
cfg = W.config(name)
idx = psb.psb_build(cfg.points(), cfg.fanout)
qd = torch.from_numpy(cfg.queries()).cuda()
ref = psb.psb_knn(idx, qd, cfg.k)
for p in map(int, sys.argv[2:]):
    out = psb.psb_knn_split(idx, qd, cfg.k, parts=p)
    same = all(torch.equal(a, b) for a, b in zip(out, ref))
    ts = []
    for i in range(12):
        flush.fill_(i & 0xFF)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(); psb.psb_knn_split(idx, qd, cfg.k, parts=p); e.record(); torch.cuda.synchronize()
        if i >= 2: ts.append(s.elapsed_time(e))
    print(f"{name} split parts={p}: {statistics.median(ts):.3f} ms same={same}", flush=True)
