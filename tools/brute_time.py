"""Brute-force batch time and FP32-pipe fraction (dev aid; bench.py --algo brute is the
measurement). usage: brute_time.py CONFIG [NQ]"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
cfg = W.config(sys.argv[1]); nq = int(sys.argv[2]) if len(sys.argv) > 2 else cfg.q
idx = psb.psb_build(cfg.points(), cfg.fanout)
qd = torch.from_numpy(cfg.queries(nq)).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
ts = []
for i in range(5):
    flush.fill_(i)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record(); psb.psb_knn_bruteforce(idx, qd, cfg.k); e.record(); torch.cuda.synchronize()
    if i >= 1: ts.append(s.elapsed_time(e))
ms = statistics.median(ts)
lane_ops = 3.0 * cfg.n * nq * cfg.d
peak = 148 * 4 * 32 * 1.965e9
print(f"{sys.argv[1]} brute q={nq}: {ms:.3f} ms  FP32 frac {lane_ops / (ms * 1e-3) / peak:.3f}")
