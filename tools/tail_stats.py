"""Per-query work distribution (psb_knn_stats leaf scans) and its rank correlation
with the pass-1 pruning distance (the cost-order key). Dev aid. usage: tail_stats.py CONFIG"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
import oracle
name = sys.argv[1]
cfg = W.config(name)
pts = cfg.points(); qs = cfg.queries()
idx = psb.psb_build(pts, cfg.fanout)
qd = torch.from_numpy(qs).cuda()
for algo in (0, 1):
    _, _, st = psb.psb_knn_stats(idx, qd, cfg.k, algo=algo)
    leaves = st[:, 1].cpu().numpy().astype(np.float64)
    p = np.percentile(leaves, [50, 90, 99, 99.9, 100])
    srt = np.sort(leaves)[::-1]
    print(f"{name} algo {algo}: leaves/q mean {leaves.mean():.1f} p50/p90/p99/p99.9/max {p.round(0)}; "
          f"top 1% hold {srt[:len(srt)//100].sum()/srt.sum()*100:.1f}% of scans, top 0.1% {srt[:len(srt)//1000].sum()/srt.sum()*100:.1f}%")
    if algo == 0:
        ids, d = psb.psb_knn(idx, qd, cfg.k)
        r = d[:, -1].cpu().numpy()
        from scipy.stats import spearmanr
        print(f"   spearman(leaves, final k-th dist) = {spearmanr(leaves, r).correlation:.3f}")
