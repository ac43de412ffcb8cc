"""One warm-up launch then one profiled launch of a tree kernel (for ncu -k/-c). Dev aid.
usage: prof_one.py CONFIG ALGO(psb|psb_split|bnb|brute) [VARIANT]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
from paper_conf_icpp_namkn16_b200 import dist as pdist

name, algo = sys.argv[1], sys.argv[2]
var = int(sys.argv[3]) if len(sys.argv) > 3 else 0
cfg = W.config(name)
if name == "C5":
    b = pdist.shard_bounds(cfg.n, 8)
    pts = cfg.points(n=b[1] - b[0], row0=0)
else:
    pts = cfg.points()
qd = torch.from_numpy(cfg.queries()).cuda()
idx = psb.psb_build(pts, cfg.fanout)
a = {"psb": 0, "psb_split": 0, "bnb": 1, "brute": 2}[algo]
for _ in range(2):
    if algo == "psb_split":
        psb.psb_knn_split(idx, qd, cfg.k, parts=0)
    else:
        psb.psb_knn_ex(idx, qd, cfg.k, algo=a, variant=var)
torch.cuda.synchronize()
idx.free()
