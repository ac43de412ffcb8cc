"""A/B of batch scheduling (closest-leaf query order vs input order) with the bench's
L2 flush between launches; checks both orders return identical rows. Dev aid."""
import os, sys, statistics
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

for name in sys.argv[1:] or ["C2", "C3", "C4", "C5"]:
    cfg = W.config(name)
    if name == "C5":
        b = pdist.shard_bounds(cfg.n, 8)
        pts = cfg.points(n=b[1] - b[0], row0=0)
    else:
        pts = cfg.points()
    qd = torch.from_numpy(cfg.queries()).cuda()
    idx = psb.psb_build(pts, cfg.fanout)
    for algo, an in (("psb", 0), ("bnb", 1)):
        r = {}
        outs = {}
        for var in (psb.PSB_VAR_INPUT_ORDER, psb.PSB_VAR_LEAF_ORDER):
            outs[var] = psb.psb_knn_ex(idx, qd, cfg.k, algo=an, variant=var)
            r[var] = t(lambda: psb.psb_knn_ex(idx, qd, cfg.k, algo=an, variant=var))
        same = all(torch.equal(a, b) for a, b in zip(outs[psb.PSB_VAR_LEAF_ORDER], outs[psb.PSB_VAR_INPUT_ORDER]))
        r[0] = r[psb.PSB_VAR_LEAF_ORDER]
        print(f"{name} {algo}: input order {r[psb.PSB_VAR_INPUT_ORDER]:.3f} ms  leaf order {r[0]:.3f} ms  "
              f"speedup {r[psb.PSB_VAR_INPUT_ORDER]/r[0]:.2f}x  identical={same}", flush=True)
    idx.free()
