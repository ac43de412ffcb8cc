"""Time the CTA query-block size (PSB_QBLOCK env knob, knn_tree.cuh cta_take) on a
config (bench-style L2 flush, median of 10). Dev aid.
usage: qblock_ab.py CONFIG ALGO QB [QB ...]"""
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
name, algo = sys.argv[1], {"psb": 0, "bnb": 1}[sys.argv[2]]
var = int(os.environ.get("VAR", "0"), 0)
cfg = W.config("C5" if name == "C5W" else name)
if name == "C5":
    b = pdist.shard_bounds(cfg.n, 8); pts = cfg.points(n=b[1] - b[0], row0=0)
else:
    pts = cfg.points()
qd = torch.from_numpy(cfg.queries()).cuda()
idx = psb.psb_build(pts, cfg.fanout)
ref = None
for v in sys.argv[3:]:
    os.environ["PSB_QBLOCK"] = v
    out = psb.psb_knn_ex(idx, qd, cfg.k, algo=algo, variant=var)
    same = True if ref is None else all(torch.equal(a, b) for a, b in zip(out, ref))
    ref = ref or out
    ms = t(lambda: psb.psb_knn_ex(idx, qd, cfg.k, algo=algo, variant=var))
    print(f"{name} {sys.argv[2]} var {var:#x} qblock {v}: {ms:.3f} ms same={same}", flush=True)
