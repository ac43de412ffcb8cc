"""Where PSB's and B&B's leaf scans go (dev aid): per algorithm, leaf scans per query split
into pass 1 / pass-2 right siblings of a changing leaf (Alg. 1 l.41) / pass-2 eligible
descents, and whether each scanned leaf was needed (leaf MINDIST <= the final k-th
distance: no exact traversal can skip it). usage: waste.py CONFIG [NQ]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
from paper_conf_icpp_namkn16_b200 import dist as pdist

name = sys.argv[1]; nq = int(sys.argv[2]) if len(sys.argv) > 2 else 2000
cfg = W.config(name)
if name == "C5":
    b = pdist.shard_bounds(cfg.n, 8); pts = cfg.points(n=b[1] - b[0], row0=0)
else:
    pts = cfg.points()
qs = cfg.queries(nq)
idx = psb.psb_build(pts, cfg.fanout)
blob = psb.psb_index_export(idx)
F, d = cfg.fanout, cfg.d
lv1 = blob["nodes"][1]                     # [nodes, d, 2, F]
lo = np.transpose(lv1[:, :, 0, :], (0, 2, 1)).reshape(-1, d)[: blob["leaves"]]
hi = np.transpose(lv1[:, :, 1, :], (0, 2, 1)).reshape(-1, d)[: blob["leaves"]]
qd = torch.from_numpy(qs).cuda()
for algo, an in (("psb", 0), ("bnb", 1)):
    ids, dd, st, tr, tl = psb.psb_knn_trace(idx, qd, cfg.k, cap=16384, algo=an)
    torch.cuda.synchronize()
    tr, tl, dk = tr.cpu().numpy(), tl.cpu().numpy(), dd[:, -1].cpu().numpy()
    cat = {"pass1": [0, 0], "right_sibling": [0, 0], "descent": [0, 0]}
    for r in range(nq):
        steps = tr[r, : tl[r]]
        lvl = (steps >> 32) & 0xFF; node = steps & 0xFFFFFFFF; fl = (steps >> 40) & 0xFF
        leaf = (lvl == 0) & ((fl & psb.PSB_TRACE_SKIPPED) == 0)
        prev_changed = np.zeros(len(steps), bool)
        prev_changed[1:] = (lvl[:-1] == 0) & ((fl[:-1] & psb.PSB_TRACE_CHANGED) != 0) & ((fl[:-1] & psb.PSB_TRACE_PASS1) == 0)
        js = node[leaf]
        q = qs[r].astype(np.float64)
        a = np.maximum(np.maximum(lo[js] - q, q - hi[js]), 0.0)
        need = (a * a).sum(1) <= float(dk[r]) * (1 + 1e-6)
        p1 = (fl[leaf] & psb.PSB_TRACE_PASS1) != 0
        rs = prev_changed[leaf] & ~p1
        for key, m in (("pass1", p1), ("right_sibling", rs), ("descent", ~p1 & ~rs)):
            cat[key][0] += int(m.sum()); cat[key][1] += int((m & need).sum())
    tot = sum(v[0] for v in cat.values()); tn = sum(v[1] for v in cat.values())
    print(f"{name} {algo}: leaves/q {tot/nq:.1f} (needed {tn/nq:.1f}) | " +
          " | ".join(f"{k} {v[0]/nq:.1f} (needed {v[1]/nq:.1f})" for k, v in cat.items()), flush=True)
