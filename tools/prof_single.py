"""One query per launch (ncu the second launch): where a lone warp's time goes. Dev aid.
usage: prof_single.py CONFIG QUERY_INDEX [ALGO]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
cfg = W.config(sys.argv[1]); qi = int(sys.argv[2]); a = {"psb": 0, "bnb": 1}[sys.argv[3] if len(sys.argv) > 3 else "psb"]
idx = psb.psb_build(cfg.points(), cfg.fanout)
qd = torch.from_numpy(cfg.queries()[qi:qi + 1].copy()).cuda()
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for i in range(4):
    s.record(); psb.psb_knn_ex(idx, qd, cfg.k, algo=a); e.record(); torch.cuda.synchronize()
    print(f"launch {i}: {s.elapsed_time(e) * 1e3:.1f} us", flush=True)
_, _, st = psb.psb_knn_stats(idx, qd, cfg.k, algo=a)
print("stats", st.cpu().numpy()[0, :6].tolist())
