"""q/s of one config at several batch sizes (tail-effect check). Dev aid.
usage: qscale.py CONFIG ALGO Q [Q ...]"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
name, algo = sys.argv[1], {"psb": 0, "bnb": 1}[sys.argv[2]]
cfg = W.config(name)
idx = psb.psb_build(cfg.points(), cfg.fanout)
allq = torch.from_numpy(cfg.queries(max(int(x) for x in sys.argv[3:]))).cuda()
for qn in map(int, sys.argv[3:]):
    qd = allq[:qn].contiguous()
    ts = []
    for i in range(12):
        flush.fill_(i & 0xFF)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(); psb.psb_knn_ex(idx, qd, cfg.k, algo=algo); e.record(); torch.cuda.synchronize()
        if i >= 2: ts.append(s.elapsed_time(e))
    ms = statistics.median(ts)
    print(f"{name} {sys.argv[2]} q={qn}: {ms:.3f} ms  {qn / ms / 1e3:.2f} Mq/s", flush=True)
