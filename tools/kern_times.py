"""Per-kernel device times of one psb_knn_ex batch (CUPTI via torch.profiler), dev aid.
usage: kern_times.py CONFIG [variant ...]   (PSB_SHARE_BUDGET is read from the environment)"""
import os, sys, collections
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from torch.profiler import ProfilerActivity, profile
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
cfg = W.config(sys.argv[1])
idx = psb.psb_build(cfg.points(), cfg.fanout)
qd = torch.from_numpy(cfg.queries()).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for var in [int(v) for v in sys.argv[2:]] or [0]:
    for _ in range(3):
        psb.psb_knn_ex(idx, qd, cfg.k, variant=var)
    agg = collections.defaultdict(list)
    for _ in range(5):
        flush.zero_(); torch.cuda.synchronize()
        with profile(activities=[ProfilerActivity.CUDA]) as prof:
            psb.psb_knn_ex(idx, qd, cfg.k, variant=var)
            torch.cuda.synchronize()
        for ev in prof.events():
            if ev.device_type == torch.autograd.DeviceType.CUDA:
                agg[ev.name.split("(")[0].replace("void ", "")[:60]].append(ev.device_time_total / 1e3)
    tot = 0.0
    for n, v in agg.items():
        v.sort(); m = v[len(v) // 2]; tot += m
        print(f"{cfg.name} var {var:2d} budget {os.environ.get('PSB_SHARE_BUDGET', '-'):>4}: {m:8.4f} ms  {n}")
    print(f"{cfg.name} var {var:2d} total {tot:.4f} ms", flush=True)
