"""Kernels of one latency-mode query (dev aid, run under ncu --metrics gpu__time_duration.sum).
usage: lat_kernels.py CONFIG"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
cfg = W.config(sys.argv[1])
idx = psb.psb_build(cfg.points(), cfg.fanout)
qd = torch.from_numpy(cfg.queries(8)).cuda()
for i in range(4):
    psb.psb_knn_split(idx, qd[i:i + 1], cfg.k, parts=0)
torch.cuda.synchronize()
