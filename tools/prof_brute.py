import os, sys
sys.path.insert(0, '/root/repo')
import torch, paper_conf_icpp_namkn16_b200 as psb, workloads as W
cfg = W.config(sys.argv[1]); nq = int(sys.argv[2])
idx = psb.psb_build(cfg.points(), cfg.fanout)
qd = torch.from_numpy(cfg.queries(nq)).cuda()
for _ in range(2): psb.psb_knn_bruteforce(idx, qd, cfg.k)
torch.cuda.synchronize()
