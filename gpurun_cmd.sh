timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
python - <<'PY'
import torch, numpy as np, workloads as W, paper_conf_icpp_namkn16_b200 as psb
cfg=W.config("C2"); idx=psb.psb_build(cfg.points(), cfg.fanout); qd=torch.from_numpy(cfg.queries(q=2000)).cuda()
for k in (1, 8, 32, 64, 128, 256, 512, 1024, 2048):
    row=[]
    for algo in (0,1,2):
        ts=[]
        for i in range(5):
            s=torch.cuda.Event(enable_timing=True); e=torch.cuda.Event(enable_timing=True)
            s.record(); psb.psb_knn_ex(idx,qd,k,algo=algo); e.record(); torch.cuda.synchronize(); ts.append(s.elapsed_time(e))
        row.append(np.median(ts[1:]))
    print(f"k={k:5d} psb {row[0]:8.3f} ms  bnb {row[1]:8.3f} ms  brute {row[2]:8.3f} ms", flush=True)
PY
