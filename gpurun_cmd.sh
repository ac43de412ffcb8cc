timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
python - <<'PY'
import torch, time, numpy as np, workloads as W, paper_conf_icpp_namkn16_b200 as psb
for name in ("C2","C3","C4"):
    cfg=W.config(name); idx=psb.psb_build(cfg.points(), cfg.fanout); qs=cfg.queries(q=64)
    hq=torch.from_numpy(qs).pin_memory()
    for parts in (1, 16, 64, 256, 1024, 0):
        lat=[]
        for i in range(40):
            x=hq[i%64:i%64+1]; torch.cuda.synchronize(); t0=time.perf_counter()
            ids,d=psb.psb_knn_split(idx,x,cfg.k,parts=parts); torch.cuda.synchronize(); lat.append((time.perf_counter()-t0)*1e6)
        lat=sorted(lat[5:]); print(name,"parts",parts,"p50 us",round(lat[len(lat)//2],1), flush=True)
    idx.free()
PY
