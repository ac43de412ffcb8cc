timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
python - <<'PY'
import torch, time, numpy as np, workloads as W, paper_conf_icpp_namkn16_b200 as psb
for name in ("C2","C4"):
    cfg=W.config(name); pts=cfg.points(); qd=torch.from_numpy(cfg.queries()).cuda()
    for pack in (psb.PSB_PACK_HILBERT, psb.PSB_PACK_KMEANS):
      for sph in (0, psb.PSB_NODE_SPHERE):
        torch.cuda.synchronize(); t0=time.time(); idx=psb.psb_build_ex(pts, cfg.fanout, packing=pack|sph); torch.cuda.synchronize(); tb=time.time()-t0
        for algo in (0,1):
            ts=[]
            for i in range(6):
                s=torch.cuda.Event(enable_timing=True); e=torch.cuda.Event(enable_timing=True)
                s.record(); psb.psb_knn_ex(idx,qd,cfg.k,algo=algo); e.record(); torch.cuda.synchronize(); ts.append(s.elapsed_time(e))
            _,_,st=psb.psb_knn_stats(idx,qd,cfg.k,algo=algo); torch.cuda.synchronize()
            m=st.float().mean(0).cpu().numpy()
            print(name, "kmeans" if pack else "hilbert", "sphere" if sph else "mbr", "psb" if algo==0 else "bnb", f"build {tb:.2f}s  {np.median(ts[2:]):.3f} ms  fetch {m[0]:.1f} leaf {m[1]:.1f}", flush=True)
        idx.free()
PY
