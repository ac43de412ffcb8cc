"""Quick per-algorithm batch timing on the GPU (development aid, not the bench)."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W

def time_it(fn, reps=15):
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    fn(); torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        s.record(); fn(); e.record(); torch.cuda.synchronize(); ts.append(s.elapsed_time(e))
    return min(ts), float(np.median(ts))

for name in [a for a in sys.argv[1:] if not a.startswith("-")] or ["C1", "C2", "C3"]:
    cfg = W.config(name)
    t0 = time.time(); pts = cfg.points(); qs = cfg.queries(); t1 = time.time()
    idx = psb.psb_build(pts, cfg.fanout); torch.cuda.synchronize(); t2 = time.time()
    if "--build" in os.environ.get("QT_FLAGS", ""):
        th = time.time(); psb.psb_build_ex(pts, cfg.fanout, packing=psb.PSB_BUILD_HOST).free(); th = time.time() - th
        print(f"{name}: host build {th:.2f}s", flush=True)
    qd = torch.from_numpy(qs).cuda()
    print(f"{name}: gen {t1-t0:.1f}s build {t2-t1:.1f}s info {idx.info()}", flush=True)
    for algo, an in (("psb", 0), ("bnb", 1), ("brute", 2)):
        for var in ((0, 1) if an < 2 else (0,)):
            if an == 2 and cfg.n * cfg.q > 2e10: 
                continue
            mn, med = time_it(lambda: psb.psb_knn_ex(idx, qd, cfg.k, algo=an, variant=var))
            print(f"  {algo:6s} var{var}: {med:9.3f} ms (min {mn:.3f})  {cfg.q/med*1e3/1e6:8.3f} Mq/s", flush=True)
    idx.free()
