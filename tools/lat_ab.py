"""Single-query latency (launch -> results in pinned host memory, p50/p99 over N
queries) of psb_knn vs psb_knn_split at several part counts. Dev aid.
usage: lat_ab.py CONFIG N P [P ...]   (P = 0: the library's auto choice)"""
import os, sys, time, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
name, n = sys.argv[1], int(sys.argv[2])
cfg = W.config(name)
pts = cfg.points(n=cfg.n // 8, row0=0) if name == "C5" else cfg.points()
idx = psb.psb_build(pts, cfg.fanout)
hq = torch.from_numpy(cfg.queries(n)).pin_memory()
hi = torch.empty((1, cfg.k), dtype=torch.int32, pin_memory=True)
hd = torch.empty((1, cfg.k), dtype=torch.float32, pin_memory=True)
def lat(call):
    ts = []
    for i in range(n + 5):
        torch.cuda.synchronize(); t0 = time.perf_counter(); call(hq[i % n:i % n + 1]); torch.cuda.synchronize()
        if i >= 5: ts.append((time.perf_counter() - t0) * 1e6)
    ts.sort()
    return ts[len(ts) // 2], ts[int(len(ts) * 0.99)]
print(f"{name} psb: p50/p99 {lat(lambda x: psb.psb_knn(idx, x, cfg.k, out=(hi, hd)))} us", flush=True)
for p in map(int, sys.argv[3:]):
    print(f"{name} split parts={p}: p50/p99 {lat(lambda x: psb.psb_knn_split(idx, x, cfg.k, parts=p, out=(hi, hd)))} us",
          flush=True)
if os.environ.get("LAT_VARIANTS"):
    for v in map(lambda s: int(s, 0), os.environ["LAT_VARIANTS"].split(",")):
        print(f"{name} psb variant {v:#x}: p50/p99 "
              f"{lat(lambda x: psb.psb_knn_ex(idx, x, cfg.k, variant=v, out=(hi, hd)))} us", flush=True)
