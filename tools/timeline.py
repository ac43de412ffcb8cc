"""Batch timeline from the per-query %globaltimer stamps of psb_knn_stats (dev aid):
when the queue drains, how long the last queries run, busy warps over time.
usage: timeline.py CONFIG [algo]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
cfg = W.config(sys.argv[1]); algo = int(sys.argv[2]) if len(sys.argv) > 2 else 0
idx = psb.psb_build(cfg.points(), cfg.fanout)
qd = torch.from_numpy(cfg.queries()).cuda()
for rep in range(3):
    _, _, st = psb.psb_knn_stats(idx, qd, cfg.k, algo=algo)
torch.cuda.synchronize()
st = st.cpu().numpy()
t0 = st[:, 6].min(); s = (st[:, 6] - t0) / 1e3; e = (st[:, 7] - t0) / 1e3
span = e.max(); drain = s.max(); dur = e - s
print(f"{cfg.name} algo {algo}: span {span:.1f} us, queue drained at {drain:.1f} us ({100*drain/span:.0f}%), "
      f"service p50 {np.median(dur):.1f} p99 {np.percentile(dur, 99):.1f} max {dur.max():.1f} us")
for f in (0.5, 0.6, 0.7, 0.8, 0.9, 0.95):
    t = f * span
    print(f"  t={t:7.1f} us: {int(((s <= t) & (e > t)).sum()):5d} queries running")
lv = st[:, 1]
late = s > drain - 0.05 * span
print(f"  queries started in the last 5% before drain: {late.sum()}, their leaves mean {lv[late].mean():.0f}; "
      f"longest query: {lv[np.argmax(dur)]} leaves, started at {s[np.argmax(dur)]:.1f} us")
c = np.corrcoef(lv, dur)[0, 1]
print(f"  corr(leaf scans, service time) = {c:.3f}; us per leaf (median) {np.median(dur / np.maximum(lv, 1)):.3f}")
ids, d = psb.psb_knn(idx, qd, cfg.k)
kd = d[:, -1].cpu().numpy()
top = np.argsort(-dur)[:10]
print("  longest queries: service us / leaves / changing / keys merged / node fetches / k-th dist")
for i in top:
    print(f"   q{i:6d}: {dur[i]:7.1f} {st[i,1]:6d} {st[i,4]:5d} {st[i,5]:6d} {st[i,0]:5d} {kd[i]:10.2f}")
print(f"  median: {np.median(dur):7.1f} {np.median(st[:,1]):6.0f} {np.median(st[:,4]):5.0f} {np.median(st[:,5]):6.0f} "
      f"{np.median(st[:,0]):5.0f} {np.median(kd):10.2f}")
