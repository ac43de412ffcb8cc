"""Batch ms of psb_knn_ex (variant 0 and a baseline variant) under different values of a
library environment knob, one subprocess per value (the library reads it once). Dev aid.
usage: env_ab.py ENVVAR CONFIG BASEVARIANT value [value ...]"""
import os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r"""
import sys, statistics, torch
sys.path.insert(0, sys.argv[1])
import paper_conf_icpp_namkn16_b200 as psb, workloads as W
from paper_conf_icpp_namkn16_b200 import dist as pdist
name = sys.argv[2]
cfg = W.config("C5" if name == "C5W" else name)
if name == "C5":
    b = pdist.shard_bounds(cfg.n, 8); pts = cfg.points(n=b[1] - b[0], row0=0)
else:
    pts = cfg.points()
idx = psb.psb_build(pts, cfg.fanout)
qd = torch.from_numpy(cfg.queries()).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
def t(var, reps=10):
    ts = []
    for i in range(reps + 2):
        flush.fill_(i & 0xFF)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(); psb.psb_knn_ex(idx, qd, cfg.k, variant=var); e.record(); torch.cuda.synchronize()
        if i >= 2: ts.append(s.elapsed_time(e))
    return statistics.median(ts)
for var in [int(v, 0) for v in sys.argv[4].split(",")]:
    print(f"{name} {sys.argv[3]} var {var:#x}: {t(var):.4f} ms", flush=True)
"""
env, cfgname, base = sys.argv[1], sys.argv[2], sys.argv[3]
for n, v in enumerate(sys.argv[4:]):
    vs = f"{base},0" if n == 0 else "0"
    subprocess.run([sys.executable, "-c", CHILD, ROOT, cfgname, f"{env}={v}", vs], env={**os.environ, env: v})
