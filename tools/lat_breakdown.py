"""Single-query latency breakdown (dev aid): where the ~50 us of a one-query call go.
usage: lat_breakdown.py CONFIG"""
import ctypes, os, statistics, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
from paper_conf_icpp_namkn16_b200 import dist as pdist

name = sys.argv[1]
cfg = W.config(name)
if name == "C5":
    b = pdist.shard_bounds(cfg.n, 8); pts = cfg.points(n=b[1] - b[0], row0=0)
else:
    pts = cfg.points()
qs = cfg.queries(2000)
idx = psb.psb_build(pts, cfg.fanout)
k = cfg.k
hq = torch.from_numpy(qs).pin_memory()
dq = hq.cuda()
hi = torch.empty((1, k), dtype=torch.int32, pin_memory=True)
hd = torch.empty((1, k), dtype=torch.float32, pin_memory=True)
di = torch.empty((1, k), dtype=torch.int32, device="cuda")
dd = torch.empty((1, k), dtype=torch.float32, device="cuda")
st = torch.cuda.current_stream()
x1 = torch.zeros(1, device="cuda")


def lat(call, n=400):
    ts = []
    for i in range(n + 20):
        torch.cuda.synchronize()
        t0 = time.perf_counter(); call(i % 2000); st.synchronize()
        if i >= 20: ts.append((time.perf_counter() - t0) * 1e6)
    return statistics.median(ts)


def ev(call, n=200):
    ts = []
    for i in range(n + 10):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(); call(i % 2000); e.record(); torch.cuda.synchronize()
        if i >= 10: ts.append(s.elapsed_time(e) * 1e3)
    return statistics.median(ts)


lib = psb._lib
h = idx.handle
sh = int(st.cuda_stream)
res = {
    "sync_only": lat(lambda i: None),
    "torch_add_sync": lat(lambda i: x1.add_(1)),
    "python_host_bufs": lat(lambda i: psb.psb_knn_ex(idx, hq[i:i + 1], k, out=(hi, hd))),
    "ctypes_host_bufs": lat(lambda i: lib.psb_knn_ex(h, hq[i:i + 1].data_ptr(), 1, k, hi.data_ptr(), hd.data_ptr(), sh, 0, 0)),
    "ctypes_dev_bufs": lat(lambda i: lib.psb_knn_ex(h, dq[i:i + 1].data_ptr(), 1, k, di.data_ptr(), dd.data_ptr(), sh, 0, 0)),
    "gpu_time_dev_bufs": ev(lambda i: lib.psb_knn_ex(h, dq[i:i + 1].data_ptr(), 1, k, di.data_ptr(), dd.data_ptr(), sh, 0, 0)),
    "gpu_time_host_bufs": ev(lambda i: lib.psb_knn_ex(h, hq[i:i + 1].data_ptr(), 1, k, hi.data_ptr(), hd.data_ptr(), sh, 0, 0)),
    "split_python_host_bufs": lat(lambda i: psb.psb_knn_split(idx, hq[i:i + 1], k, parts=0, out=(hi, hd))),
    "split_gpu_time_dev_bufs": ev(lambda i: lib.psb_knn_split(h, dq[i:i + 1].data_ptr(), 1, k, 0, di.data_ptr(), dd.data_ptr(), sh)),
}
t0 = time.perf_counter()
for i in range(2000):
    lib.psb_knn_ex(h, dq[i:i + 1].data_ptr(), 1, k, di.data_ptr(), dd.data_ptr(), sh, 0, 0)
t1 = time.perf_counter()
torch.cuda.synchronize()
res["host_api_us_per_call_dev_bufs"] = (t1 - t0) / 2000 * 1e6
print(name, {a: round(v, 1) for a, v in res.items()})
