"""Would a Hilbert-key pre-pass order the batch as well as the closest-leaf pre-pass?
(dev aid) Queries sorted on the host by their Hilbert key (the bulk loader's transform,
b = min(64 // d, 21) bits per axis, over the points' bounding box), then run in input
order, against the default (closest-leaf pre-pass + sort inside the launch).
usage: hilbert_order_ab.py CONFIG"""
import os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
from paper_conf_icpp_namkn16_b200 import dist as pdist


def hilbert_keys(x, mn, mx, b):
    n, d = x.shape
    top = (1 << b) - 1
    ext = (mx - mn).astype(np.float64)
    u = np.floor(np.where(ext > 0, (x.astype(np.float64) - mn) / np.where(ext > 0, ext, 1) * top, 0.0))
    X = np.clip(u, 0, top).astype(np.uint64)
    M = np.uint64(1 << (b - 1))
    Q = M
    while Q > 1:
        P = Q - np.uint64(1)
        for j in range(d):
            hit = (X[:, j] & Q) != 0
            X[hit, 0] ^= P
            t = (X[~hit, 0] ^ X[~hit, j]) & P
            X[~hit, 0] ^= t
            X[~hit, j] ^= t
        Q >>= np.uint64(1)
    for j in range(1, d):
        X[:, j] ^= X[:, j - 1]
    t = np.zeros(n, np.uint64)
    Q = M
    while Q > 1:
        t[(X[:, d - 1] & Q) != 0] ^= Q - np.uint64(1)
        Q >>= np.uint64(1)
    X ^= t[:, None]
    hi = np.zeros(n, np.uint64)
    lo = np.zeros(n, np.uint64)
    for q in range(b - 1, -1, -1):
        for j in range(d):
            hi = (hi << np.uint64(1)) | (lo >> np.uint64(63))
            lo = (lo << np.uint64(1)) | ((X[:, j] >> np.uint64(q)) & np.uint64(1))
    return hi, lo


name = sys.argv[1]
cfg = W.config(name)
if name == "C5":
    bnd = pdist.shard_bounds(cfg.n, 8); pts = cfg.points(n=bnd[1] - bnd[0], row0=0)
else:
    pts = cfg.points()
qs = cfg.queries()
idx = psb.psb_build(pts, cfg.fanout)
b = int(sys.argv[2]) if len(sys.argv) > 2 else min(64 // cfg.d, 21)
khi, klo = hilbert_keys(qs, pts.min(0), pts.max(0), b)
perm = np.lexsort((klo, khi))
qd = torch.from_numpy(qs).cuda()
qh = torch.from_numpy(qs[perm].copy()).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def t(fn, reps=10):
    ts = []
    for i in range(reps + 2):
        flush.fill_(i & 0xFF)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(); fn(); e.record(); torch.cuda.synchronize()
        if i >= 2: ts.append(s.elapsed_time(e))
    return statistics.median(ts)


ref = psb.psb_knn_ex(idx, qd, cfg.k)
got = psb.psb_knn_ex(idx, qh, cfg.k, variant=psb.PSB_VAR_INPUT_ORDER)
inv = np.empty_like(perm); inv[perm] = np.arange(len(perm))
same = all(torch.equal(a[torch.from_numpy(inv).cuda()], r) for a, r in zip(got, ref))
print(f"{name}: default (closest-leaf pre-pass + sort) {t(lambda: psb.psb_knn_ex(idx, qd, cfg.k)):.3f} ms | "
      f"input order, unsorted {t(lambda: psb.psb_knn_ex(idx, qd, cfg.k, variant=psb.PSB_VAR_INPUT_ORDER)):.3f} ms | "
      f"input order, host Hilbert-sorted ({b} bits/axis) "
      f"{t(lambda: psb.psb_knn_ex(idx, qh, cfg.k, variant=psb.PSB_VAR_INPUT_ORDER)):.3f} ms | rows equal {same}")
