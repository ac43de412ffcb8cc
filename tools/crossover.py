"""C4 crossover study (BASELINE.json configs[3], paper Fig. 5 σ values
P:L758-766): 16-D clustered points, n = 16M, F = 128, k = 64, 10^4 queries, for
σ ∈ {10, 40, 160, 640, 2560, 10240}. PSB vs GPU B&B vs GPU brute force: batch time
(L2 flushed, median of 10) and single-query latency (launch -> results in pinned host
memory, p50 of 40), per-query leaf scans; rows checked equal across the three GPU
routes and against the CPU oracle's brute force on 16 queries.
usage: crossover.py [sigma ...]   (prints one JSON line per σ)"""
import json, os, statistics, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W
import oracle

flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def batch_ms(fn, reps=10):
    ts = []
    for i in range(reps + 2):
        flush.fill_(i & 0xFF)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(); fn(); e.record(); torch.cuda.synchronize()
        if i >= 2: ts.append(s.elapsed_time(e))
    return statistics.median(ts)


def lat_us(call, hq, n=40):
    lat = []
    for i in range(n + 5):
        torch.cuda.synchronize()
        t0 = time.perf_counter(); call(hq[i % hq.shape[0]:i % hq.shape[0] + 1]); torch.cuda.synchronize()
        if i >= 5: lat.append((time.perf_counter() - t0) * 1e6)
    return statistics.median(lat)


for sigma in [float(s) for s in sys.argv[1:]] or [10, 40, 160, 640, 2560, 10240]:
    cfg = W.config("C4", sigma=sigma)
    pts, qs = cfg.points(), cfg.queries()
    idx = psb.psb_build(pts, cfg.fanout)
    qd = torch.from_numpy(qs).cuda()
    k = cfg.k
    res, ms = {}, {}
    for name, a in (("psb", 0), ("bnb", 1), ("brute", 2)):
        res[name] = psb.psb_knn_ex(idx, qd, k, algo=a)
        ms[name] = batch_ms(lambda: psb.psb_knn_ex(idx, qd, k, algo=a))
    res["psb_split"] = psb.psb_knn_split(idx, qd, k, parts=0)          # auto parts (tail splitting)
    ms["psb_split"] = batch_ms(lambda: psb.psb_knn_split(idx, qd, k, parts=0))
    same = all(torch.equal(res["psb"][j], res[o][j]) for o in ("bnb", "brute", "psb_split") for j in (0, 1))
    ei, ed = oracle.knn_bruteforce(pts, qs[:16], k)
    ok = bool(np.array_equal(res["psb"][0][:16].cpu().numpy(), ei) and
              np.array_equal(res["psb"][1][:16].cpu().numpy().view(np.uint32), ed.view(np.uint32)))
    leaves = {}
    for name, a in (("psb", 0), ("bnb", 1)):
        _, _, st = psb.psb_knn_stats(idx, qd, k, algo=a)
        leaves[name] = float(st[:, 1].double().mean())
    hq = torch.from_numpy(qs[:64].copy()).pin_memory()
    hi = torch.empty((1, k), dtype=torch.int32, pin_memory=True)
    hd = torch.empty((1, k), dtype=torch.float32, pin_memory=True)
    lat = {"psb": lat_us(lambda x: psb.psb_knn_ex(idx, x, k, algo=0, out=(hi, hd)), hq),
           "psb_split": lat_us(lambda x: psb.psb_knn_split(idx, x, k, parts=0, out=(hi, hd)), hq),
           "bnb": lat_us(lambda x: psb.psb_knn_ex(idx, x, k, algo=1, out=(hi, hd)), hq),
           "brute": lat_us(lambda x: psb.psb_knn_ex(idx, x, k, algo=2, out=(hi, hd)), hq, n=20)}
    print(json.dumps({"sigma": sigma, "batch_ms": ms, "queries_per_s": {a: cfg.q / (v / 1e3) for a, v in ms.items()},
                      "latency_p50_us": lat, "leaves_per_query": leaves, "kth_dist_median":
                      float(res["psb"][1][:, -1].median()), "routes_equal": same, "oracle_16_equal": ok}), flush=True)
    idx.free()
