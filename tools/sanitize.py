"""Small runs of every kernel family for compute-sanitizer (memcheck, racecheck,
synccheck, initcheck): C1-shaped and C2/C3-sampled inputs (the C3 sample runs the
d = 8 kernels with the eligibility reuse), all algorithms, latency mode and batch
split, stats and trace, merge, export/import, the L2 probe and the GPU bulk loader."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_namkn16_b200 as psb
import workloads as W

for name, n, q in (("C1", None, 100), ("C2", 100_000, 64), ("C3", 100_000, 64)):
    cfg = W.config(name)
    pts = cfg.points(n=n)
    qd = torch.from_numpy(cfg.queries(q=q)).cuda()
    idx = psb.psb_build(pts, cfg.fanout)
    for algo in (0, 1, 2):
        psb.psb_knn_ex(idx, qd, cfg.k, algo=algo)
    for var in (psb.PSB_VAR_KTH_MAXDIST, psb.PSB_VAR_P1_INDEX_TIE, psb.PSB_VAR_PREFETCH_NEXT | psb.PSB_VAR_PREFETCH_IDS,
                psb.PSB_VAR_LEAF_ORDER, psb.PSB_VAR_NOCACHE):
        psb.psb_knn_ex(idx, qd, cfg.k, variant=var)
    # pinned host outputs: rows stored by the kernels straight into host memory
    hi = torch.empty((q, cfg.k), dtype=torch.int32, pin_memory=True)
    hd = torch.empty((q, cfg.k), dtype=torch.float32, pin_memory=True)
    for algo in (0, 1, 2):
        psb.psb_knn_ex(idx, qd.cpu().pin_memory(), cfg.k, algo=algo, out=(hi, hd))
    psb.psb_knn_stats(idx, qd, cfg.k, algo=0)
    psb.psb_knn_trace(idx, qd, cfg.k, cap=512)
    psb.psb_knn_split(idx, qd[:4], cfg.k, parts=16)
    # batch split over interleaved level-1 nodes (tasks fill the GPU)
    qb = torch.from_numpy(cfg.queries(q=1500)).cuda()
    psb.psb_knn_split(idx, qb, cfg.k, parts=4)
    # export / import round trip
    psb.psb_index_import(psb.psb_index_export_raw(idx)).free()
    ids, d = psb.psb_knn(idx, qd, cfg.k)
    psb.psb_merge_topk(torch.stack([ids, ids]), torch.stack([d, d]), cfg.k)
    torch.cuda.synchronize()
    idx.free()
psb.psb_probe_l2_read(2 << 20, 2, 1)
print("sanitize workload done")
