#!/usr/bin/env python3
"""bench.py — PSB exact kNN throughput on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--mode query|data]
                    [--algo psb|bnb|brute] [--impl ours|reference] [--weak] [--chunks C]

A step is one pass of the whole hot path (one psb_knn
launch) over one batch of synthetic queries of the named config, inputs resident
in HBM. N=1 default workload: BASELINE.json configs[2] (C3: 8-D uniform n=4M,
fanout 128, 100,000 queries, k=16), the config the metric's "1/2/4/8 B200" is
quoted on. Multi-GPU (torchrun, one rank per GPU):
  --mode query (default): replicated index, the fixed batch of q queries is
      split into N contiguous slices, one per rank, no collective (strong
      scaling; --weak: every rank answers its own q queries instead);
  --mode data: each rank holds a sub-tree over a slab of the points, every rank
      answers the same q queries, and the per-shard lists are merged from peer
      memory (psb_exchange, chunked so the exchange overlaps the search) or by
      NCCL all-gather + on-device merge (--exchange nccl).
L2 is flushed (256 MiB write) between timed steps; each step is timed with CUDA
events on the launching stream; the reported time is the max over ranks.
Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import workloads as W  # noqa: E402

METRIC = "kNN queries/s (PSB exact kNN, batch throughput)"
UNIT = "queries/s"
FALLBACK_HBM_GBS = 6650.0


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--config", default="C3", choices=sorted(W.CONFIGS))
    ap.add_argument("--queries", type=int, default=0, help="override q per step (0 = config's)")
    ap.add_argument("--mode", default="query", choices=["query", "data"])
    ap.add_argument("--weak", action="store_true",
                    help="query mode, N>1: every rank answers its own q queries (weak scaling)")
    ap.add_argument("--chunks", type=int, default=4,
                    help="data mode, N>1, p2p exchange: query chunks (merge of chunk c overlaps search of c+1)")
    ap.add_argument("--latency-queries", type=int, default=1000,
                    help="single-query latency sample (SURVEY §8(d): 1,000 distinct queries)")
    ap.add_argument("--slab", type=int, default=0,
                    help="data mode on ONE GPU: run rank 0's local step of a P-way data-sharded job")
    ap.add_argument("--exchange", default="p2p", choices=["p2p", "nccl"],
                    help="data mode, N>1: merge straight from peer memory (psb_exchange) or NCCL all-gather + merge")
    ap.add_argument("--algo", default="psb", choices=["psb", "psb_split", "bnb", "brute"],
                    help="psb_split: psb_knn_split with the library's automatic part count")
    ap.add_argument("--variant", type=int, default=0)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-extras", action="store_true", help="skip latency/e2e/comparator legs")
    ap.add_argument("--profile", action="store_true", help="short run for ncu (no extras)")
    return ap.parse_args()


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks/throttle sampling DURING the timed region (B200_PROFILING.md)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,utilization.gpu,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index: int):
        self.dev = device_index
        self.rows = []
        self.proc = None
        self.t = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.dev}", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "50"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
            return
        self.t = threading.Thread(target=self._read, daemon=True)
        self.t.start()

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([c.strip() for c in line.split(",")])

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.12)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        rows = [r for r in self.rows if len(r) >= 9]
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        busy = [float(r[1]) for r in rows if r[4].isdigit() and int(r[4]) > 0] or sm
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(busy) if busy else None,
                "sm_max_mhz": float(rows[0][2]) if rows[0][2].replace(".", "").isdigit() else None,
                "reasons": reasons, "samples": len(rows), "samples_busy": len(busy)}


# ----------------------------------------------------------------------------- helpers
def peaks() -> tuple[float, str]:
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        return float(json.load(open(p))["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


def traffic_from_profiles(config: str, algo: str, key: str = "dram_bytes_per_launch"):
    """Per-launch figures (dram read+write bytes, L2 bytes, warp instructions) of
    the kernel from the committed ncu --set full summary (profiles/traffic.json)."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        return json.load(open(p))[f"{config}/{algo}"].get(key)
    except Exception:
        return None


def issue_peak() -> float:
    """Warp-instruction issue ceiling, G warp-inst/s: 148 SMs x 4 schedulers x 1 issue
    per cycle at the max SM clock (B200_PROFILING.md; MEASURED_PEAKS.json sm_max_mhz)."""
    try:
        mhz = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["sm_max_mhz"])
    except Exception:
        mhz = 1965.0
    return 148 * 4 * mhz / 1e3


def alu_peak() -> float:
    """FP32 arithmetic ceiling, T ops/s (an add, a subtract or a multiply each one
    op): 148 SMs x 128 FP32 lanes x the max SM clock (MEASURED_PEAKS.json
    sm_max_mhz) = 148 x 4 SMSPs x one packed pair instruction (64 ops) per 2
    cycles; DESIGN.md §6 derives it."""
    return issue_peak() * 32 / 1e3


def cpu_baseline(cfg, pts, qs, k, gpu_ids=None, gpu_d=None) -> dict:
    """The oracle as it stands, on this host's cores (bounded sample)."""
    import oracle
    threads = os.cpu_count() or 1
    t0 = time.perf_counter()
    tree = oracle.Tree(pts)
    t_build = time.perf_counter() - t0
    reps = []
    res = None
    for _ in range(3):
        t0 = time.perf_counter()
        res = tree.knn(qs, k, threads=threads)
        reps.append(time.perf_counter() - t0)
    bnb_qps = len(qs) / statistics.median(reps)
    # one thread on a bounded sample (a single-thread number too)
    n1 = min(len(qs), 2000)
    t0 = time.perf_counter()
    tree.knn(qs[:n1], k, threads=1)
    single_qps = n1 / (time.perf_counter() - t0)
    nb = min(len(qs), 1000 if cfg.n <= 2_000_000 else 100)
    t0 = time.perf_counter()
    bf = oracle.knn_bruteforce(pts, qs[:nb], k, threads=threads)
    bf_qps = nb / (time.perf_counter() - t0)
    out = {"value": bnb_qps, "unit": UNIT, "cores": threads, "kind": "oracle",
           "sample": f"all {len(qs)} queries of {cfg.name} via the oracle's recursive B&B (median of 3; "
                     f"tree build {t_build:.2f}s excluded); single thread on the first {n1}; "
                     f"brute-force route on {nb} queries",
           "single_thread_value": single_qps,
           "bruteforce_value": bf_qps,
           "oracle_routes_agree": bool(np.array_equal(bf[0], res[0][:nb]))}
    if gpu_ids is not None:
        out["agrees_with_gpu"] = bool(np.array_equal(gpu_ids, res[0]) and
                                      np.array_equal(gpu_d.view(np.uint32), res[1].view(np.uint32)))
    return out


# ----------------------------------------------------------------------------- reference arm
def run_reference(args, rank, world):
    """--impl reference: the CPU oracle on the host cores (the tier's reference arm),
    on this arm's config, metric and unit. Each step is a bounded sample of the
    workload's query batch (sized from a calibration run so the whole
    --steps/--warmup run takes about a minute); rank 0 alone runs it."""
    if rank != 0:
        return
    import oracle
    cfg = W.config(args.config)
    q = args.queries or cfg.q
    pts = cfg.points()
    qs = cfg.queries(q)
    tree = oracle.Tree(pts)
    threads = os.cpu_count() or 1
    t0 = time.perf_counter()
    tree.knn(qs[: min(q, 1000)], cfg.k, threads=threads)                 # calibration (+ warm-up)
    per_q = (time.perf_counter() - t0) / min(q, 1000)
    budget_s = 60.0 / max(1, args.steps + args.warmup)
    sample = int(max(256, min(q, budget_s / max(per_q, 1e-9))))
    for i in range(max(0, args.warmup)):
        o = (i * sample) % q
        tree.knn(qs[o:o + sample], cfg.k, threads=threads)
    times = []
    done = 0
    for i in range(args.steps):
        o = (i * sample) % q
        batch = qs[o:o + sample]
        t0 = time.perf_counter()
        tree.knn(batch, cfg.k, threads=threads)
        times.append(time.perf_counter() - t0)
        done += len(batch)
    total = sum(times)
    val = done / total
    desc = (f"each step: {sample} consecutive queries of the {q}-query {cfg.name} batch (bounded sample) via the "
            f"oracle's recursive B&B on {threads} host threads")
    line = {"metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * total / args.steps, "higher_is_better": True,
            "scaling": "weak" if args.weak else "strong", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic (workloads/, seeded)", "impl": "reference",
            "config": {**cfg.describe(), "q": q, "parallelism": "host threads (rank 0 only)"},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": desc},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- our arm
def issue_roof(config, algo, kern_s):
    """Instruction issue: ncu's warp-instruction count per launch (same kernel,
    committed profiles/traffic.json) over the live mean launch time, against the
    issue ceiling."""
    inst = traffic_from_profiles(config, algo, "warp_inst_per_launch")
    if not inst:
        return None
    a = inst / kern_s / 1e9
    return {"achieved": a, "peak": issue_peak(), "unit": "G warp-inst/s", "frac": a / issue_peak(),
            "warp_inst_per_launch": inst, "source": "profiles/traffic.json (ncu smsp__inst_executed.sum)"}


def roofline(algo, idx, q, k, alg_bytes, kern_s, prof_cfg, l2_peak):
    """The dominant kernel against the ceilings that can bind it.

    Tree traversals: their algorithmic bytes (every node and leaf block each
    query touches, counted per query) are served from L1/L2, not DRAM, at every
    config but the cold first touch, so the primary roofline is those bytes over
    the launch time against the L2 read bandwidth MEASURED in this run
    (psb_probe_l2_read). Next to it: DRAM bytes (ncu dram__bytes, committed
    profiles/traffic.json) against the measured HBM peak, ncu's L2 bytes against
    the same L2 peak, and warp instructions against the issue ceiling. Brute
    force: bound by FP32 arithmetic, 1.5 lane-instructions per point-dimension
    (packed subtract / square / add pairs) against the lane-instruction ceiling."""
    hbm, hbm_src = peaks()
    if algo == "brute":
        ops = 3.0 * idx.n * q * idx.d
        a = ops / kern_s / 1e12
        prim = {"bound": "alu", "achieved": a, "peak": alu_peak(), "unit": "T FP32-op/s", "frac": a / alu_peak(),
                "algorithmic_fp32_ops_per_launch": ops,
                "peak_source": "148 SMs x 128 FP32 lanes x sm_max_mhz: packed FADD2/FFMA2 pairs issue at one "
                               "per 2 cycles per SMSP (ncu: fma pipe busy 2 cycles per packed instruction; "
                               "DESIGN.md §6)"}
    elif alg_bytes is None:                   # split mode: ncu's L2 bytes of the split kernel
        l2b = traffic_from_profiles(prof_cfg, algo, "l2_bytes_per_launch") or 0.0
        a = l2b / kern_s / 1e9
        prim = {"bound": "l2", "achieved": a, "peak": l2_peak, "unit": "GB/s", "frac": a / l2_peak,
                "l2_bytes_per_launch": l2b, "note": "split mode has no per-part traversal counters: "
                "achieved = ncu lts bytes of psb_split_kernel (profiles/traffic.json) / live launch time",
                "peak_source": "measured in this run: psb_probe_l2_read (64 MiB L2-resident; best of 16-B x1, 16-B x4, 32-B x1, 32-B x2 ld.global.cg loads per thread)"}
    else:
        a = alg_bytes / kern_s / 1e9
        prim = {"bound": "l2", "achieved": a, "peak": l2_peak, "unit": "GB/s", "frac": a / l2_peak,
                "algorithmic_bytes_per_launch": alg_bytes,
                "peak_source": "measured in this run: psb_probe_l2_read (64 MiB L2-resident; best of 16-B x1, 16-B x4, 32-B x1, 32-B x2 ld.global.cg loads per thread)"}
    dram = traffic_from_profiles(prof_cfg, algo, "dram_bytes_per_launch")
    prim["traffic"] = dram
    prim["avg_launch_ms"] = kern_s * 1e3
    levels = {}
    if dram:
        levels["hbm"] = {"achieved": dram / kern_s / 1e9, "peak": hbm, "unit": "GB/s",
                         "frac": dram / kern_s / 1e9 / hbm, "dram_bytes_per_launch": dram,
                         "peak_source": hbm_src, "source": "profiles/traffic.json (ncu dram__bytes read+write)"}
    l2b = traffic_from_profiles(prof_cfg, algo, "l2_bytes_per_launch")
    if l2b:
        levels["l2_ncu"] = {"achieved": l2b / kern_s / 1e9, "peak": l2_peak, "unit": "GB/s",
                            "frac": l2b / kern_s / 1e9 / l2_peak, "l2_bytes_per_launch": l2b,
                            "source": "profiles/traffic.json (ncu lts__t_bytes)"}
    iss = issue_roof(prof_cfg, algo, kern_s)
    if iss:
        levels["issue"] = iss
    prim.update(levels)
    cands = {prim["bound"]: prim["frac"], **{n: v["frac"] for n, v in levels.items()}}
    prim["binding"] = max(cands, key=cands.get)
    return prim


def count_launches(step):
    """Kernels one step launches, counted by the CUDA profiler (CUPTI via
    torch.profiler) on an untimed extra step: {name: count} and the total."""
    import torch
    from torch.profiler import ProfilerActivity, profile
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        step()
        torch.cuda.synchronize()
    names = {}
    for ev in prof.events():
        if ev.device_type == torch.autograd.DeviceType.CUDA and not ev.name.startswith(("Memcpy", "Memset")):
            short = ev.name.split("(")[0].replace("void ", "")
            names[short] = names.get(short, 0) + 1
    return sum(names.values()), names


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world)

    import torch
    import torch.distributed as dist
    import paper_conf_icpp_namkn16_b200 as psb
    from paper_conf_icpp_namkn16_b200 import dist as pdist

    # PSB_BENCH_DEVICE / PSB_DIST_BACKEND: test hooks (several ranks on one GPU over gloo)
    torch.cuda.set_device(int(os.environ.get("PSB_BENCH_DEVICE", local)))
    backend = os.environ.get("PSB_DIST_BACKEND", "nccl")
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", torch.cuda.current_device()))
        else:
            dist.init_process_group(backend)
    red_dev = "cuda" if backend == "nccl" else "cpu"
    if args.profile:
        args.no_extras = True
        args.no_cpu_baseline = True

    cfg = W.config(args.config)
    q = args.queries or cfg.q
    k = cfg.k
    algo = {"psb": psb.PSB_ALGO_PSB, "psb_split": psb.PSB_ALGO_PSB, "bnb": psb.PSB_ALGO_BNB,
            "brute": psb.PSB_ALGO_BRUTE}[args.algo]
    weak = args.mode == "query" and args.weak
    if args.mode == "query":
        # replicated index; strong scaling: rank r answers slice r of the fixed
        # batch of q queries (weak: its own batch of q)
        pts = cfg.points()
        if weak:
            qs = cfg.queries(q * world)[rank * q:(rank + 1) * q]
        else:
            qs = cfg.queries(q)[pdist.query_slice(q, world, rank)]
        idx = psb.psb_build(pts, cfg.fanout)
    else:
        # rank r holds slab r of the points (global ids via id_base); all ranks see all q queries
        parts = max(world, args.slab or 1)
        b = pdist.shard_bounds(cfg.n, parts)
        pts = cfg.points(n=b[rank + 1] - b[rank], row0=b[rank])
        qs = cfg.queries(q)
        idx = psb.psb_build_ex(pts, cfg.fanout, id_base=b[rank])
    ql = len(qs)                                   # queries this rank searches per step
    stream = torch.cuda.current_stream()
    qd = torch.from_numpy(qs).cuda()
    out_i = torch.empty((ql, k), dtype=torch.int32, device="cuda")
    out_d = torch.empty((ql, k), dtype=torch.float32, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")

    # algorithmic bytes of one launch (deterministic traversal counters)
    if algo == psb.PSB_ALGO_BRUTE:
        alg_bytes = idx.leaves * idx.fanout * (idx.d * 4) * ql + ql * (4 * idx.d + 8 * k)
        stats_sum = None
        in_batch = None
    elif args.algo == "psb_split":            # no per-part counters: the roofline uses ncu's L2 bytes
        alg_bytes = None
        stats_sum = None
        in_batch = None
    else:
        _, _, st = psb.psb_knn_stats(idx, qd, k, algo=algo, variant=args.variant, out=(out_i, out_d))
        stn = st.cpu().numpy()
        stats_sum = stn[:, :6].sum(0).tolist()
        alg_bytes = psb.algorithmic_bytes(idx, stats_sum, ql, k)
        # in-batch service time per query (%globaltimer stamps of the counting launch,
        # SURVEY §8(d) latency (b)); the counting kernel is the runtime-d instantiation
        svc = np.sort((stn[:, 7] - stn[:, 6]) / 1e3)
        span = (stn[:, 7].max() - stn[:, 6].min()) / 1e3
        last_start = (stn[:, 6].max() - stn[:, 6].min()) / 1e3
        in_batch = {"p50": float(svc[len(svc) // 2]), "p99": float(svc[min(len(svc) - 1, int(len(svc) * 0.99))]),
                    "max": float(svc[-1]), "batch_span_us": float(span), "last_query_start_us": float(last_start),
                    "definition": "per-query service time inside one batch launch (%globaltimer when the warp "
                                  "took / finished the query), counting-kernel instantiation"}

    def local_knn(qq, kk):
        o = (out_i, out_d) if qq.shape[0] == ql else None
        if args.algo == "psb_split":
            return psb.psb_knn_split(idx, qq, kk, parts=0, out=o)
        return psb.psb_knn_ex(idx, qq, kk, algo=algo, variant=args.variant, out=o)

    ex = None
    chunks = max(1, args.chunks)
    if args.mode == "data" and world > 1 and args.exchange == "p2p":
        ex = pdist.peer_exchange(q, k)
        rows = sum(r.stop - r.start for r in pdist.chunk_rows(q, world, rank, chunks))
        merged = (torch.empty((rows, k), dtype=torch.int32, device="cuda"),
                  torch.empty((rows, k), dtype=torch.float32, device="cuda"))

    def step():
        if args.mode == "query" or world == 1:
            local_knn(qd, k)
        elif ex is not None:
            pdist.data_sharded_knn_p2p(ex, idx, qd, algo=algo, variant=args.variant, chunks=chunks, out=merged)
        else:
            pdist.data_sharded_knn(local_knn, pdist.device_merge, qd, k)

    for _ in range(max(3, args.warmup)):
        step()
    torch.cuda.synchronize()
    launches_per_step, launch_names = count_launches(step)

    sampler = ClockSampler(local)
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler.start()
    time.sleep(0.15)
    for i in range(args.steps):
        flush.fill_(i & 0xFF)                      # evict the index from L2 between steps
        evs[i][0].record(stream)
        step()
        evs[i][1].record(stream)
    torch.cuda.synchronize()
    clocks = sampler.stop()
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in evs]
    total_ms = torch.tensor([sum(step_ms)], dtype=torch.float64, device=red_dev)
    if world > 1:
        dist.all_reduce(total_ms, op=dist.ReduceOp.MAX)
    total_ms = float(total_ms.item())
    units = q * world if weak else q
    value = units * args.steps / (total_ms / 1e3)
    ms_per_step = total_ms / args.steps
    kern_s = statistics.mean(step_ms) / 1e3
    l2_peak = psb.psb_probe_l2_read()             # GB/s, this GPU, this run
    # profiles/traffic.json key: the one-GPU slab of a data-sharded run is profiled
    # as its own workload (tools/prof_one.py C5 = slab 0 of 8 -> "C5slab")
    prof_cfg = args.config + ("slab" if args.mode == "data" and world == 1 and (args.slab or 1) == 8 else "")
    roof = roofline(args.algo, idx, ql, k, alg_bytes, kern_s, prof_cfg, l2_peak)
    roof["kernel"] = {"psb": "psb_kernel", "psb_split": "psb_split_kernel", "bnb": "bnb_kernel",
                      "brute": "brute_smem_kernel"}[args.algo]
    if stats_sum is not None:
        roof["counters_per_query"] = {"node_fetches": stats_sum[0] / ql, "leaf_scans": stats_sum[1] / ql,
                                      "id_loads": stats_sum[2] / ql, "cache_hits": stats_sum[3] / ql,
                                      "changing_leaf_scans": stats_sum[4] / ql, "keys_merged": stats_sum[5] / ql}

    extras = {}
    if not args.no_extras:
        # e2e through the public API with HOST (pinned) buffers: H2D + kernel + D2H each step
        hq = torch.from_numpy(qs).pin_memory()

        def local_e2e(x, oi, od):
            if args.algo == "psb_split":
                return psb.psb_knn_split(idx, x, k, parts=0, out=(oi, od))
            return psb.psb_knn_ex(idx, x, k, algo=algo, variant=args.variant, out=(oi, od))

        hi = torch.empty((ql, k), dtype=torch.int32, pin_memory=True)
        hd = torch.empty((ql, k), dtype=torch.float32, pin_memory=True)
        e2e_ms = []
        for i in range(max(3, args.warmup) + args.steps):
            flush.fill_(i & 0xFF)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            local_e2e(hq, hi, hd)
            stream.synchronize()
            if i >= max(3, args.warmup):
                e2e_ms.append((time.perf_counter() - t0) * 1e3)
        e2e_t = torch.tensor([sum(e2e_ms)], dtype=torch.float64, device=red_dev)
        if world > 1:
            dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
        extras["e2e"] = {"value": units * args.steps / (float(e2e_t.item()) / 1e3), "unit": UNIT,
                         "h2d_bytes_per_step": int(ql * idx.d * 4), "d2h_bytes_per_step": int(ql * k * 8),
                         "api": "psb_knn_ex with pinned host buffers (batches of <= 16,384 queries: the kernels read "
                                "the queries in place over the host link; larger batches: one H2D copy on the stream; "
                                "the kernel writes each result row straight into the pinned host output)"}
        if args.mode == "data" and world > 1:
            extras["e2e"]["note"] = "local search only (the data-sharded exchange runs on device buffers)"
        # single-query latency: launch -> results on the host,
        # for PSB (one warp), PSB latency mode (query split over many warps), B&B, brute force
        h1i = torch.empty((1, k), dtype=torch.int32, pin_memory=True)
        h1d = torch.empty((1, k), dtype=torch.float32, pin_memory=True)
        nl = min(ql, args.latency_queries)

        def lat_of(call, n_lat):
            lat = []
            for i in range(n_lat + 5):
                h1q = hq[i % ql:i % ql + 1]
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                call(h1q)
                stream.synchronize()
                if i >= 5:
                    lat.append((time.perf_counter() - t0) * 1e6)
            lat.sort()
            return {"p50": lat[len(lat) // 2], "p99": lat[min(len(lat) - 1, int(len(lat) * 0.99))],
                    "queries": n_lat}

        lats = {
            args.algo: lat_of(lambda x: local_e2e(x, h1i, h1d), nl),
            "psb_split": lat_of(lambda x: psb.psb_knn_split(idx, x, k, parts=0, out=(h1i, h1d)), nl),
            "bnb": lat_of(lambda x: psb.psb_knn_ex(idx, x, k, algo=psb.PSB_ALGO_BNB, out=(h1i, h1d)), nl),
            "brute": lat_of(lambda x: psb.psb_knn_ex(idx, x, k, algo=psb.PSB_ALGO_BRUTE, out=(h1i, h1d)),
                            min(nl, 50)),
        }
        extras["latency_us"] = {**lats[args.algo], "by_algo": lats, "in_batch": in_batch,
                                "definition": "one query per call, launch to results in pinned host memory "
                                              "(PAPER.md L835-838 'query response time')"}
        # comparators on the same batch (same timing protocol, fewer steps)
        comp = {}
        for name, a in (("psb", psb.PSB_ALGO_PSB), ("psb_split", -1), ("bnb", psb.PSB_ALGO_BNB),
                        ("brute", psb.PSB_ALGO_BRUTE)):
            if name == "brute" and idx.n * ql > 2e11:
                comp[name] = {"skipped": f"n*q = {idx.n * ql:.2e} pairs (minutes per batch)"}
                continue
            reps = 20 if name != "brute" else 3
            reps = reps if ql * idx.n < 1e12 else 3
            ts = []
            for i in range(reps + 2):
                flush.fill_(i & 0xFF)
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s.record(stream)
                if a < 0:                              # psb_knn_split, auto parts (tail splitting)
                    psb.psb_knn_split(idx, qd, k, parts=0, out=(out_i, out_d))
                else:
                    psb.psb_knn_ex(idx, qd, k, algo=a, out=(out_i, out_d))
                e.record(stream)
                torch.cuda.synchronize()
                if i >= 2:
                    ts.append(s.elapsed_time(e))
            comp[name] = {"queries_per_s": ql / (statistics.median(ts) / 1e3), "ms": statistics.median(ts)}
        extras["comparators_1gpu"] = comp

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline and (args.mode == "query" or (args.slab or 1) == 1):
        psb.psb_knn_ex(idx, qd, k, algo=algo, variant=args.variant, out=(out_i, out_d))
        torch.cuda.synchronize()
        cpu = cpu_baseline(cfg, pts, qs, k, out_i.cpu().numpy(), out_d.cpu().numpy())

    if rank == 0:
        if args.mode == "query":
            par = (f"query-sharded x{world} (replicated index; " +
                   (f"each rank its own {q} queries, weak)" if weak else f"the {q}-query batch split {world} ways)"))
        elif world > 1:
            par = (f"data-sharded x{world} (merge from peer memory, psb_exchange, {chunks} chunks)" if ex is not None
                   else f"data-sharded x{world} (NCCL all-gather + merge)")
        else:
            par = f"data-sharded slab 0 of {max(1, args.slab)} (local step only, 1 GPU)"
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": max(3, args.warmup), "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "weak" if weak else "strong", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic (workloads/: seeded SplitMix64 uniform / 100-cluster Gaussian)",
            "config": {**cfg.describe(), "q": q, "q_per_rank": ql, "algo": args.algo,
                       "variant": args.variant, "parallelism": par,
                       "points_on_this_gpu": int(pts.shape[0]),
                       "l2": "flushed between steps (256 MiB write)", "index_bytes": idx.device_bytes},
            "roofline": roof,
            "clocks": clocks,
            "gpu_launches": args.steps * launches_per_step,
            "gpu_launch_names": launch_names,
            **extras,
        }
        if cpu is not None:
            line["cpu_baseline"] = cpu
        print(json.dumps(line), flush=True)
    if ex is not None:
        if ex.timed_out():
            raise RuntimeError("psb_exchange: a peer wait timed out")
        dist.barrier()
        ex.free()
    idx.free()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
