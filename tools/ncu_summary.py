#!/usr/bin/env python3
"""Summarise ncu reports into profiles/: key metrics per kernel launch, plus
profiles/traffic.json (dram read+write bytes per launch, read by bench.py).

    python tools/ncu_summary.py --round r01 --tag C2/psb gpurun_out/prof_psb_c2.ncu-rep [...]
Each report is tagged `<config>/<algo>`, e.g. C2/psb.
"""
import argparse
import csv
import io
import json
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

WANT = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "lts__t_bytes.sum": "l2_bytes",
    "lts__t_sector_hit_rate.pct": "l2_hit_pct",
    "l1tex__t_bytes.sum": "l1_bytes",
    "smsp__thread_inst_executed_per_inst_executed.ratio": "threads_per_inst",
    "smsp__sass_branch_targets_threads_divergent.sum": "branch_divergent",
    "smsp__inst_executed_op_branch.sum": "branch_inst",
    "smsp__thread_inst_executed_pred_on_per_inst_executed.ratio": "threads_pred_on_per_inst",
    "lts__t_sectors.sum": "l2_sectors",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "achieved_occupancy_pct",
    "sm__warps_active.avg.per_cycle_active": "warps_per_sm",
    "launch__registers_per_thread": "registers",
    "launch__occupancy_limit_registers": "block_limit_regs",
    "smsp__inst_executed.sum": "warp_inst",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_throughput_pct",
    "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed": "mem_throughput_pct",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_throughput_pct",
    "sm__instruction_throughput.avg.pct_of_peak_sustained_active": "issue_pct",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
}
STALLS = "smsp__average_warps_issue_stalled_"


def to_bytes(v, unit):
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    return float(v) * mult.get(unit, 1)


def to_us(v, unit):
    return float(v) * {"ns": 1e-3, "us": 1, "usecond": 1, "ms": 1e3, "msecond": 1e3, "s": 1e6}.get(unit, 1)


def read(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    launches = []
    for r in rows[2:]:
        d = {}
        stalls = {}
        for h, u, v in zip(hdr, units, r):
            if h == "Kernel Name":
                d["kernel"] = v
            if h in WANT:
                k = WANT[h]
                try:
                    if "bytes" in h and "pct" not in h:
                        d[k] = to_bytes(v.replace(",", ""), u)
                    elif h == "gpu__time_duration.sum":
                        d[k] = to_us(v.replace(",", ""), u)
                    else:
                        d[k] = float(v.replace(",", ""))
                except ValueError:
                    d[k] = v
            if h.startswith(STALLS) and h.endswith("_per_issue_active.ratio"):
                try:
                    stalls[h[len(STALLS):-len("_per_issue_active.ratio")]] = float(v)
                except ValueError:
                    pass
        d["top_stalls"] = dict(sorted(stalls.items(), key=lambda t: -t[1])[:6])
        if "threads_per_inst" in d:
            d["warp_exec_efficiency_pct"] = 100.0 * d["threads_per_inst"] / 32.0
        if d.get("branch_inst"):
            d["branch_divergence_pct"] = 100.0 * d.get("branch_divergent", 0) / d["branch_inst"]
        if "l2_sectors" in d:
            d["l2_bytes"] = 32.0 * d["l2_sectors"]
        launches.append(d)
    return launches


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--round", required=True)
    ap.add_argument("--tag", action="append", required=True)
    ap.add_argument("reports", nargs="+")
    a = ap.parse_args()
    assert len(a.tag) == len(a.reports)
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    traffic = json.load(open(tpath)) if os.path.exists(tpath) else {}
    md = [f"# ncu --set full summaries ({a.round})", "",
          "One launch per report (`--clock-control none`, ncu's default cache flush before the",
          "launch: DRAM bytes are cold-cache). Warp execution efficiency = threads per executed",
          "instruction / 32; branch divergence = divergent branch targets / branch targets.", ""]
    summary = {}
    for tag, rep in zip(a.tag, a.reports):
        ls = read(rep)
        for d in ls:
            summary.setdefault(tag, []).append(d)
            md.append(f"## {tag}: `{d.get('kernel', '?')[:110]}`")
            md.append("")
            md.append("| metric | value |")
            md.append("|---|---|")
            for k in ("duration", "dram_read", "dram_write", "l2_bytes", "l2_hit_pct", "l1_bytes",
                      "warp_exec_efficiency_pct", "threads_pred_on_per_inst", "branch_inst", "branch_divergent",
                      "branch_divergence_pct", "achieved_occupancy_pct",
                      "warps_per_sm", "registers", "block_limit_regs", "warp_inst", "issue_active_pct",
                      "sm_throughput_pct", "mem_throughput_pct", "dram_throughput_pct", "grid", "block"):
                if k in d:
                    v = d[k]
                    md.append(f"| {k} | {v:,.3f} |" if isinstance(v, float) else f"| {k} | {v} |")
            md.append(f"| top stalls (warps per issue) | {json.dumps({k: round(v, 3) for k, v in d['top_stalls'].items()})} |")
            md.append("")
        d0 = ls[0]
        traffic[tag] = {"dram_bytes_per_launch": d0.get("dram_read", 0) + d0.get("dram_write", 0),
                        "l2_bytes_per_launch": d0.get("l2_bytes"),
                        "warp_inst_per_launch": d0.get("warp_inst"),
                        "issue_active_pct": d0.get("issue_active_pct"),
                        "source": f"profiles/{a.round}_ncu.md ({os.path.basename(rep)})",
                        "note": "ncu flushes caches before the replayed launch (cold)"}
    open(os.path.join(ROOT, "profiles", f"{a.round}_ncu.md"), "w").write("\n".join(md) + "\n")
    json.dump(summary, open(os.path.join(ROOT, "profiles", f"{a.round}_ncu.json"), "w"), indent=1)
    json.dump(traffic, open(tpath, "w"), indent=1)
    print("\n".join(md))


if __name__ == "__main__":
    main()
