"""Print duration, issue activity, occupancy, instruction count and the warp-stall
breakdown (warps per issue) of each ncu report. Dev aid.  usage: ncu_stalls.py REP..."""
import csv, io, subprocess, sys
for rep in sys.argv[1:]:
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out))); h, v = r[0], r[2]
    g = lambda n: v[h.index(n)] if n in h else "?"
    print(f"== {rep.split('/')[-1]}: {g('gpu__time_duration.sum')} ns  inst {g('smsp__inst_executed.sum')}  "
          f"issue {g('smsp__issue_active.avg.pct_of_peak_sustained_active')}%  warps/sm {g('sm__warps_active.avg.per_cycle_active')}  "
          f"L2 hit {g('lts__t_sector_hit_rate.pct')}%  dram {g('dram__bytes_read.sum')}  regs {g('launch__registers_per_thread')}")
    st = []
    for i, n in enumerate(h):
        if n.startswith("smsp__average_warps_issue_stalled_") and n.endswith("_per_issue_active.ratio"):
            try: st.append((float(v[i].replace(",", "")), n[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
            except ValueError: pass
    print("   " + "  ".join(f"{n} {x:.2f}" for x, n in sorted(st, reverse=True)[:9]))
