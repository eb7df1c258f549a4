"""Per-CUDA-line instruction / stall shares of one kernel from an `ncu --page source
--print-source cuda,sass --csv` dump, plus the main raw metrics (profiling aid).
usage: python tools/ncu_lines.py CS_CSV [REP] [N]"""
import csv, subprocess, sys
rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if r and r[0] == "Line No"][0]
h = rows[hi]
ie, iss = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
L = {}
for r in rows[hi + 1:]:
    if r and r[0] != "" and len(r) > max(ie, iss):
        try:
            L[int(r[0])] = (float(r[ie] or 0), float(r[iss] or 0), r[1].strip())
        except ValueError:
            pass
tot = sum(v[0] for v in L.values()); ts = sum(v[1] for v in L.values()) or 1
print("total warp instructions %.3e, stall samples %.0f" % (tot, ts))
n = int(sys.argv[3]) if len(sys.argv) > 3 else 40
for k, v in sorted(L.items(), key=lambda kv: -kv[1][0])[:n]:
    print("%5d %6.2f%% inst %6.2f%% stall  %s" % (k, 100 * v[0] / tot, 100 * v[1] / ts, v[2][:95]))
if len(sys.argv) > 2:
    out = subprocess.run(["ncu", "-i", sys.argv[2], "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(out.splitlines()))
    hdr, val = rr[0], rr[2]
    for m in ["gpu__time_duration.sum", "smsp__inst_executed.sum", "sm__inst_executed.avg.per_cycle_active",
              "sm__warps_active.avg.pct_of_peak_sustained_active", "dram__bytes_read.sum", "dram__bytes_write.sum",
              "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "launch__registers_per_thread",
              "launch__occupancy_limit_shared_mem", "sm__warps_active.avg.per_cycle_active"]:
        if m in hdr:
            print(m, val[hdr.index(m)], rr[1][hdr.index(m)])
    st = [(c, val[i]) for i, c in enumerate(hdr) if c.startswith("smsp__average_warps_issue_stalled_") and c.endswith("_per_issue_active.ratio")]
    st = sorted(((float(v or 0), c[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]) for c, v in st), reverse=True)[:8]
    print("stalls per issue:", ", ".join("%s %.2f" % (c, v) for v, c in st))
