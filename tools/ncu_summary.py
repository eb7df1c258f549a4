#!/usr/bin/env python
"""Summarise an ncu capture (--set full .ncu-rep) and a launch list (--metrics
gpu__time_duration.sum CSV) into profiles/ (JSON + Markdown).  Profiling aid."""
import csv
import io
import json
import subprocess
import sys
from collections import defaultdict

METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
           "smsp__inst_executed.sum", "sm__inst_executed.avg.per_cycle_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
           "launch__registers_per_thread", "lts__t_sector_hit_rate.pct", "lts__t_sectors_srcunit_tex_op_write.sum",
           "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
           "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
           "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
           "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
           "smsp__sass_thread_inst_executed_op_dfma_pred_on.sum",
           "smsp__sass_thread_inst_executed_op_dadd_pred_on.sum",
           "smsp__sass_thread_inst_executed_op_dmul_pred_on.sum",
           "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for m in METRICS:
            if m in hdr:
                d[m] = r[hdr.index(m)] + (" " + units[hdr.index(m)] if units[hdr.index(m)] else "")
        stalls = {}
        for i, h in enumerate(hdr):
            if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio"):
                try:
                    v = float(r[i])
                except ValueError:
                    continue
                if v >= 0.3:
                    stalls[h[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]] = v
        d["stalls_per_issued_inst"] = dict(sorted(stalls.items(), key=lambda kv: -kv[1]))
        res.append(d)
    return res


def launches(path):
    if path == "-":   # no launch list for this capture
        return []
    rows = list(csv.reader(open(path)))
    hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[hdr_i]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[hdr_i + 1:]:
        if len(r) > vi and r[mi] == "gpu__time_duration.sum":
            name = r[ki].split("(")[0].replace("void ", "")
            agg[name][0] += 1
            agg[name][1] += float(r[vi].replace(",", ""))
    tot = sum(v[1] for v in agg.values()) or 1.0
    return [{"kernel": k, "launches": v[0], "total_ns": v[1], "share": v[1] / tot}
            for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1])]


if __name__ == "__main__":
    rep, lcsv, out = sys.argv[1], sys.argv[2], sys.argv[3]
    res = {"capture": raw(rep), "launch_list": launches(lcsv)}
    with open(out + ".json", "w") as f:
        json.dump(res, f, indent=1)
    with open(out + ".md", "w") as f:
        f.write(f"# ncu summary: {rep.split('/')[-1]} + {lcsv.split('/')[-1]}\n\n")
        f.write("## Launch list (cold-cache, serialised; compare shares)\n\n| kernel | launches | total us | share |\n|---|---|---|---|\n")
        for l in res["launch_list"]:
            f.write(f"| {l['kernel']} | {l['launches']} | {l['total_ns']/1e3:.1f} | {l['share']*100:.1f}% |\n")
        for c in res["capture"]:
            f.write(f"\n## {c['kernel'][:90]}\n\n")
            for k, v in c.items():
                if k not in ("kernel", "stalls_per_issued_inst"):
                    f.write(f"- {k}: {v}\n")
            f.write(f"- stalls per issued instruction: {c['stalls_per_issued_inst']}\n")
    print(open(out + ".md").read())
