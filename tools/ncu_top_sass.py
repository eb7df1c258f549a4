"""Top stalled SASS instructions of one kernel in an .ncu-rep (profiling aid).
usage: python tools/ncu_top_sass.py REP KERNEL_REGEX [N]"""
import csv, io, subprocess, sys
rep, kre = sys.argv[1], sys.argv[2]
n = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k", "regex:" + kre],
                     capture_output=True, text=True).stdout
lines = out.splitlines()
starts = [i for i, l in enumerate(lines) if l.startswith('"Kernel Name"')]
blk = lines[starts[0]:starts[1] if len(starts) > 1 else None]
rows = list(csv.reader(io.StringIO("\n".join(blk[1:]))))
h, data = rows[0], rows[1:]
col = lambda name: h.index(name)
iS, iE = col("Warp Stall Sampling (All Samples)"), col("Instructions Executed")
keys = ["stall_long_sb", "stall_short_sb", "stall_wait", "stall_mio", "stall_lg", "stall_math", "stall_branch_resolving"]
tot = sum(float(r[iS] or 0) for r in data)
print("kernel:", blk[0][:100], " samples", tot)
for r in sorted(data, key=lambda r: -float(r[iS] or 0))[:n]:
    st = " ".join(f"{k[6:]}={r[col(k)]}" for k in keys if float(r[col(k)] or 0) > 0.1 * float(r[iS] or 1))
    print(f"{r[0][-5:]} {r[1][:58]:58s} {float(r[iS]) / tot * 100:5.1f}% exec={r[iE]} {st}")
