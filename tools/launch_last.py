"""Per-kernel times (us) of the last call in an ncu launch-list CSV, starting at the last
launch of the kernel named by the second argument (profiling aid)."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
h = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
hd = rows[h]; ik = hd.index("Kernel Name"); iv = hd.index("Metric Value"); iu = hd.index("Metric Unit")
ks = []
for r in rows[h + 1:]:
    if len(r) > iv:
        v = float(r[iv].replace(",", ""))
        v = v / 1e3 if r[iu] == "nsecond" else v * 1e3 if r[iu] == "msecond" else v
        ks.append((r[ik], v))
idx = [i for i, (k, v) in enumerate(ks) if sys.argv[2] in k]
last = ks[idx[-1]:]
for k, v in last:
    print("%-60s %9.1f us" % (k[:60], v))
print("total %.1f us" % sum(v for k, v in last))
