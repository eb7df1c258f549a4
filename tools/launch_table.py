"""Per-kernel totals of an ncu launch list (--metrics gpu__time_duration.sum --csv):
python tools/launch_table.py LIST.csv [n_steps]  (totals divided by n_steps)."""
import collections, csv, sys
rows = list(csv.reader(open(sys.argv[1])))
steps = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
i0 = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
h = rows[i0]
iK, iU, iV = h.index("Kernel Name"), h.index("Metric Unit"), h.index("Metric Value")
agg = collections.OrderedDict()
for r in rows[i0 + 1:]:
    if len(r) <= iV:
        continue
    k = r[iK].split("(")[0].replace("void ", "").replace("(anonymous namespace)::", "").replace("hdb::", "")
    v = float(r[iV].replace(",", ""))
    scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(r[iU], 1.0)
    a = agg.setdefault(k, [0, 0.0])
    a[0] += 1
    a[1] += v * scale
tot = sum(v for _, v in agg.values())
for k, (c, v) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{k[:60]:60s} {c / steps:5.1f} {v / steps:10.1f} us {100 * v / tot:5.1f}%")
print(f"{'total':60s} {'':5s} {tot / steps:10.1f} us")
