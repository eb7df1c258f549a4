"""Aggregate an ncu --metrics gpu__time_duration.sum CSV launch list by kernel."""
import collections
import csv
import re
import sys

path = sys.argv[1]
div = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0   # e.g. number of steps in the list
agg = collections.defaultdict(lambda: [0, 0.0])
h = None
for r in csv.reader(open(path)):
    if "Kernel Name" in r:
        h = r
        continue
    if h is None or len(r) != len(h):
        continue
    d = dict(zip(h, r))
    if d.get("Metric Name") != "gpu__time_duration.sum":
        continue
    k = re.sub(r"\(.*", "", d["Kernel Name"]).replace("unnamed>::", "")[:70]
    v = float(d["Metric Value"].replace(",", ""))
    u = d.get("Metric Unit", "ns")
    v *= {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(u, 1e-3)
    agg[k][0] += 1
    agg[k][1] += v
tot = sum(t for _, t in agg.values())
print(f"{'launches':>8} {'us total/div':>14} {'share':>6}  kernel")
for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{c:8d} {t / div:14.1f} {100 * t / tot:5.1f}%  {k}")
