"""profiles/traffic.json: measured DRAM bytes (dram__bytes_read.sum +
dram__bytes_write.sum, ncu) of the table kernels that bench.py's roofline
covers, per launch, for every bench workload -- the single pass k_fused, or
the two-pass write phase (k_emit + the sparse queries' k_sparse<write>).
bench.py reads the key matching its run into roofline.traffic.

usage (on the GPU box): python tools/traffic.py [WORKLOAD ...] -> merges into profiles/traffic.json
"""
import csv
import io
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402

METRICS = "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum"


def capture(wl, dtype="f64", kernel=0, split=0):
    log = f"/tmp/traffic_{wl}.csv"
    cmd = ["ncu", "--metrics", METRICS, "--clock-control", "none", "--csv", "--log-file", log,
           "-k", "regex:k_fused|k_emit|k_sparse|k_qlanes", sys.executable, os.path.join(ROOT, "bench.py"),
           "--workload", wl, "--steps", "1", "--warmup", "0", "--e2e-steps", "0", "--no-cpu-baseline",
           "--dtype", dtype, "--kernel", str(kernel), "--cell-split", str(split)]
    subprocess.run(cmd, check=True, capture_output=True)
    rows = list(csv.reader(io.StringIO(open(log).read())))
    i0 = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    h = rows[i0]
    iid, ik, im, iu, iv = (h.index(x) for x in ("ID", "Kernel Name", "Metric Name", "Metric Unit", "Metric Value"))
    per = {}
    for r in rows[i0 + 1:]:
        if len(r) <= iv:
            continue
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
                 "msecond": 1e-3, "ns": 1e-9, "us": 1e-6, "ms": 1e-3}.get(r[iu], 1)
        d = per.setdefault(r[iid], {"kernel": r[ik]})
        d[r[im]] = float(r[iv].replace(",", "")) * scale
    launches = list(per.values())
    # single pass: k_fused (+ k_sparse_fused / k_qlanes for the sparse / small groups of the split)
    fused = [d for d in launches if "k_fused" in d["kernel"] or "k_sparse_fused" in d["kernel"]
             or "k_qlanes" in d["kernel"]]
    if fused:
        pick, single = fused, True
    else:   # two passes: the write phase = k_emit + k_sparse<..., true>
        sparse_write = re.compile(r"k_sparse<[^,>]*,\s*(true|\(bool\)1|1)>")
        pick = [d for d in launches if "k_emit" in d["kernel"] or sparse_write.search(d["kernel"])]
        single = False
    tb = sum(d["dram__bytes_read.sum"] + d["dram__bytes_write.sum"] for d in pick)
    key = f"{wl}-{dtype}-k{kernel}-s{split}" + ("" if single else "-2p")
    return key, int(tb), {"kernels": [d["kernel"][:60] for d in pick],
                          "read": sum(d["dram__bytes_read.sum"] for d in pick),
                          "write": sum(d["dram__bytes_write.sum"] for d in pick),
                          "seconds": sum(d["gpu__time_duration.sum"] for d in pick)}


def main():
    wls = sys.argv[1:] or sorted(bench.WORKLOADS)
    path = os.path.join(ROOT, "profiles", "traffic.json")
    data = json.load(open(path)) if os.path.exists(path) else {}
    detail = data.setdefault("_detail", {})
    for wl in wls:
        key, tb, d = capture(wl)
        data[key] = tb
        detail[key] = d
        print(key, tb, d, flush=True)
    data["_note"] = ("dram__bytes_read.sum + dram__bytes_write.sum per launch of the table kernels bench.py's "
                     "roofline covers (ncu, tools/traffic.py): keys without -2p = the single pass k_fused; "
                     "-2p = the two-pass write phase (k_emit + k_sparse<write>)")
    for out in (path, os.path.join(ROOT, "gpurun_out", "traffic.json")):
        os.makedirs(os.path.dirname(out), exist_ok=True)
        with open(out, "w") as f:
            json.dump(data, f, indent=1)


if __name__ == "__main__":
    main()
