#!/bin/bash
# Tuning aid for the dense/sparse split (HDB_SPARSE_TESTS): ms/step and kernel
# times per workload and threshold.  Usage (via gpurun): bash tools/sparse_sweep.sh "0 1024" "C3-eps0.20 C2-eps0.45"
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for wl in ${2:-C2-eps0.15 C2-eps0.45 C2-eps1.40 C3-eps0.20 C3L-eps0.07}; do
  for t in ${1:-0 256 1024 4096}; do
    HDB_SPARSE_TESTS=$t timeout 300 python bench.py --workload $wl --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ss.json 2> gpurun_out/ss.err
    python - "$wl" "$t" <<'PY'
import json, sys
try:
    d = json.load(open("gpurun_out/ss.json")); s = d["stats"]
    print("%-12s T=%-5s ms/step %7.3f grid %6.3f count %6.3f scan %6.3f write %6.3f sparse_q %9d groups %8d" % (
        sys.argv[1], sys.argv[2], d["ms_per_step"], s["ms_grid"], s["ms_count"], s["ms_scan"], s["ms_write_kernel"],
        s["n_sparse_queries"], s["n_groups"]))
except Exception as e:
    print(sys.argv[1], sys.argv[2], "FAILED", e, open("gpurun_out/ss.err").read()[-500:])
PY
  done
done
