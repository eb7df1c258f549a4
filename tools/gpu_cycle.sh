#!/bin/bash
# One GPU iteration: parity tests (quick subset unless FULL=1) + short bench.
# Usage (via gpurun): bash tools/gpu_cycle.sh [bench args...]
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
if [ "${FULL:-0}" = "1" ]; then SEL=""; else SEL="-k c1_full or workload or near_ties or lattice or batching or shards or exact_f64 or dbscan_end or grid_structure or sparse or cell_split or device_dbscan"; fi
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 ${SEL:+-k "${SEL#-k }"} > gpurun_out/cycle_pytest.txt 2>&1
echo "PYTEST: $(tail -1 gpurun_out/cycle_pytest.txt)"
grep -E "FAILED|Error" gpurun_out/cycle_pytest.txt | head -5
timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline "$@" > gpurun_out/cycle_bench.json 2> gpurun_out/cycle_bench.err
python - <<'PY'
import json
try:
    d = json.load(open("gpurun_out/cycle_bench.json"))
    s = d["stats"]
    print("BENCH: ms/step %.3f value %.3e  grid %.3f sample %.3f count %.3f scan %.3f write %.3f  frac %.3f" % (
        d["ms_per_step"], d["value"], s["ms_grid"], s["ms_sample"], s["ms_count"], s["ms_scan"], s["ms_write_kernel"],
        d["roofline"]["frac"]))
except Exception as e:
    print("BENCH FAILED", e)
    print(open("gpurun_out/cycle_bench.err").read()[-2000:])
PY
