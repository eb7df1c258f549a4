#!/bin/bash
# One GPU iteration: GPU tests (all, or -k SEL), bench lines, launch lists.
# Usage: bash tools/r2_cycle.sh TAG "WORKLOADS" [pytest -k selection]
cd "$(dirname "$0")/.."
T=${1:-r2x}; WLS=${2:-"C5-eps0.5 C2-eps0.45"}; SEL=$3
mkdir -p gpurun_out
if [ "$SEL" != "none" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 ${SEL:+-k "$SEL"} > gpurun_out/${T}_pytest.txt 2>&1
  echo "PYTEST: $(tail -1 gpurun_out/${T}_pytest.txt)"; grep -E "^FAILED|^E  " gpurun_out/${T}_pytest.txt | head -8
fi
for wl in $WLS; do
  timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/${T}_bench_$wl.json 2>> gpurun_out/${T}_bench.err
  python -c "
import json;d=json.load(open('gpurun_out/${T}_bench_$wl.json'));s=d['stats']
print('BENCH $wl ms/step %.3f grid %.3f write %.3f count %.3f frac %.3f sm %s' % (d['ms_per_step'], s['ms_grid'], s['ms_write_kernel'], s['ms_count'], d['roofline']['frac'], d['clocks']['sm_mhz']))" || tail -3 gpurun_out/${T}_bench.err
  if [ -n "$LAUNCH" ]; then
    ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches_$wl.csv \
      python bench.py --workload $wl --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
  fi
done
