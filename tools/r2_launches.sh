#!/bin/bash
# Launch lists (cold-cache, serialised) of the C2 and C5 bench steps + short bench lines.
cd "$(dirname "$0")/.."
T=${1:-r2b}
mkdir -p gpurun_out
for wl in C5-eps0.5 C2-eps0.45 C3-eps0.07; do
  python bench.py --workload $wl --steps 8 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/${T}_bench_$wl.json 2>> gpurun_out/${T}_bench.err
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches_$wl.csv \
    python bench.py --workload $wl --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
done
ls -la gpurun_out | grep $T
