#!/bin/bash
# ncu --set full of k_fused on the given workloads: bash tools/r2_ncu.sh TAG "WL1 WL2"
cd "$(dirname "$0")/.."
T=$1; WLS=${2:-"C5-eps0.5 C2-eps0.45"}
mkdir -p gpurun_out
for wl in $WLS; do
  ncu --set full --clock-control none --import-source on -k regex:"k_fused" -c 1 -o gpurun_out/${T}_prof_$wl \
    python bench.py --workload $wl --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > gpurun_out/${T}_ncu_$wl.log 2>&1
done
ls -la gpurun_out | grep $T
