#!/bin/bash
# ncu --set full (with source) of one kernel on one workload: bash tools/ncu_kernel.sh TAG WORKLOAD KREGEX
cd "$(dirname "$0")/.."
T=$1; WL=$2; K=$3
ncu --set full --clock-control none --import-source on -k regex:"$K" -c 1 -o gpurun_out/${T}_prof_$WL \
  python bench.py --workload $WL --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > gpurun_out/${T}_ncu_$WL.log 2>&1
ncu -i gpurun_out/${T}_prof_$WL.ncu-rep --page source --csv --print-source cuda,sass -k regex:"$K" > gpurun_out/${T}_cs_$WL.csv 2>&1
python tools/ncu_summary.py gpurun_out/${T}_prof_$WL.ncu-rep > gpurun_out/${T}_sum_$WL.txt 2>&1
