#!/bin/bash
# Round evidence on one GPU: the default bench line (C2 eps 0.45, with e2e and the
# CPU baselines), supplementary lines (C3, C3L, C5, C4 sweep), the ncu launch list of
# the default bench and one full capture of its count + write kernels.
# Usage (via gpurun): bash tools/round_evidence.sh TAG
cd "$(dirname "$0")/.."
T=${1:-r1}
mkdir -p gpurun_out
python bench.py --steps 10 --warmup 3 > gpurun_out/${T}_bench_c2_eps045.json 2> gpurun_out/${T}_bench.err
for wl in C2-eps0.15 C2-eps1.40 C3-eps0.07 C3-eps0.20 C3L-eps0.07 C3L-eps0.20 C5-eps0.5; do
  python bench.py --workload $wl --steps 8 --warmup 3 --e2e-steps 2 --no-cpu-baseline > gpurun_out/${T}_bench_$wl.json 2>> gpurun_out/${T}_bench.err
done
python bench.py --workload C4-sweep --steps 3 --warmup 1 > gpurun_out/${T}_bench_C4.json 2>> gpurun_out/${T}_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches_c2_eps045.csv \
    python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_fused|k_count|k_emit" -c 2 -o gpurun_out/${T}_prof_c2 \
    python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
# the single pass on C5 (50M points) and the two-pass kernels on C3L (the dense/sparse split keeps them)
ncu --set full --clock-control none --import-source on -k regex:"k_fused" -c 1 -o gpurun_out/${T}_prof_c5 \
    python bench.py --workload C5-eps0.5 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_count|k_emit|k_sparse" -c 4 -o gpurun_out/${T}_prof_c3l \
    python bench.py --workload C3L-eps0.07 --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out | grep $T
