#!/bin/bash
# Round-2 evidence on one GPU: the GPU test suite, the default bench line (C5, with e2e
# and the CPU baselines), the other workloads' lines, the reference arm, launch lists and
# ncu captures of k_fused (C5, C2), the shard simulation and the Table II analogue.
# Usage (via gpurun): bash tools/round_evidence_r2.sh TAG
cd "$(dirname "$0")/.."
T=${1:-r2z}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/${T}_pytest.txt 2>&1
echo "PYTEST: $(tail -1 gpurun_out/${T}_pytest.txt)"; grep -E "^FAILED|^E  " gpurun_out/${T}_pytest.txt | head -5
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/${T}_bench_default.json 2> gpurun_out/${T}_bench.err
echo "default rc=$?"
for wl in C1-eps0.5 C2-eps0.45 C2-eps0.15 C2-eps1.40 C3-eps0.07 C3-eps0.20 C3L-eps0.07 C3L-eps0.20 C5-eps1.0; do
  timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --e2e-steps 2 --no-cpu-baseline > gpurun_out/${T}_bench_$wl.json 2>> gpurun_out/${T}_bench.err
done
timeout 600 python bench.py --workload C2-eps0.45 --dtype f32 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/${T}_bench_C2-eps0.45-f32.json 2>> gpurun_out/${T}_bench.err
timeout 900 python bench.py --workload C4-sweep --steps 3 --warmup 1 > gpurun_out/${T}_bench_C4.json 2>> gpurun_out/${T}_bench.err
timeout 900 python bench.py --impl reference --steps 5 --warmup 1 > gpurun_out/${T}_bench_reference.json 2>> gpurun_out/${T}_bench.err
for wl in C5-eps0.5 C2-eps0.45; do
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches_$wl.csv \
    python bench.py --workload $wl --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
  ncu --set full --clock-control none --import-source on -k regex:"k_fused|k_qlanes" -c 2 -o gpurun_out/${T}_prof_$wl \
    python bench.py --workload $wl --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
done
timeout 900 python tools/shard_sim.py C5-eps0.5 > gpurun_out/${T}_shards_C5.json 2>> gpurun_out/${T}_bench.err
timeout 900 python tools/table2.py --reps 3 > gpurun_out/${T}_table2.md 2>> gpurun_out/${T}_bench.err
ls -la gpurun_out | grep $T
