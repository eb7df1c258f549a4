#!/bin/bash
# compute-sanitizer passes (memcheck, racecheck, synccheck, initcheck) over a
# subset of the GPU parity tests that reaches every kernel family on small inputs.
# Usage (via gpurun): bash tools/sanitize.sh TAG
cd "$(dirname "$0")/.."
T=${1:-r1}
mkdir -p gpurun_out
SEL="c1_full_table or edge_cases or lattice or single_pass or cell_split or sparse_dense_hybrid or device_dbscan_matches or paper_kernels_match or batching_fault or dbscan_end_to_end or shard_bands or virtual_devices"
for tool in memcheck racecheck synccheck initcheck; do
  extra=""
  [ $tool = racecheck ] && extra="--racecheck-report hazard"
  timeout 1200 compute-sanitizer --tool $tool $extra --error-exitcode 99 --target-processes all \
      python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "$SEL" > gpurun_out/${T}_sanitize_$tool.txt 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|passed|failed' gpurun_out/${T}_sanitize_$tool.txt | tail -3 | tr '\n' ' ')"
done
