#!/bin/bash
# Host / sharding evidence: PCIe peaks, host DBSCAN threads, timelines, shard simulation.
cd "$(dirname "$0")/.."
T=${1:-r2l}
mkdir -p gpurun_out
HDB_TIMELINE=1 timeout 900 python tools/host_evidence.py > gpurun_out/${T}_host_evidence.json 2> gpurun_out/${T}_timelines.jsonl
echo "host_evidence rc=$?"; tail -c 600 gpurun_out/${T}_host_evidence.json
for wl in C5-eps0.5 C2-eps0.45; do
  timeout 900 python tools/shard_sim.py $wl > gpurun_out/${T}_shards_$wl.json 2> gpurun_out/${T}_shards_$wl.err
  echo "shard_sim $wl rc=$?"; python -c "
import json;d=json.load(open('gpurun_out/${T}_shards_$wl.json'))
print('P',d['P'],'est err',d['sample']['rel_error'])
for R,x in d['per_R'].items(): print(R, 'max ms %.3f'%x['step_ms_max_over_ranks'], 'speedup %.2f'%x.get('simulated_speedup',0), 'imb %.3f'%x['pair_imbalance_max_over_mean'], 'ok', x['pairs_total_equals_P'], 'grid', ['%.2f'%g for g in x['grid_ms_per_rank']])"
done
