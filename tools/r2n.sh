cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 -k "shard or band or every_row or c1_full or workload or partition or sweep or dbscan" > gpurun_out/r2n_pytest.txt 2>&1
echo "PYTEST: $(tail -1 gpurun_out/r2n_pytest.txt)"; grep -E "^FAILED|^E  " gpurun_out/r2n_pytest.txt | head -8
timeout 900 python tools/shard_sim.py C5-eps0.5 --no-estimate > gpurun_out/r2n_shards_C5.json 2> gpurun_out/r2n_shards.err
python -c "
import json;d=json.load(open('gpurun_out/r2n_shards_C5.json'))
for R,x in d['per_R'].items(): print(R, 'max ms %.3f'%x['step_ms_max_over_ranks'], 'speedup %.2f'%x.get('simulated_speedup',0), 'imb %.3f'%x['pair_imbalance_max_over_mean'], 'grid', ['%.2f'%g for g in x['grid_ms_per_rank']], 'step', ['%.2f'%g for g in x['step_ms_per_rank']], x['points_per_rank_grid'])"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2n_launches_shard8_r3.csv python tools/shard_sim.py C5-eps0.5 --no-estimate --ranks 8 --only-rank 3 --reps 1 > /dev/null 2>&1
