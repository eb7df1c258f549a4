cd $GRAFT_REPO_ROOT
timeout 900 python tools/shard_sim.py C5-eps0.5 --no-estimate > gpurun_out/r2o_shards_C5.json 2> gpurun_out/r2o_shards.err
python -c "
import json;d=json.load(open('gpurun_out/r2o_shards_C5.json'))
for R,x in d['per_R'].items(): print(R, 'max ms %.3f'%x['step_ms_max_over_ranks'], 'speedup %.2f'%x.get('simulated_speedup',0), 'imb %.3f'%x['pair_imbalance_max_over_mean'], 'grid', ['%.2f'%g for g in x['grid_ms_per_rank']], 'step', ['%.2f'%g for g in x['step_ms_per_rank']], x['points_per_rank_grid'])"
ncu --set full --clock-control none -k regex:"k_scan_lookback" -c 3 -o gpurun_out/r2o_prof_scan python tools/shard_sim.py C5-eps0.5 --no-estimate --ranks 8 --only-rank 3 --reps 1 > /dev/null 2>&1
ls -la gpurun_out | grep r2o
