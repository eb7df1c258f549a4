cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 > gpurun_out/r2p_pytest.txt 2>&1
echo "PYTEST: $(tail -1 gpurun_out/r2p_pytest.txt)"; grep -E "^FAILED|^E  " gpurun_out/r2p_pytest.txt | head -8
timeout 900 python tools/shard_sim.py C5-eps0.5 > gpurun_out/r2p_shards_C5.json 2> gpurun_out/r2p_shards.err
python -c "
import json;d=json.load(open('gpurun_out/r2p_shards_C5.json'))
for R,x in d['per_R'].items(): print(R, 'max ms %.3f'%x['step_ms_max_over_ranks'], 'speedup %.2f'%x.get('simulated_speedup',0), 'imb %.3f'%x['pair_imbalance_max_over_mean'], 'ok', x['pairs_total_equals_P'], 'grid', ['%.2f'%g for g in x['grid_ms_per_rank']], 'step', ['%.2f'%g for g in x['step_ms_per_rank']])"
for wl in C5-eps0.5 C2-eps0.45; do
  timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/r2p_bench_$wl.json 2>> gpurun_out/r2p_bench.err
  python -c "
import json;d=json.load(open('gpurun_out/r2p_bench_$wl.json'));s=d['stats']
print('BENCH $wl ms/step %.3f grid %.3f write %.3f frac %.3f' % (d['ms_per_step'], s['ms_grid'], s['ms_write_kernel'], d['roofline']['frac']))"
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2p_launches_C5.csv python bench.py --workload C5-eps0.5 --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
