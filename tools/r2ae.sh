cd $GRAFT_REPO_ROOT
for k in 1 2 3; do
  timeout 600 python bench.py --workload C5-eps0.5 --cell-split $k --steps 5 --warmup 2 --e2e-steps 0 --no-cpu-baseline > gpurun_out/r2ae_k$k.json 2>/dev/null
  python -c "
import json;d=json.load(open('gpurun_out/r2ae_k$k.json'));s=d['stats']
print('k=$k ms/step %.3f grid %.3f write %.3f tests %.3e groups %d' % (d['ms_per_step'], s['ms_grid'], s['ms_write_kernel'], s['candidate_tests'], s['n_groups']))"
done
