cd $GRAFT_REPO_ROOT
for wl in C2-eps0.45 C2-eps1.40 C2-eps0.15; do for k in 0 1 2 3 4 5; do
python bench.py --workload $wl --cell-split $k --steps 8 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /tmp/o.json 2>/dev/null
python -c "
import json;d=json.load(open('/tmp/o.json'));s=d['stats']
print('$wl split=$k ms %.3f grid %.3f count %.3f write %.3f single %d tests %.3e'%(d['ms_per_step'],s['ms_grid'],s['ms_count'],s['ms_write_kernel'],s['single_pass'],s['candidate_tests']))"
done; done
