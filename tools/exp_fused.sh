cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for wl in C2-eps0.45 C2-eps0.15 C2-eps1.40 C3L-eps0.07 C5-eps0.5; do
 for k in ${KS:-0 5}; do
  python bench.py --workload $wl --kernel $k --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /tmp/o.json 2>/tmp/e.txt
  python -c "
import json;d=json.load(open('/tmp/o.json'));s=d['stats']
print('$wl k=$k ms %.3f grid %.3f count %.3f write %.3f single %s frac %.3f'%(d['ms_per_step'],s['ms_grid'],s['ms_count'],s['ms_write_kernel'],s['single_pass'],d['roofline']['frac']))" || tail -3 /tmp/e.txt
 done
done
