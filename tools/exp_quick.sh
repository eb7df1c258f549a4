#!/bin/bash
# quick GPU iteration: a parity subset, then ms/step per workload for the kernel variants in KS
cd "$(dirname "$0")/.."; mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -k "${SEL:-c1_full or workload or near_ties or lattice or batching or shards or sparse or cell_split or kernel_variant}" 2>&1 | tail -2
for wl in ${WLS:-C2-eps0.45 C2-eps0.15 C2-eps1.40 C3L-eps0.07 C5-eps0.5}; do
 for k in ${KS:-0}; do
  python bench.py --workload $wl --kernel $k --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /tmp/o.json 2>/tmp/e.txt
  python -c "
import json;d=json.load(open('/tmp/o.json'));s=d['stats']
print('$wl k=$k ms %.3f grid %.3f sample %.3f count %.3f scan %.3f write %.3f frac %.3f'%(d['ms_per_step'],s['ms_grid'],s['ms_sample'],s['ms_count'],s['ms_scan'],s['ms_write_kernel'],d['roofline']['frac']))" || tail -3 /tmp/e.txt
 done
done
