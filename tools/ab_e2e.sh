#!/bin/bash
# A/B of the end-to-end (host-table) metric between library builds ab/libhdb_<V>.so
cd "$(dirname "$0")/.."
for wl in ${WLS:-C2-eps0.45}; do for r in $(seq ${REPS:-2}); do for v in ${VARS:-A B}; do
  HDB_LIB=ab/libhdb_$v.so python bench.py --workload $wl --steps 3 --warmup 2 --e2e-steps ${E2E:-3} --no-cpu-baseline > /tmp/o.json 2>/dev/null
  python -c "
import json;d=json.load(open('/tmp/o.json'));e=d['e2e']
print('%-12s %-4s e2e %.3e pairs/s  s/step %.4f  hybrid %.3e pts/s  device %.3e pts/s'%('$wl','$v',e['value'],e['s_per_step'],e['points_clustered_per_sec_hybrid'],e['points_clustered_per_sec_device']))"
done; done; done
