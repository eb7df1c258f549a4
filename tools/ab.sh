#!/bin/bash
# A/B timing of library builds on one box: ab/libhdb_<V>.so for V in $VARS (env
# "V:KEY=VAL" sets a runtime knob), interleaved $REPS times, per workload in $WLS.
cd "$(dirname "$0")/.."
for wl in ${WLS:-C2-eps0.45}; do
 for r in $(seq ${REPS:-3}); do
  for v in ${VARS:-A B}; do
   lib=${v%%:*}; kv=""; [[ "$v" == *:* ]] && kv=${v#*:}
   kern=0; [[ "$kv" == *KERNEL=* ]] && kern=$(echo "$kv" | sed 's/.*KERNEL=\([0-9]*\).*/\1/')
   env $kv HDB_LIB=ab/libhdb_$lib.so python bench.py --kernel $kern --workload $wl --steps ${STEPS:-10} --warmup 3 --e2e-steps 0 --no-cpu-baseline > /tmp/o.json 2>/tmp/e.txt
   python -c "
import json;d=json.load(open('/tmp/o.json'));s=d['stats']
print('%-12s %-16s ms %.3f grid %.3f count %.3f write %.3f sm %s'%('$wl','$v',d['ms_per_step'],s['ms_grid'],s['ms_count'],s['ms_write_kernel'],d['clocks']['sm_mhz']))" || tail -3 /tmp/e.txt
  done
 done
done
