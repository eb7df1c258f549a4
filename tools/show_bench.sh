#!/bin/bash
# one line per bench JSON: ms/step, dominant kernel ms, frac, sparse queries, launches
for f in "$@"; do python - "$f" <<'PY'
import json,sys
f=sys.argv[1]
try:
  d=json.loads(open(f).read().strip().splitlines()[-1]); r=d['roofline']; s=d['stats']
  print(f.split('/')[-1], round(d['ms_per_step'],3), 'kern', round(r['kernel_ms'],3), 'frac', round(r['frac'],3), 'sparse', s['n_sparse_queries'], 'launch', s['kernel_launches'], 'tbl', round(d['latency']['table_kernels_ms'],3))
except Exception as e: print(f, 'ERR', e)
PY
done
