"""Host DBSCAN (the paper's split: host table T, all host cores) timed on a workload's
host table (profiling aid).  usage: python tools/host_dbscan_time.py [C5|C2] [eps] [reps]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import datagen
from paper_conf_ipps_gowanlockrblp17_b200 import hdb

which = sys.argv[1] if len(sys.argv) > 1 else "C5"
eps = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
xy = torch.from_numpy(datagen.dense_skew() if which == "C5" else datagen.tec_like()).cuda()
n = xy.shape[0]
ctx = hdb.hdb_ctx_create()
g = hdb.hdb_grid_build(ctx, xy, eps)
t = hdb.hdb_neighbor_table(ctx, g)
hdb.hdb_grid_free(g)
lab = torch.empty(n, dtype=torch.int32).pin_memory().numpy()
core = torch.empty(n, dtype=torch.uint8).pin_memory().numpy()
hdb.hdb_dbscan(t, 4, labels=lab, is_core=core)
ts = []
for _ in range(reps):
    t0 = time.perf_counter()
    _, _, k = hdb.hdb_dbscan(t, 4, labels=lab, is_core=core)
    ts.append(time.perf_counter() - t0)
print(json.dumps({"workload": which, "eps": eps, "threads": os.cpu_count(), "host_dbscan_s": min(ts),
                  "all_s": ts, "clusters": k, "lib": os.environ.get("HDB_LIB", "libhdb.so")}))
