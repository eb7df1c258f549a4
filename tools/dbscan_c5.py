"""One device DBSCAN on the C5 (or given) device table after a warm-up run (profiling aid:
ncu launch lists of the DBSCAN kernels).  usage: python tools/dbscan_c5.py [C5|C2] [eps] [reps]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import datagen
from paper_conf_ipps_gowanlockrblp17_b200 import hdb

which = sys.argv[1] if len(sys.argv) > 1 else "C5"
eps = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 1
xy = torch.from_numpy(datagen.dense_skew() if which == "C5" else datagen.tec_like()).cuda()
ctx = hdb.hdb_ctx_create()
g = hdb.hdb_grid_build(ctx, xy, eps)
t = hdb.hdb_neighbor_table_device(ctx, g)
hdb.hdb_grid_free(g)
n = xy.shape[0]
lab = torch.empty(n, dtype=torch.int32, device="cuda")
core = torch.empty(n, dtype=torch.uint8, device="cuda")
hdb.hdb_dbscan(t, 4, labels=lab, is_core=core)
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(reps):
    _, _, k = hdb.hdb_dbscan(t, 4, labels=lab, is_core=core)
torch.cuda.synchronize()
print("device dbscan ms", (time.perf_counter() - t0) / reps * 1e3, "clusters", k, flush=True)
