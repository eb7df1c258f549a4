"""Position-space clustering (hdb_sweep, sweep_on_device=1) vs the id-space device path
(device table + hdb_dbscan): identical labels, and their times (profiling aid).
usage: python tools/pos_space_check.py [C5|C2] [eps] [minpts]"""
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
mp = int(sys.argv[3]) if len(sys.argv) > 3 else 4
host = os.environ.get("HOST") == "1"   # the bench's buffers: pinned host points and labels
xy = torch.from_numpy(datagen.dense_skew() if which == "C5" else datagen.tec_like())
xy = xy.pin_memory() if host else xy.cuda()
n = xy.shape[0]
ctx = hdb.hdb_ctx_create(sweep_on_device=1)
if host:
    lab_s = torch.empty((1, 1, n), dtype=torch.int32).pin_memory()
    lab_i = torch.empty(n, dtype=torch.int32).pin_memory()
else:
    lab_s = torch.empty((1, 1, n), dtype=torch.int32, device="cuda")
    lab_i = torch.empty(n, dtype=torch.int32, device="cuda")


def id_space():
    g = hdb.hdb_grid_build(ctx, xy, eps)
    t = hdb.hdb_neighbor_table_device(ctx, g)
    hdb.hdb_grid_free(g)
    _, _, k = hdb.hdb_dbscan(t, mp, labels=lab_i.numpy() if host else lab_i)
    hdb.hdb_table_free(t)
    return k


def pos_space():
    return int(hdb.hdb_sweep(ctx, xy, [eps], [mp], labels=lab_s.numpy() if host else lab_s)[1][0, 0])


res = {}
for name, fn in (("id_space", id_space), ("pos_space", pos_space)):
    fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(3):
        k = fn()
    torch.cuda.synchronize()
    res[name] = {"ms": (time.perf_counter() - t0) / 3 * 1e3, "clusters": k}
res["labels_equal"] = bool(torch.equal(lab_i, lab_s[0, 0]))
print(json.dumps({"workload": which, "eps": eps, "minpts": mp, "host_buffers": host, **res}))
