"""Break the bench's device clustering leg (pinned host points -> device table -> GPU
DBSCAN -> labels to the host) into its parts, each timed with a device sync on both
sides (profiling aid; C5 by default).  usage: python tools/e2e_device_breakdown.py [WORKLOAD]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import datagen
from paper_conf_ipps_gowanlockrblp17_b200 import hdb

wl = sys.argv[1] if len(sys.argv) > 1 else "C5-eps0.5"
name, eps = wl.split("-eps")
eps = float(eps)
gen = {"C5": datagen.dense_skew, "C2": datagen.tec_like, "C3": datagen.sdss_like}[name]
xy_np = gen()
n = xy_np.shape[0]
xy_pin = torch.from_numpy(xy_np).pin_memory()
ctx = hdb.hdb_ctx_create()
lab_h = np.empty(n, np.int32)
core_h = np.empty(n, np.uint8)
lab_d = torch.empty(n, dtype=torch.int32, device="cuda")
core_d = torch.empty(n, dtype=torch.uint8, device="cuda")


def tic():
    torch.cuda.synchronize()
    return time.perf_counter()


res = {}
for rep in range(4):
    t0 = tic()
    xy_d = xy_pin.cuda(non_blocking=True)
    t1 = tic()
    g = hdb.hdb_grid_build(ctx, xy_d, eps)
    t2 = tic()
    t = hdb.hdb_neighbor_table_device(ctx, g)
    t3 = tic()
    hdb.hdb_grid_free(g)
    _, _, k = hdb.hdb_dbscan(t, 4, labels=lab_d, is_core=core_d)
    t4 = tic()
    _, _, k2 = hdb.hdb_dbscan(t, 4, labels=lab_h, is_core=core_h)   # host label arrays (the bench's leg)
    t5 = tic()
    hdb.hdb_table_free(t)
    t6 = tic()
    g = hdb.hdb_grid_build(ctx, xy_pin, eps)   # the bench's call: from pinned host points
    t = hdb.hdb_neighbor_table_device(ctx, g)
    hdb.hdb_grid_free(g)
    hdb.hdb_dbscan(t, 4, labels=lab_h, is_core=core_h)
    hdb.hdb_table_free(t)
    t7 = tic()
    if rep:
        for key, v in (("h2d_ms", t1 - t0), ("grid_ms", t2 - t1), ("table_ms", t3 - t2), ("dbscan_dev_labels_ms", t4 - t3),
                       ("dbscan_host_labels_ms", t5 - t4), ("table_free_ms", t6 - t5), ("bench_leg_ms", t7 - t6)):
            res.setdefault(key, []).append(v * 1e3)
print(json.dumps({"workload": wl, "n": n, "clusters": k, "clusters_host_labels": k2,
                  **{k_: round(float(np.median(v)), 3) for k_, v in res.items()}}))
