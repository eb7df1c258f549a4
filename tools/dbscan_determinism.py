"""Repeat the device DBSCAN and compare with the host DBSCAN (debug aid)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import datagen
from paper_conf_ipps_gowanlockrblp17_b200 import hdb
xy = datagen.subsample(datagen.tec_like(), 40_000, seed=1)
for eps, minpts in ((0.45, 4), (0.15, 8)):
    ctx = hdb.hdb_ctx_create()
    g = hdb.hdb_grid_build(ctx, xy, eps)
    th = hdb.hdb_neighbor_table(ctx, g)
    td = hdb.hdb_neighbor_table_device(ctx, g)
    ref, refc, refk = hdb.hdb_dbscan(th, minpts, n_threads=1)
    bad = 0
    for it in range(20):
        lab, core, k = hdb.hdb_dbscan(td, minpts)
        if not np.array_equal(lab, ref):
            bad += 1
            d = np.nonzero(lab != ref)[0]
            if bad <= 2:
                print("mismatch", eps, it, "k", k, refk, "n_diff", d.size, "core?", refc[d[:5]], lab[d[:5]], ref[d[:5]])
    print(eps, minpts, "bad runs", bad, "/ 20")
