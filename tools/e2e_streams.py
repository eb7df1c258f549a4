"""e2e (pinned host points -> host table) time vs the number of D2H streams (profiling aid).
usage: python tools/e2e_streams.py [WORKLOAD]"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ipps_gowanlockrblp17_b200 import hdb  # noqa: E402

wl = bench.WORKLOADS[sys.argv[1] if len(sys.argv) > 1 else "C5-eps0.5"]
xy = torch.from_numpy(wl["gen"]()).pin_memory()
for ns in (1, 2, 3, 4):
    for bp in (0, 1 << 28):
        ctx = hdb.hdb_ctx_create(n_streams=ns, batch_pairs=bp)
        ts = []
        for r in range(4):
            t0 = time.perf_counter()
            g = hdb.hdb_grid_build(ctx, xy, wl["eps"])
            t = hdb.hdb_neighbor_table(ctx, g)
            hdb.hdb_grid_free(g)
            P = hdb.hdb_table_view_get(t).npairs
            st = hdb.hdb_stats_get(ctx)
            hdb.hdb_table_free(t)
            ts.append(time.perf_counter() - t0)
        hdb.hdb_ctx_destroy(ctx)
        te = float(np.median(ts[1:]))
        print(f"streams {ns} batch_pairs {bp}: {te * 1e3:.1f} ms  {P / te:.3e} pairs/s  batches {st['n_batches']}", flush=True)
