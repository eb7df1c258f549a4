"""Time the device DBSCAN (NEXT-4) and the host DBSCAN on the C2 table (profiling aid)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import datagen
from paper_conf_ipps_gowanlockrblp17_b200 import hdb

eps = float(sys.argv[1]) if len(sys.argv) > 1 else 0.45
xy = torch.from_numpy(datagen.tec_like()).cuda()
ctx = hdb.hdb_ctx_create(search_kernel=int(os.environ.get("SK", "0")))   # SK=3: two passes
g = hdb.hdb_grid_build(ctx, xy, eps)
t = hdb.hdb_neighbor_table_device(ctx, g)
n = xy.shape[0]
lab = torch.empty(n, dtype=torch.int32, device="cuda")
for _ in range(2):
    hdb.hdb_dbscan(t, 4, labels=lab)
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(5):
    _, _, k = hdb.hdb_dbscan(t, 4, labels=lab)
torch.cuda.synchronize()
print("device dbscan ms", (time.perf_counter() - t0) / 5 * 1e3, "clusters", k)
th = hdb.hdb_neighbor_table(ctx, g)
if os.environ.get("GIANT"):
    import ctypes
    L = lab.cpu().numpy()
    v = hdb.hdb_table_view_get(th)
    cnt_np = np.ctypeslib.as_array(ctypes.cast(v.count, ctypes.POINTER(ctypes.c_uint32)), shape=(n,))
    sizes = np.bincount(L[L >= 0])
    top = np.argsort(sizes)[::-1][:5]
    pairs = np.bincount(L[L >= 0], weights=cnt_np[L >= 0].astype(np.float64))
    print("top clusters: point share", [round(sizes[c] / n, 3) for c in top],
          "pair share", [round(pairs[c] / v.npairs, 3) for c in top], flush=True)
labh = np.empty(n, np.int32)
for threads in ((1, 16, 0) if not os.environ.get("NOHOST") else ()):
    t0 = time.perf_counter()
    _, _, kh = hdb.hdb_dbscan(th, 4, n_threads=threads, labels=labh)
    print("host dbscan threads", threads, "ms", (time.perf_counter() - t0) * 1e3, "clusters", kh)
