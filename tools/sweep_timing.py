"""One warm + one measured device sweep (C4) for launch-list profiling."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import datagen
from paper_conf_ipps_gowanlockrblp17_b200 import hdb

hybrid = len(sys.argv) > 1 and sys.argv[1] == "hybrid"
xy = torch.from_numpy(datagen.tec_like()).cuda()
ctx = hdb.hdb_ctx_create(sweep_on_device=0 if hybrid else 1)
eps, mp = list(datagen.C4_EPS), list(datagen.C4_MINPTS)
lab = torch.empty((len(eps), len(mp), xy.shape[0]), dtype=torch.int32, device="cuda")
if hybrid:
    import numpy as np
    lab = np.empty((len(eps), len(mp), xy.shape[0]), np.int32)
for i in range(2):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    hdb.hdb_sweep(ctx, xy, eps, mp, labels=lab)
    torch.cuda.synchronize()
    print("sweep s", time.perf_counter() - t0)
