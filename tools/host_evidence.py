"""Host-side evidence on one GPU box, printed as one JSON line:

* PCIe: pinned host <-> device copy rates (1 stream; 3 concurrent streams, the
  batching layer's default), so the e2e D2H rate is a fraction of a
  measured peak;
* host DBSCAN on one C2 host table (eps 0.45): each minpts variant with one
  thread (the sequential Alg. 1 BFS) and with all cores, and the S3 pattern of
  P:1163-1219 -- 16 minpts variants on the same table run one after the other
  with one thread vs concurrently (one thread each);
* with HDB_TIMELINE=1 in the environment the library prints the GPU timeline
  of the batched host-table write (kernels and D2H copies per stream) and the
  host timeline of the hybrid sweep (build of T(eps_i+1) vs clustering of
  T(eps_i)) to stderr -- tools/r2_evidence.sh keeps them.

usage: HDB_TIMELINE=1 python tools/host_evidence.py 2> timeline.jsonl > evidence.json
"""
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import datagen  # noqa: E402
from paper_conf_ipps_gowanlockrblp17_b200 import hdb  # noqa: E402


def pcie(nbytes=2 << 30, reps=5):
    dev = torch.device("cuda", 0)
    h = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    d = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    out = {}
    for name, fn in (("d2h", lambda a, b: a.copy_(b, non_blocking=True)), ("h2d", lambda a, b: b.copy_(a, non_blocking=True))):
        for ns in (1, 3):
            streams = [torch.cuda.Stream(dev) for _ in range(ns)]
            part = nbytes // ns
            best = 0.0
            for _ in range(reps):
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                for i, st in enumerate(streams):
                    with torch.cuda.stream(st):
                        fn(h[i * part:(i + 1) * part], d[i * part:(i + 1) * part])
                torch.cuda.synchronize()
                best = max(best, part * ns / (time.perf_counter() - t0) / 1e9)
            out[f"{name}_{ns}stream_gbs"] = best
    out["bytes_per_copy"] = nbytes
    out["how"] = "pinned host tensor <-> device tensor copy_, wall clock around the copies, best of %d" % reps
    return out


def dbscan_threads(eps=0.45):
    xy = datagen.tec_like()
    ctx = hdb.hdb_ctx_create()
    g = hdb.hdb_grid_build(ctx, xy, eps)
    t = hdb.hdb_neighbor_table(ctx, g)
    hdb.hdb_grid_free(g)
    cores = os.cpu_count() or 1
    res = {"workload": f"C2 n={xy.shape[0]} eps={eps}", "host_cores": cores, "variants": {}}

    def run(m, th):
        t0 = time.perf_counter()
        lab, core, k = hdb.hdb_dbscan(t, m, n_threads=th)
        return time.perf_counter() - t0, k, lab

    for m in (4, 8, 16):
        run(m, 0)   # warm
        s1, k1, l1 = run(m, 1)
        sa, ka, la = run(m, 0)
        res["variants"][m] = {"single_thread_s": s1, "all_cores_s": sa, "speedup": s1 / sa, "clusters": k1,
                              "labels_equal": bool(np.array_equal(l1, la))}
    # S3: 16 minpts variants on one table -- sequentially with one thread vs
    # concurrently, one host thread each (the paper's 1 -> 16 thread reuse experiment)
    mps = [4 + 4 * i for i in range(16)]
    t0 = time.perf_counter()
    for m in mps:
        hdb.hdb_dbscan(t, m, n_threads=1)
    seq = time.perf_counter() - t0
    ths = [threading.Thread(target=lambda m=m: hdb.hdb_dbscan(t, m, n_threads=1)) for m in mps]
    t0 = time.perf_counter()
    for x in ths:
        x.start()
    for x in ths:
        x.join()
    par = time.perf_counter() - t0
    res["s3_16_minpts"] = {"minpts": mps, "sequential_1_thread_s": seq, "concurrent_16_threads_s": par,
                           "speedup": seq / par,
                           "paper": "SW1 4.37x (eps 0.3) .. 6.07x (eps 0.7) with 16 threads on a Xeon E5-2630 v3 (P:1213-1219)"}
    hdb.hdb_table_free(t)
    hdb.hdb_ctx_destroy(ctx)
    return res


def timelines():
    """Runs that print their timelines (HDB_TIMELINE=1) to stderr."""
    xy = datagen.tec_like()
    ctx = hdb.hdb_ctx_create()
    for eps in (0.45, 1.40):
        g = hdb.hdb_grid_build(ctx, xy, eps)
        t = hdb.hdb_neighbor_table(ctx, g)
        hdb.hdb_grid_free(g)
        hdb.hdb_table_free(t)
    hdb.hdb_ctx_destroy(ctx)
    ctx = hdb.hdb_ctx_create(sweep_on_device=0)
    eps, mp = list(datagen.C4_EPS), list(datagen.C4_MINPTS)
    hdb.hdb_sweep(ctx, xy, eps, mp)   # warm: grows the pinned pool
    t0 = time.perf_counter()
    hdb.hdb_sweep(ctx, xy, eps, mp)
    hyb = time.perf_counter() - t0
    hdb.hdb_ctx_destroy(ctx)
    return {"hybrid_c4_sweep_s": hyb}


if __name__ == "__main__":
    torch.cuda.set_device(0)
    out = {"pcie": pcie(), "host_dbscan": dbscan_threads()}
    if os.environ.get("HDB_TIMELINE") == "1":
        out["timelines"] = timelines()
    print(json.dumps(out))
