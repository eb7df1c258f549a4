"""Per-shard evidence on ONE GPU: for R = 1, 2, 4, 8 process
shards, every rank's step (grid build of its band + its device table) is run
one after the other and timed with CUDA events; reported per R: the slowest
rank's step (what an R-GPU strong-scaling run is bounded by, without NCCL /
PCIe effects), the per-shard pair imbalance (max / mean pairs), the band
sizes, and the sampled-estimate error |a_b - P| / P of the paper's f = 0.01
estimator on the whole set.

usage: python tools/shard_sim.py [WORKLOAD] [--reps 3]  -> one JSON line
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ipps_gowanlockrblp17_b200 import hdb  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload", nargs="?", default="C5-eps0.5")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--ranks", default="1,2,4,8")
    ap.add_argument("--only-rank", type=int, default=-1, help="run only this rank of each R (profiling)")
    ap.add_argument("--no-estimate", action="store_true")
    args = ap.parse_args()
    wl = bench.WORKLOADS[args.workload]
    xy = wl["gen"]()
    eps = wl["eps"]
    n = xy.shape[0]
    dev = torch.device("cuda", 0)
    xy_dev = torch.from_numpy(xy).to(dev)
    stream = torch.cuda.current_stream(dev)
    out = {"workload": args.workload, "n": n, "eps": eps, "per_R": {}}

    # sampled estimate vs exact P (the paper's estimator, f = 0.01, on the whole set)
    if args.no_estimate:
        ctx = None
    else:
        ctx = hdb.hdb_ctx_create(search_kernel=3)   # two passes: the sample is always taken
    if ctx is None:
        P = None
    else:
        g = hdb.hdb_grid_build(ctx, xy_dev, eps)
        t = hdb.hdb_neighbor_table_device(ctx, g)
        st = hdb.hdb_stats_get(ctx)
        P = hdb.hdb_table_view_get(t).npairs
        hdb.hdb_table_free(t)
        hdb.hdb_grid_free(g)
        hdb.hdb_ctx_destroy(ctx)
        out["sample"] = {"f": 0.01, "sample_size": st["sample_size"], "est_pairs": st["est_pairs"],
                         "rel_error": abs(st["est_pairs"] - P) / P,
                         "planned_batches": st["planned_batches"], "planned_batch_pairs": st["planned_batch_pairs"]}
    out["P"] = P

    for R in [int(r) for r in args.ranks.split(",")]:
        rank_ms, rank_pairs, rank_pts, rank_grid = [], [], [], []
        for r in range(R):
            if args.only_rank >= 0 and r != args.only_rank:
                continue
            opts = dict(shard_rank=r, shard_count=R) if R > 1 else {}
            ctx = hdb.hdb_ctx_create(**opts)
            hdb.hdb_ctx_set_stream(ctx, stream.cuda_stream)

            def step():
                g = hdb.hdb_grid_build(ctx, xy_dev, eps)
                gv = hdb.hdb_grid_view_get(g)
                t = hdb.hdb_neighbor_table_device(ctx, g)
                v = hdb.hdb_table_view_get(t)
                s_ = hdb.hdb_stats_get(ctx)
                hdb.hdb_table_free(t)
                hdb.hdb_grid_free(g)
                return gv.n, v.npairs, s_["ms_grid"]

            step()
            torch.cuda.synchronize()
            ms = []
            for _ in range(args.reps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                npts, pairs, mg = step()
                e1.record(stream)
                torch.cuda.synchronize()
                ms.append(e0.elapsed_time(e1))
            hdb.hdb_ctx_destroy(ctx)
            rank_ms.append(float(np.median(ms)))
            rank_pairs.append(int(pairs))
            rank_pts.append(int(npts))
            rank_grid.append(float(mg))
        tot = sum(rank_pairs)
        out["per_R"][R] = {"step_ms_max_over_ranks": max(rank_ms), "step_ms_per_rank": rank_ms,
                           "grid_ms_per_rank": rank_grid, "pairs_per_rank": rank_pairs,
                           "pairs_total": tot, "pairs_total_equals_P": tot == P,
                           "pair_imbalance_max_over_mean": max(rank_pairs) / (tot / len(rank_pairs)),
                           "points_per_rank_grid": rank_pts,
                           "simulated_pairs_per_s": tot / (max(rank_ms) / 1e3)}
    base = out["per_R"].get(1)
    if base:
        for R, d in out["per_R"].items():
            d["simulated_speedup"] = base["step_ms_max_over_ranks"] / d["step_ms_max_over_ranks"]
    print(json.dumps(out))


if __name__ == "__main__":
    main()
