#!/usr/bin/env python
"""Table II analogue on one B200 (Exp. Scenario 1, Sec. VII-C):
single-invocation kernel time of the paper's GPUCalcGlobal (Alg. 2) and
GPUCalcShared (Alg. 3), compiled for sm_100a (search_kernel 7 / 8, eps cells),
beside this library's count + write kernels, on the synthetic stand-ins of the
paper's datasets at the paper's eps:

  SW1   eps 0.20 -> C2 TEC-like, n = 1,864,620 (seed 2)
  SW4   eps 0.07 -> TEC-like, n = 5,159,737 (seed 6; -12% non-empty cells vs SW4)
  SDSS1 eps 0.20 -> C3 SDSS-like, n = 2,000,000 (seed 3)
  SDSS2 eps 0.07 -> C3 SDSS-like, n = 5,000,000 (seed 4)

The paper's K20c numbers are printed beside (context, other hardware: K20c
~208 GB/s vs B200 ~8 TB/s).  Also reported: nGPU (threads launched, the
paper's definition), non-empty cells, |R| and the key sort that the paper's
result set needs before T exists (Alg. 4 line 7).  Profiling aid: writes
gpurun_out/table2.json and prints a Markdown table.

Usage: python tools/table2.py [--reps 5] [--only SW1,SDSS1]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import datagen  # noqa: E402

PAPER = {  # Table II: (eps, Global ms, nGPU, Shared ms, nGPU)
    "SW1": (0.2, 503.270, 1_864_704, 531.411, 37_409_792),
    "SW4": (0.07, 518.245, 5_159_936, 1258.0, 255_272_704),
    "SDSS1": (0.2, 72.677, 2_000_128, 544.745, 110_757_120),
    "SDSS2": (0.07, 80.038, 5_000_192, 1699.0, 649_954_560),
}
DATA = {
    "SW1": lambda: datagen.tec_like(),
    "SW4": lambda: datagen.tec_like(5_159_737, seed=6),
    "SDSS1": lambda: datagen.sdss_like(),
    "SDSS2": lambda: datagen.sdss_like(datagen.C3_N_LARGE, seed=4),
}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--only", default="")
    args = ap.parse_args()
    import torch
    from paper_conf_ipps_gowanlockrblp17_b200 import hdb
    torch.cuda.set_device(0)
    names = [s for s in args.only.split(",") if s] or list(PAPER)
    rows = []
    for name in names:
        eps, pg, png, ps, psn = PAPER[name]
        xy = torch.from_numpy(DATA[name]()).cuda()
        n = xy.shape[0]
        res = {"dataset": name, "n": n, "eps": eps,
               "paper_k20c": {"global_ms": pg, "global_nGPU": png, "shared_ms": ps, "shared_nGPU": psn}}
        for label, kern, split in (("global", 7, 1), ("shared", 8, 1), ("ours", 0, 0)):
            ctx = hdb.hdb_ctx_create(search_kernel=kern, cell_split=split)
            ks, ss, ts = [], [], []
            for r in range(args.reps + 1):
                g = hdb.hdb_grid_build(ctx, xy, eps)
                gv = hdb.hdb_grid_view_get(g)
                t = hdb.hdb_neighbor_table_device(ctx, g)
                st = hdb.hdb_stats_get(ctx)
                P = hdb.hdb_table_view_get(t).npairs
                hdb.hdb_table_free(t)
                hdb.hdb_grid_free(g)
                if r == 0:
                    continue   # warm-up
                if kern:
                    ks.append(st["ms_write_kernel"])
                    ss.append(st["ms_sort"])
                else:
                    ks.append(st["ms_count"] + st["ms_scan"] + st["ms_write_kernel"])
                ts.append(st["ms_table_wall"])
            hdb.hdb_ctx_destroy(ctx)
            d = {"kernel_ms": float(np.median(ks)), "pairs": int(P), "nonempty_cells": int(gv.n_nonempty),
                 "table_wall_ms": float(np.median(ts)), "cell_split": int(split) if split else "auto"}
            if kern == 7:
                d["nGPU"] = int((n + 255) // 256 * 256)
            elif kern == 8:
                d["nGPU"] = int(gv.n_nonempty) * 256
            if kern:
                d["sort_ms"] = float(np.median(ss))
                d["kernel_plus_sort_ms"] = d["kernel_ms"] + d["sort_ms"]
            else:
                d["note"] = "count + scan + write kernels (table complete, no sort needed)"
            res[label] = d
        res["speedup_ours_vs_global_kernel"] = res["global"]["kernel_ms"] / res["ours"]["kernel_ms"]
        res["speedup_ours_vs_global_table"] = res["global"]["kernel_plus_sort_ms"] / res["ours"]["kernel_ms"]
        res["shared_over_global"] = res["shared"]["kernel_ms"] / res["global"]["kernel_ms"]
        rows.append(res)
        print(json.dumps(res), flush=True)
        del xy
        torch.cuda.empty_cache()
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", "table2.json"), "w") as f:
        json.dump({"gpu": torch.cuda.get_device_name(0), "rows": rows}, f, indent=1)
    print("\n| dataset | eps | P | Global ms (nGPU) | Shared ms (nGPU) | Shared/Global | sort of R ms | "
          "ours ms (count+scan+write) | ours vs Global kernel | ours vs Global + sort | K20c Global / Shared ms |")
    print("|---|---|---|---|---|---|---|---|---|---|---|")
    for r in rows:
        print(f"| {r['dataset']} | {r['eps']} | {r['ours']['pairs']:.3e} | {r['global']['kernel_ms']:.3f} "
              f"({r['global']['nGPU']:,}) | {r['shared']['kernel_ms']:.3f} ({r['shared']['nGPU']:,}) | "
              f"{r['shared_over_global']:.2f} | {r['global']['sort_ms']:.3f} | {r['ours']['kernel_ms']:.3f} | "
              f"{r['speedup_ours_vs_global_kernel']:.1f}x | {r['speedup_ours_vs_global_table']:.1f}x | "
              f"{r['paper_k20c']['global_ms']} / {r['paper_k20c']['shared_ms']} |")


if __name__ == "__main__":
    main()
