#!/usr/bin/env python
"""bench.py -- HYBRID-DBSCAN hot path on B200: eps-neighbour pairs/s.

One step = one pass of the whole device hot path over the workload: grid build
(bbox, keys, radix sort, cell offsets, groups), sampled count + plan, exact
count, scan, neighbour write into a device-resident table.
``value`` = pairs/s with the points resident in HBM; ``e2e`` = the same metric
through the C-ABI from pinned HOST points to a HOST table plus the host DBSCAN
(a1-a11), with the H2D/D2H copies inside the timed region.

Workload (default): C5, the dense-skew batching stress set (BASELINE.json
configs[4]): 50,000,000 points in [0,1000)^2, 10% of them in 1% of the area,
eps = 0.5, minpts = 4 -- the config BASELINE names for 1/2/4/8 GPUs.  The C2
(TEC-like, configs[1]) and C3 lines are kept under profiles/.

Multi-GPU (torchrun): every rank holds the full point set, builds the grid of
its band of cell rows (plus the halo rows its stencils reach) and computes the
table of the band's queries; the only
collective is an all_gather of the per-shard pair counts.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import datagen  # noqa: E402

WORKLOADS = {
    # C1 (BASELINE configs[0]): the oracle's small case; its bench line is a latency figure
    "C1-eps0.5": dict(gen=datagen.c1, eps=datagen.C1_EPS, desc="uniform n=10,000 in [0,100)^2 eps=0.5 minpts=4"),
    "C2-eps0.45": dict(gen=datagen.tec_like, eps=0.45, desc="TEC-like n=1,864,620 eps=0.45 minpts=4"),
    "C2-eps0.15": dict(gen=datagen.tec_like, eps=0.15, desc="TEC-like n=1,864,620 eps=0.15 minpts=4"),
    "C2-eps1.40": dict(gen=datagen.tec_like, eps=1.40, desc="TEC-like n=1,864,620 eps=1.40 minpts=4"),
    **{f"C3-eps{e:.2f}": dict(gen=datagen.sdss_like, eps=e, desc=f"SDSS-like n=2,000,000 eps={e:.2f} minpts=4")
       for e in datagen.C3_EPS},
    **{f"C3L-eps{e:.2f}": dict(gen=lambda: datagen.sdss_like(datagen.C3_N_LARGE, seed=4), eps=e,
                               desc=f"SDSS-like n=5,000,000 eps={e:.2f} minpts=4") for e in datagen.C3_EPS},
    "C5-eps0.5": dict(gen=datagen.dense_skew, eps=0.5, desc="dense-skew n=50,000,000 eps=0.5 minpts=4"),
    # the stretch point of the dense-skew set (BASELINE configs[4]: "large eps"): ~4x the pairs
    "C5-eps1.0": dict(gen=datagen.dense_skew, eps=1.0, desc="dense-skew n=50,000,000 eps=1.0 minpts=4"),
}
MINPTS = 4
SWEEP_WORKLOADS = {
    "C4-sweep": dict(gen=datagen.tec_like, eps=datagen.C4_EPS, minpts=datagen.C4_MINPTS,
                     desc="TEC-like n=1,864,620, eps {0.15,0.20,0.30,0.45,0.60,0.80,1.00,1.40} x minpts "
                          "{4,8,16}: 8 tables, each reused for 3 minpts"),
}


def pcie_d2h_peak(torch, dev, nbytes=1 << 30, reps=5):
    """Measured D2H rate into pinned host memory (the e2e table's bound)."""
    h = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    d = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    best = 0.0
    for _ in range(reps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        h.copy_(d, non_blocking=True)
        torch.cuda.synchronize()
        best = max(best, nbytes / (time.perf_counter() - t0) / 1e9)
    del h, d
    return best


def run_config(args, wl, ws):
    """The config dict both arms print (same keys and values for the same run)."""
    return {"workload": args.workload, "desc": wl["desc"], "eps": wl["eps"], "dtype": args.dtype,
            "parallelism": f"query-shard{ws}",
            "l2": "not flushed: every step writes the whole neighbour table (GBs, >> 126 MB L2)"}


def sweep_config(args, wl, ws):
    return {"workload": args.workload, "desc": wl["desc"], "dtype": args.dtype,
            "variants": len(wl["eps"]) * len(wl["minpts"]), "parallelism": f"eps-shard{ws}",
            "l2": "not flushed: every step writes 8 tables totalling ~88 GB (>> 126 MB L2)"}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


class ClockSampler:
    """SM clocks + throttle reasons sampled DURING the timed region.

    NVML (pynvml) polled every ~2 ms from a thread that is started before the
    region (timed regions here are tens of ms: an nvidia-smi process would not
    deliver its first sample in time); one sample is also taken at exit, so a
    region always has >= 1.  Falls back to `nvidia-smi -lms` when NVML is missing."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None
        self.nvml = None
        self.stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nvml = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.bits = [pynvml.nvmlClocksEventReasonHwSlowdown, pynvml.nvmlClocksEventReasonHwThermalSlowdown,
                         pynvml.nvmlClocksEventReasonSwThermalSlowdown, pynvml.nvmlClocksEventReasonSwPowerCap]
            self.max_sm = float(pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM))
        except Exception:
            self.nvml = None

    def _sample(self):
        sm = float(self.nvml.nvmlDeviceGetClockInfo(self.h, self.nvml.NVML_CLOCK_SM))
        r = self.nvml.nvmlDeviceGetCurrentClocksEventReasons(self.h)
        self.rows.append([sm, self.max_sm] + [bool(r & b) for b in self.bits])

    def _poll(self):
        while not self.stop.is_set():
            try:
                self._sample()
            except Exception:
                return
            time.sleep(0.002)

    def __enter__(self):
        if self.nvml is not None:
            self.t = threading.Thread(target=self._poll, daemon=True)
            self.t.start()
            return self
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) == 6 and parts[0].replace(".", "").isdigit():
                self.rows.append([float(parts[0]), float(parts[1]) if parts[1].replace(".", "").isdigit() else None]
                                 + [p.lower() == "active" for p in parts[2:]])

    def __exit__(self, *a):
        if self.nvml is not None:
            self.stop.set()
            self.t.join(timeout=2)
            try:
                self._sample()
            except Exception:
                pass
            return
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
            self.t.join(timeout=2)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        sm = [r[0] for r in self.rows]
        mx = [r[1] for r in self.rows if r[1] is not None]
        reasons = sorted({self.NAMES[i] for r in self.rows for i in range(4) if r[2 + i]})
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": max(mx) if mx else None, "reasons": reasons,
                "samples": len(self.rows), "source": "nvml" if self.nvml is not None else "nvidia-smi"}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def cpu_baseline_run(xy, eps, budget_s=12.0, rows=None, dtype="f64"):
    """The oracle as it stands (brute-force rows, OpenMP) on a bounded sample."""
    import oracle
    n = xy.shape[0]
    if rows is None:
        # calibrate on a small sample, then size the sample to ~budget_s
        probe = np.linspace(0, n - 1, min(n, 512)).astype(np.int64)
        oracle.eps_join_rowhash(xy, eps, probe[:8], dtype=dtype)   # warm (thread pool, pages)
        t0 = time.perf_counter()
        oracle.eps_join_rowhash(xy, eps, probe, dtype=dtype)
        dt = max(time.perf_counter() - t0, 1e-3)
        m = int(min(n, max(probe.size, probe.size * budget_s / dt)))
        rows = np.linspace(0, n - 1, m).astype(np.int64)
    t0 = time.perf_counter()
    cnt, _ = oracle.eps_join_rowhash(xy, eps, rows, dtype=dtype)
    dt = time.perf_counter() - t0
    pairs = int(cnt.sum())
    return dict(value=pairs / dt, unit="pairs/s", cores=oracle.threads(), kind="oracle", seconds=dt,
                sample=f"{rows.size} evenly spaced query rows x all {n} points, brute force "
                       f"({pairs} pairs, {rows.size * n:.3g} tests, {dt:.2f} s)"), rows


def cpu_gridjoin_run(xy, eps, dtype="f64", budget_s=4.0):
    """CPU grid-join comparator (cpu_baseline/, SURVEY 8(d) baselines 2 and 3):
    one core, then all cores, on an evenly spaced sample of query rows against
    the full grid; the grid build over all n points is timed separately."""
    import cpu_baseline
    n = xy.shape[0]
    probe = np.linspace(0, n - 1, min(n, 2000)).astype(np.int64)
    t = {}
    cpu_baseline.gridjoin_rows(xy, eps, probe, dtype=dtype, threads=1, timings=t)
    m = int(min(n, max(2000, 2000 * budget_s / max(t["join_s"], 1e-4))))
    rows = np.linspace(0, n - 1, m).astype(np.int64)
    out = {}
    cores = os.cpu_count() or 1
    for key, th in (("single_thread", 1), ("all_cores", cores)):
        t = {}
        off, _ = cpu_baseline.gridjoin_rows(xy, eps, rows, dtype=dtype, threads=th, timings=t)
        pairs = int(off[-1])
        out[key] = dict(value=pairs / t["join_s"], unit="pairs/s", cores=th, kind="cpu_grid_join",
                        grid_build_s=t["build_s"],
                        sample=f"{m} evenly spaced query rows vs the eps-grid of all {n} points "
                               f"({pairs} pairs, join {t['join_s']:.2f} s; grid build over all n "
                               f"{t['build_s']:.2f} s, 1 thread, qsort)")
    return out


def all_host_cores():
    """The reference arm runs on rank 0 alone: give the oracle's OpenMP every host
    core (torchrun exports OMP_NUM_THREADS=1 to each rank); set before liboracle loads."""
    try:
        cores = len(os.sched_getaffinity(0))
    except Exception:
        cores = os.cpu_count() or 1
    os.environ["OMP_NUM_THREADS"] = str(cores)


def run_reference(args, wl, ws, rank):
    if rank != 0:
        return
    all_host_cores()
    xy = wl["gen"]()
    K, W = args.steps, args.warmup
    res, rows = cpu_baseline_run(xy, wl["eps"], budget_s=max(2.0, 60.0 / max(K + W, 1)))
    for _ in range(W):
        cpu_baseline_run(xy, wl["eps"], rows=rows)
    vals = []
    t_all = time.perf_counter()
    for _ in range(K):
        r, _ = cpu_baseline_run(xy, wl["eps"], rows=rows)
        vals.append(r["value"])
    t_all = time.perf_counter() - t_all
    v = float(np.median(vals))
    line = {"impl": "reference", "metric": "eps_neighbor_pairs_per_sec", "value": v, "unit": "pairs/s",
            "n_gpus": ws, "steps": K, "warmup": W, "ms_per_step": 1000 * t_all / max(K, 1),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": run_config(args, wl, ws),
            "cpu_baseline": dict(res, value=v),
            "e2e": {"value": v, "unit": "pairs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_sweep(args, wl, ws, rank, local):
    """C4 (BASELINE.json configs[3]): the multi-clustering sweep.  One step = one
    hdb_sweep over all (eps, minpts) variants; metric = points clustered/s =
    n * |variants| / step time.  value: points and labels in HBM, tables in HBM,
    GPU DBSCAN (sweep_on_device=1).  e2e: the same call from pinned HOST points
    into HOST labels.  "hybrid": the paper's pipeline (tables D2H into host
    memory, host DBSCAN on T(eps_i) while the GPU builds T(eps_i+1)).
    N > 1: the eps values (independent tables) are dealt round-robin to ranks."""
    eps_all, mp = list(wl["eps"]), list(wl["minpts"])
    xy_np = wl["gen"]()
    if args.dtype == "f32":
        xy_np = xy_np.astype(np.float32)
    n = xy_np.shape[0]
    variants = len(eps_all) * len(mp)
    if args.impl == "reference":
        if rank != 0:
            return
        all_host_cores()
        # the oracle as it stands: brute-force rows (sampled) + Alg. 1 would need
        # the full table; time the brute-force join on a bounded row sample per eps
        K, W = args.steps, args.warmup
        res, t_full = [], 0.0
        for e in eps_all:
            r, rows = cpu_baseline_run(xy_np, e, budget_s=max(1.0, 40.0 / len(eps_all) / max(K + W, 1)))
            res.append(r)
            t_full += r["seconds"] * n / rows.size
        v = n * variants / t_full   # extrapolated: full brute-force tables; DBSCAN on T is negligible beside it
        line = {"impl": "reference", "metric": "points_clustered_per_sec", "value": v, "unit": "points/s",
                "n_gpus": ws, "steps": K, "warmup": W, "ms_per_step": 1e3 * t_full,
                "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
                "config": sweep_config(args, wl, ws),
                "cpu_baseline": {"value": v, "unit": "points/s", "cores": res[0]["cores"], "kind": "oracle",
                                 "sample": "per eps, brute-force rows (extrapolated to all n rows): "
                                           + "; ".join(r["sample"] for r in res)},
                "e2e": {"value": v, "unit": "points/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line), flush=True)
        return

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_gowanlockrblp17_b200 import hdb

    assert torch.cuda.is_available(), "bench.py needs a GPU"
    ndev = torch.cuda.device_count()
    local_dev = local % ndev
    torch.cuda.set_device(local_dev)
    if ws > 1:
        if ndev >= ws:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_dev))
        else:
            dist.init_process_group("gloo")
    dev = torch.device("cuda", local_dev)
    coll_dev = dev if (ws == 1 or ndev >= ws) else torch.device("cpu")
    my_eps = eps_all[rank::ws]
    xy_dev = torch.from_numpy(xy_np).to(dev)
    ctx = hdb.hdb_ctx_create(sweep_on_device=1, cell_split=args.cell_split, search_kernel=args.kernel)
    lab_dev = torch.empty((max(len(my_eps), 1), len(mp), n), dtype=torch.int32, device=dev)

    def step():
        if my_eps:
            return hdb.hdb_sweep(ctx, xy_dev, my_eps, mp, labels=lab_dev)[1]
        return None

    for _ in range(max(args.warmup, 0)):
        step()
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream(dev)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    l0 = hdb.hdb_kernel_launches()
    with ClockSampler(local_dev) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            k_dev = step()
        ev1.record(stream)
        torch.cuda.synchronize()
    launches = hdb.hdb_kernel_launches() - l0
    ms = ev0.elapsed_time(ev1)
    if ws > 1:
        t = torch.tensor([ms], device=coll_dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    value = n * variants * args.steps / (ms / 1e3)
    line = {"metric": "points_clustered_per_sec", "value": value, "unit": "points/s", "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": args.dtype,
            "data": "synthetic",
            "config": sweep_config(args, wl, ws), "n": n,
            "step": "hdb_sweep, sweep_on_device=1: per eps grid + device table; per minpts GPU "
                    "DBSCAN into device labels",
            "gpu_launches": launches, "clocks": clk.summary()}
    if rank == 0 and ws == 1:
        # e2e: same call from pinned host points into host labels
        xy_pin = torch.from_numpy(xy_np).pin_memory()
        lab_host = torch.empty((len(eps_all), len(mp), n), dtype=torch.int32).pin_memory().numpy()
        hdb.hdb_sweep(ctx, xy_pin, eps_all, mp, labels=lab_host)
        ts = []
        for _ in range(max(1, min(args.steps, 3))):
            t0 = time.perf_counter()
            _, k_host = hdb.hdb_sweep(ctx, xy_pin, eps_all, mp, labels=lab_host)
            ts.append(time.perf_counter() - t0)
        te = float(np.median(ts))
        esz = xy_np.itemsize * 2
        line["e2e"] = {"value": n * variants / te, "unit": "points/s", "h2d_bytes_per_step": esz * n * len(eps_all),
                       "d2h_bytes_per_step": 4 * n * variants, "s_per_step": te,
                       "includes": "pinned host points -> per eps: H2D, grid, device table, GPU DBSCAN x3 "
                                   "minpts, labels D2H"}
        same = bool(np.array_equal(lab_dev.cpu().numpy(), lab_host)) if len(my_eps) == len(eps_all) else None
        line["e2e"]["labels_equal_device_run"] = same
        line["n_clusters"] = k_host.tolist()
        if args.hybrid_steps > 0:
            ctx_h = hdb.hdb_ctx_create(sweep_on_device=0, cell_split=args.cell_split, search_kernel=args.kernel)
            lab_h = np.empty_like(lab_host)
            t0 = time.perf_counter()
            hdb.hdb_sweep(ctx_h, xy_pin, eps_all, mp, labels=lab_h)   # warm-up: grows the pinned pool
            first = time.perf_counter() - t0
            ts = []
            for _ in range(args.hybrid_steps):
                t0 = time.perf_counter()
                _, k_h = hdb.hdb_sweep(ctx_h, xy_pin, eps_all, mp, labels=lab_h)
                ts.append(time.perf_counter() - t0)
            hdb.hdb_ctx_destroy(ctx_h)
            th = float(np.median(ts))
            line["hybrid"] = {"value": n * variants / th, "unit": "points/s", "s_per_step": th,
                              "first_run_s": first, "first_run_note": "includes growing the pinned host pool to "
                                                                      "two resident tables (P:748-749: pinned "
                                                                      "allocation is expensive; reported apart)",
                              "labels_equal": bool(np.array_equal(lab_h, lab_host)),
                              "desc": "the paper's S2/S3 pipeline: tables D2H into pinned host memory, host "
                                      "DBSCAN (3 minpts threads) on T(eps_i) while the GPU builds T(eps_i+1)"}
        del k_dev
    hdb.hdb_ctx_destroy(ctx)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="hdb", choices=["hdb", "reference"])
    ap.add_argument("--workload", default="C5-eps0.5", choices=sorted(WORKLOADS) + sorted(SWEEP_WORKLOADS))
    ap.add_argument("--hybrid-steps", type=int, default=1,
                    help="C4-sweep: timed runs of the paper's hybrid sweep (host tables + host DBSCAN)")
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--kernel", type=int, default=0, help="search kernel variant (hdb_opts.search_kernel)")
    ap.add_argument("--cell-split", type=int, default=0, help="hdb_opts.cell_split (0 = library default)")
    args = ap.parse_args()
    ws, rank, local = dist_env()
    if args.workload in SWEEP_WORKLOADS:
        return run_sweep(args, SWEEP_WORKLOADS[args.workload], ws, rank, local)
    wl = WORKLOADS[args.workload]
    if args.impl == "reference":
        return run_reference(args, wl, ws, rank)

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_gowanlockrblp17_b200 import hdb

    assert torch.cuda.is_available(), "bench.py needs a GPU"
    ndev = torch.cuda.device_count()
    local_dev = local % ndev
    torch.cuda.set_device(local_dev)
    if ws > 1:
        # one process per GPU over NCCL; ranks sharing a GPU (testing on fewer GPUs than ranks)
        # fall back to gloo for the one collective (the gather of per-shard pair counts)
        if ndev >= ws:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_dev))
        else:
            dist.init_process_group("gloo")
    dev = torch.device("cuda", local_dev)
    coll_dev = dev if (ws == 1 or ndev >= ws) else torch.device("cpu")
    xy_np = wl["gen"]()
    if args.dtype == "f32":
        xy_np = xy_np.astype(np.float32)
    n = xy_np.shape[0]
    eps = wl["eps"]
    xy_dev = torch.from_numpy(xy_np).to(dev)
    stream = torch.cuda.current_stream(dev)
    opts = dict(shard_rank=rank, shard_count=ws) if ws > 1 else {}
    ctx = hdb.hdb_ctx_create(search_kernel=args.kernel, cell_split=args.cell_split, **opts)
    hdb.hdb_ctx_set_stream(ctx, stream.cuda_stream)

    def step():
        g = hdb.hdb_grid_build(ctx, xy_dev, eps)
        t = hdb.hdb_neighbor_table_device(ctx, g)
        st = hdb.hdb_stats_get(ctx)
        v = hdb.hdb_table_view_get(t)
        hdb.hdb_table_free(t)
        hdb.hdb_grid_free(g)
        return st, v

    for _ in range(max(args.warmup, 0)):
        step()
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    write_ms, count_ms, pairs_local, launches = [], [], 0, 0
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    l0 = hdb.hdb_kernel_launches()
    with ClockSampler(local_dev) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            st, v = step()
            write_ms.append(st["ms_write_kernel"])
            count_ms.append(st["ms_count"])
            pairs_local += v.npairs
        ev1.record(stream)
        torch.cuda.synchronize()
    launches = hdb.hdb_kernel_launches() - l0
    ms = ev0.elapsed_time(ev1)
    if ws > 1:
        from paper_conf_ipps_gowanlockrblp17_b200 import dist as hdist
        t = torch.tensor([ms], device=coll_dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
        # the path's one exchange: the gather of per-shard pair counts
        _, pairs_total = hdist.gather_pair_counts(pairs_local, device=coll_dev)
    else:
        pairs_total = pairs_local
    P = pairs_total // max(args.steps, 1)
    value = pairs_total / (ms / 1000.0)

    # roofline of the dominant kernel, HBM-write bound:
    #  * single pass (k_fused, device-resident tables): 4 B per pair written + per query
    #    12 B (begin/count by id) + the reads of the sorted coordinates and ids (16 B f64 /
    #    8 B f32 + 4 B) + 4 B per non-empty cell (its spans' starts) = 4P + 32n + 4C (f64);
    #  * two-pass write kernel (k_emit): 4 B per pair + 12 B per query (offset + id map).
    hbm, peak_kind = load_peaks()
    n_shard = (v.end_query - v.first_query) if ws > 1 else n
    single = bool(st.get("single_pass", 0))
    paper = args.kernel in (7, 8)   # the paper's GPUCalcGlobal / GPUCalcShared (Table II baseline)
    esz = 16 if args.dtype == "f64" else 8
    #  * paper kernels: the key/value result set R, 8 B per pair, + the query's coordinates and id
    alg_bytes = (8 * v.npairs + (esz + 4) * n_shard if paper else
                 4 * v.npairs + ((esz + 16) * n_shard + 4 * st["n_nonempty"] if single else 12 * n_shard))
    wms = float(np.mean(write_ms))
    achieved = alg_bytes / (wms / 1000.0) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        with open(tp) as f:
            # keyed by the kernel that ran (single pass / two passes); per-launch bytes of an
            # unsharded run only
            key = f"{args.workload}-{args.dtype}-k{args.kernel}-s{args.cell_split}" + ("" if single else "-2p")
            traffic = json.load(f).get(key) if ws == 1 else None
    # whole-step view: SURVEY 8(d) B_alg = 4P + 64n + 8C (f64) over the step time
    b_step = 4 * P + (4 * esz + 32) * n + 8 * st["n_nonempty"]
    cms = float(np.mean(count_ms))

    line = {"metric": "eps_neighbor_pairs_per_sec", "value": value, "unit": "pairs/s", "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": args.dtype,
            "data": "synthetic",
            "config": run_config(args, wl, ws),
            "n": n, "pairs_per_step": P, "table_gb": 4 * P / 1e9,
            "step": (("grid build + single-pass count/reserve/write (k_fused, capacity = the grid's "
                      "candidate tests, no sample; device-resident table)") if single and not st["est_pairs"] else
                     "grid build + sampled count + single-pass count/reserve/write (k_fused, "
                     "device-resident table)" if single else
                     "grid build + sampled count + count + scan + write (device-resident table)")
            + (" -- per rank: the grid of its band of cell rows (+ halo), its queries' table" if ws > 1 else ""),
            "gpu_launches": launches,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                         "frac": achieved / hbm, "traffic": traffic, "peak_kind": peak_kind,
                         "kernel": ({7: "k_paper_global (GPUCalcGlobal, Alg. 2)",
                                     8: "k_paper_shared (GPUCalcShared, Alg. 3)"}[args.kernel] if paper else
                                    ("k_fused (single pass: count + reserve + emit, a6-a8)"
                                     + ((" + k_qlanes (the small groups' queries, one per lane)" if st["query_lanes"]
                                         else " + k_sparse_fused (the sparse queries)") if st["n_sparse_queries"] else ""))
                                    if single
                                    else "k_emit (neighbour write, a8)"),
                         "kernel_ms": wms, "alg_bytes": alg_bytes},
            "count_kernel": ({"bound": "alu", "kernel": "k_fused (count part, a6)", "ms": wms,
                              "tests": st["candidate_tests"],
                              "tests_per_s": st["candidate_tests"] / (wms / 1e3) if wms > 0 else None,
                              "note": "single pass: the count and write share one kernel"} if single else
                             {"bound": "alu", "kernel": "k_count (count + hit masks, a6)", "ms": cms,
                              "tests": st["candidate_tests"],
                              "tests_per_s": st["candidate_tests"] / (cms / 1e3) if cms > 0 else None}),
            "step_roofline": {"alg_bytes": b_step, "achieved_gbs": b_step / (ms / args.steps / 1e3) / 1e9,
                              "frac": b_step / (ms / args.steps / 1e3) / 1e9 / hbm},
            "clocks": clk.summary(),
            "latency": {"ms_per_step": ms / args.steps, "grid_build_ms": st["ms_grid"],
                        "table_kernels_ms": wms, "table_wall_ms": st["ms_table_wall"]},
            "stats": {k: st[k] for k in ("n_nonempty", "n_groups", "candidate_tests", "ms_grid", "ms_sample",
                                         "ms_count", "ms_scan", "ms_write_kernel", "kernel_launches",
                                         "single_pass", "est_pairs", "ms_sort", "n_sparse_queries",
                                         "query_lanes")}}

    # ---- e2e through the C-ABI from pinned HOST points (H2D inside the timed region):
    #   value: the same metric (pairs/s) with the table delivered to a HOST table (D2H inside);
    #   plus points clustered/s for the paper's hybrid (host table + host DBSCAN) and for the
    #   device path (device table + GPU DBSCAN, labels D2H).
    if rank == 0 and ws == 1 and args.e2e_steps > 0 and not paper:
        hdb.hdb_ctx_set_stream(ctx, None)
        xy_pin = torch.from_numpy(xy_np).pin_memory()
        # the step's results land in pinned host buffers, like its inputs come from them
        labels = torch.empty(n, dtype=torch.int32).pin_memory().numpy()
        core = torch.empty(n, dtype=torch.uint8).pin_memory().numpy()

        def table_to_host():
            g = hdb.hdb_grid_build(ctx, xy_pin, eps)
            t = hdb.hdb_neighbor_table(ctx, g)
            hdb.hdb_grid_free(g)
            return t

        def timed(fn, reps):
            fn()   # warm the pinned pool / device pools
            ts = []
            out = None
            for _ in range(reps):
                t0 = time.perf_counter()
                out = fn()
                ts.append(time.perf_counter() - t0)
            return float(np.median(ts)), out

        def e2e_table():
            t = table_to_host()
            P_ = hdb.hdb_table_view_get(t).npairs
            hdb.hdb_table_free(t)
            return P_

        def e2e_hybrid():
            t = table_to_host()
            _, _, k = hdb.hdb_dbscan(t, MINPTS, labels=labels, is_core=core)
            hdb.hdb_table_free(t)
            return k

        # the device path through the public clustering call: hdb_sweep with one (eps, minpts) on a
        # sweep_on_device context -- grid, device table (position space) and GPU DBSCAN, labels D2H
        ctx_dev = hdb.hdb_ctx_create(sweep_on_device=1, cell_split=args.cell_split, search_kernel=args.kernel)
        lab_sweep = labels.reshape(1, 1, n)

        def e2e_device():
            return int(hdb.hdb_sweep(ctx_dev, xy_pin, [eps], [MINPTS], labels=lab_sweep)[1][0, 0])

        te, Pe = timed(e2e_table, args.e2e_steps)
        d2h_peak = pcie_d2h_peak(torch, dev)
        th, kh = timed(e2e_hybrid, max(1, args.e2e_steps - 1))
        lab_hybrid = labels.copy()
        td, kd = timed(e2e_device, args.e2e_steps)
        same_labels = bool(np.array_equal(lab_hybrid, labels))
        hdb.hdb_ctx_destroy(ctx_dev)
        line["e2e"] = {"value": Pe / te, "unit": "pairs/s", "h2d_bytes_per_step": esz * n,
                       "d2h_bytes_per_step": 4 * Pe + 12 * n, "s_per_step": te,
                       "includes": "pinned host points -> H2D -> grid -> count -> batched write + D2H on 3 streams "
                                   "straight into the host table T (a1-a10)",
                       "points_clustered_per_sec_hybrid": n / th, "s_per_step_hybrid": th,
                       "hybrid": "e2e + host DBSCAN on T (minpts=4, all host cores) -- the paper's split",
                       "points_clustered_per_sec_device": n / td, "s_per_step_device": td,
                       "device": "pinned host points -> hdb_sweep(sweep_on_device, one eps / minpts): grid, device "
                                 "table in position space, GPU DBSCAN -> labels D2H (NEXT-4)",
                       "n_clusters": kh, "n_clusters_device": kd, "labels_equal_hybrid_device": same_labels,
                       "pcie": {"d2h_peak_gbs": d2h_peak, "e2e_d2h_gbs": (4 * Pe + 12 * n) / te / 1e9,
                                "frac": (4 * Pe + 12 * n) / te / 1e9 / d2h_peak,
                                "peak_how": "pinned host <- device copy of 1 GiB, best of 5, measured in this run"}}
    elif ws > 1 and args.e2e_steps > 0 and not paper:
        # N ranks: every rank takes the pinned host points to a HOST table of its query shard
        # (H2D of all points, its shard's D2H); time = max over ranks (barriers around each
        # step), value = the pairs of all shards / that time.  Clustering needs the whole table
        # in one process and is reported at N = 1 only.
        hdb.hdb_ctx_set_stream(ctx, None)
        xy_pin = torch.from_numpy(xy_np).pin_memory()

        def shard_to_host():
            g = hdb.hdb_grid_build(ctx, xy_pin, eps)
            t = hdb.hdb_neighbor_table(ctx, g)
            hdb.hdb_grid_free(g)
            P_ = hdb.hdb_table_view_get(t).npairs
            hdb.hdb_table_free(t)
            return P_

        shard_to_host()   # warm the pinned pool / device pools
        ts, Ps = [], 0
        for _ in range(args.e2e_steps):
            dist.barrier()
            t0 = time.perf_counter()
            Ps = shard_to_host()
            tt = torch.tensor([time.perf_counter() - t0], device=coll_dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            ts.append(float(tt.item()))
        pt = torch.tensor([float(Ps)], device=coll_dev, dtype=torch.float64)
        dist.all_reduce(pt)
        te = float(np.median(ts))
        line["e2e"] = {"value": float(pt.item()) / te, "unit": "pairs/s", "h2d_bytes_per_step": esz * n * ws,
                       "d2h_bytes_per_step": 4 * int(pt.item()) + 12 * n, "s_per_step": te,
                       "includes": "per rank: pinned host points -> H2D -> grid -> count -> batched write + D2H of "
                                   "its query shard into a host table (a1-a10); max over ranks",
                       "points_clustered_per_sec_hybrid": None, "points_clustered_per_sec_device": None}
    else:
        line["e2e"] = None
    if rank == 0 and not args.no_cpu_baseline:
        line["cpu_baseline"], _ = cpu_baseline_run(xy_np, eps, dtype=args.dtype)
        line["cpu_baseline"]["grid_join"] = cpu_gridjoin_run(xy_np, eps, dtype=args.dtype)
    hdb.hdb_ctx_destroy(ctx)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
