"""GPU parity: the CUDA path (through the C-ABI) against the CPU oracle.

Neighbour tables must be bit-exact after per-row sorting (counts first, then
lists); DBSCAN core flags, noise and labels must be equal (the library emits
the canonical labelling, so labels are simply equal).  Inputs are the seeded
generators of datagen/ at sizes the oracle finishes in seconds (several tiles,
ragged tails) plus sampled rows at the bench's full sizes.
"""
import math

import numpy as np
import pytest

import datagen
import oracle
from paper_conf_ipps_gowanlockrblp17_b200 import hdb

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    return torch


def _ctx(**opts):
    return hdb.hdb_ctx_create(**opts)


def _canon(begin, count, nbrs):
    """rows in id order, lists ascending -> (off, flat)"""
    n = count.size
    off = np.zeros(n + 1, np.uint64)
    np.cumsum(count.astype(np.uint64), out=off[1:])
    rows = np.repeat(np.arange(n, dtype=np.int64), count.astype(np.int64))
    src = (np.repeat(begin.astype(np.int64), count.astype(np.int64))
           + (np.arange(rows.size, dtype=np.int64) - np.repeat(off[:-1].astype(np.int64), count.astype(np.int64))))
    vals = nbrs[src] if rows.size else np.zeros(0, np.uint32)
    order = np.lexsort((vals, rows))
    return off, vals[order]


def lib_table(xy, eps, device=False, ctx=None, **opts):
    own = ctx is None
    if own:
        ctx = _ctx(**opts)
    try:
        g = hdb.hdb_grid_build(ctx, xy, eps)
        try:
            t = (hdb.hdb_neighbor_table_device if device else hdb.hdb_neighbor_table)(ctx, g)
        finally:
            hdb.hdb_grid_free(g)
        try:
            b, c, v = hdb.hdb_table_copy_to_host(t)
            view = hdb.hdb_table_view_get(t)
        finally:
            hdb.hdb_table_free(t)
        stats = hdb.hdb_stats_get(ctx)
    finally:
        if own:
            hdb.hdb_ctx_destroy(ctx)
    return b, c, v, view, stats


def assert_table_equal(xy, eps, b, c, v, dtype="f64"):
    off, nbr = oracle.eps_join(xy, eps, dtype=dtype)
    want_cnt = np.diff(off.astype(np.int64))
    assert np.array_equal(c.astype(np.int64), want_cnt), \
        f"count mismatch at rows {np.nonzero(c.astype(np.int64) != want_cnt)[0][:10]}"
    loff, lnbr = _canon(b, c, v)
    assert np.array_equal(lnbr, nbr)


# ------------------------------------------------------------------ tables
@pytest.mark.parametrize("device", [False, True])
@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_c1_full_table(torch_cuda, device, dtype):
    xy = datagen.c1()
    if dtype == "f32":
        xy = xy.astype(np.float32)
    b, c, v, view, st = lib_table(xy, datagen.C1_EPS, device=device)
    assert view.npairs == c.astype(np.int64).sum() == v.size
    assert st["npairs"] == view.npairs
    assert_table_equal(xy, datagen.C1_EPS, b, c, v, dtype)


@pytest.mark.parametrize("name,gen,eps_list", [
    ("tec", lambda: datagen.subsample(datagen.tec_like(), 40_000, seed=1), (0.15, 0.45, 1.40, 3.0)),
    ("sdss", lambda: datagen.subsample(datagen.sdss_like(), 40_000, seed=2), (0.07, 0.2, 0.6, 2.0)),
    ("skew", lambda: datagen.dense_skew(30_000, seed=7), (0.5, 4.0, 15.0)),
])
def test_workload_subsets(torch_cuda, name, gen, eps_list):
    xy = gen()
    for eps in eps_list:
        b, c, v, view, st = lib_table(xy, eps, device=True)
        assert_table_equal(xy, eps, b, c, v)


def test_input_from_device_tensor(torch_cuda):
    torch = torch_cuda
    xy = datagen.subsample(datagen.tec_like(), 20_000, seed=3)
    b, c, v, _, _ = lib_table(torch.from_numpy(xy).cuda(), 0.45, device=True)
    assert_table_equal(xy, 0.45, b, c, v)


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_near_ties_adversarial(torch_cuda, dtype):
    for eps in (0.45, 0.1, 1.4, 0.07):
        xy = datagen.near_ties(4000, eps, seed=int(eps * 100))
        if dtype == "f32":
            xy = xy.astype(np.float32)
        b, c, v, _, _ = lib_table(xy, eps, device=True)
        assert_table_equal(xy, eps, b, c, v, dtype)


def test_lattice_ties(torch_cuda):
    for k, eps in ((40, 1.0), (40, math.sqrt(2.0)), (33, 0.5), (20, 2.0)):
        xy = datagen.lattice(k, spacing=1.0 if eps >= 1 else 0.5, origin=(-7.25, 3.5))
        b, c, v, _, _ = lib_table(xy, eps)
        assert_table_equal(xy, eps, b, c, v)


def test_decimal_steps_on_a_line(torch_cuda):
    # points k*eps apart: membership decided by the rounded arithmetic
    x = np.array([k * 0.1 for k in range(3000)])
    xy = np.stack([x, np.zeros_like(x)], axis=1)
    for eps in (0.1, 0.2, 0.30000000000000004, 0.3):
        b, c, v, _, _ = lib_table(xy, eps)
        assert_table_equal(xy, eps, b, c, v)


def test_edge_cases(torch_cuda):
    # n = 0
    b, c, v, view, _ = lib_table(np.zeros((0, 2)), 1.0)
    assert view.n == 0 and view.npairs == 0
    # n = 1
    b, c, v, view, _ = lib_table(np.array([[3.0, -2.0]]), 0.5)
    assert c.tolist() == [1] and v.tolist() == [0]
    # duplicates, identical points -> P = n^2
    same = np.tile([[1.5, 2.5]], (700, 1))
    b, c, v, view, _ = lib_table(same, 0.01)
    assert view.npairs == 700 * 700 and np.all(c == 700)
    # all in one cell; negative coordinates; points on the bbox max
    xy = np.array([[-1.0, -1.0], [-0.9, -1.0], [-1.0, -0.95], [5.0, 5.0], [4.5, 5.0], [5.0, 4.5]])
    b, c, v, _, _ = lib_table(xy, 0.5)
    assert_table_equal(xy, 0.5, b, c, v)
    # ragged: 33 points in a single cell with one isolated far point
    rng = np.random.default_rng(1)
    xy = np.concatenate([rng.uniform(0, 0.1, (33, 2)), [[50.0, 50.0]]])
    b, c, v, _, _ = lib_table(xy, 0.2)
    assert_table_equal(xy, 0.2, b, c, v)


def test_dense_cell_bigger_than_group(torch_cuda):
    rng = np.random.default_rng(5)
    xy = np.concatenate([rng.normal(0, 0.05, (5000, 2)), rng.uniform(-5, 5, (3000, 2))])
    b, c, v, _, _ = lib_table(xy, 0.3, device=True)
    assert_table_equal(xy, 0.3, b, c, v)


def test_errors(torch_cuda):
    ctx = _ctx()
    try:
        for bad_eps in (0.0, -1.0, float("nan"), float("inf")):
            with pytest.raises(hdb.HdbError) as e:
                hdb.hdb_grid_build(ctx, datagen.c1(), bad_eps)
            assert e.value.status == hdb.HDB_EINVAL
        for bad in (float("nan"), float("inf"), -float("inf")):
            xy = datagen.c1()
            xy[17, 1] = bad
            with pytest.raises(hdb.HdbError) as e:
                hdb.hdb_grid_build(ctx, xy, 0.5)
            assert e.value.status == hdb.HDB_EINVAL
        xy = np.array([[-1e9, 0.0], [1e9, 1.0]])
        with pytest.raises(hdb.HdbError) as e:
            hdb.hdb_grid_build(ctx, xy, 1e-3)
        assert e.value.status == hdb.HDB_ERANGE
    finally:
        hdb.hdb_ctx_destroy(ctx)


# ------------------------------------------------------------------ grid structure
def test_grid_structure_fig1(torch_cuda):
    """Fig. 1: G holds per-cell ranges into A, |A| = |D|, the ids of
    a cell are contiguous in A; here also: cells in key order, stable (ids
    ascending inside a cell), keys = floor((x - xmin) / w)."""
    xy = datagen.subsample(datagen.tec_like(), 50_000, seed=4)
    eps = 0.45
    ctx = _ctx()
    try:
        g = hdb.hdb_grid_build(ctx, xy, eps)
        gg = hdb.hdb_grid_copy_to_host(g)
        hdb.hdb_grid_free(g)
    finally:
        hdb.hdb_ctx_destroy(ctx)
    v = gg["view"]
    ids, ckeys, start = gg["ids"], gg["cell_keys"], gg["cell_start"]
    n = xy.shape[0]
    assert np.array_equal(np.sort(ids), np.arange(n))                 # |A| = |D|, a permutation
    assert np.all(np.diff(ckeys.astype(np.int64)) > 0)                 # non-empty cells, ascending keys
    assert start[0] == 0 and start[-1] == n and np.all(np.diff(start.astype(np.int64)) > 0)
    keys = np.repeat(ckeys, np.diff(start.astype(np.int64)))           # key of every sorted position
    w = eps * (1 + 2.0 ** -19)
    assert v.cell_w == w
    inv = 1.0 / w
    cx = np.floor((xy[:, 0] - xy[:, 0].min()) * inv).astype(np.int64)
    cy = np.floor((xy[:, 1] - xy[:, 1].min()) * inv).astype(np.int64)
    assert v.nx == cx.max() + 1 and v.ny == cy.max() + 1
    want_key = cy * v.nx + cx
    assert np.array_equal(keys.astype(np.int64), want_key[ids])
    assert np.array_equal(gg["xy_sorted"], xy[ids])
    # stable: ids ascending inside each cell
    h = keys.astype(np.int64)
    same = h[1:] == h[:-1]
    assert np.all(ids[1:][same] > ids[:-1][same])
    assert v.n_nonempty == np.unique(want_key).size == ckeys.size
    assert v.n_groups == int(np.sum((np.diff(start.astype(np.int64)) + 31) // 32))


def test_sparse_extent_compact_grid(torch_cuda):
    """A few points spread over a huge extent: 10^12 grid cells, only the
    non-empty ones are stored (dense grids would not fit)."""
    rng = np.random.default_rng(3)
    centers = rng.uniform(-5e5, 5e5, (50, 2))
    xy = (centers[:, None, :] + rng.normal(0, 0.5, (50, 40, 2))).reshape(-1, 2)
    b, c, v, view, st = lib_table(xy, 1.0)
    assert st["n_cells"] > 10 ** 11
    assert_table_equal(xy, 1.0, b, c, v)


# ------------------------------------------------------------------ batching / streams / shards
def test_batching_fault_injection(torch_cuda):
    xy = datagen.subsample(datagen.tec_like(), 30_000, seed=5)
    eps = 0.8
    off, nbr = oracle.eps_join(xy, eps)
    P = int(off[-1])
    ref = None
    configs = [dict(), dict(batch_pairs=997), dict(batch_pairs=P // 7 + 1, n_streams=1),
               dict(batch_pairs=50_000, n_streams=5), dict(sample_fraction=1.0), dict(sample_fraction=0.5),
               dict(batch_pairs=1)]
    for cfg in configs:
        b, c, v, view, st = lib_table(xy, eps, **cfg)
        assert_table_equal(xy, eps, b, c, v)
        assert st["npairs"] == P
        if "batch_pairs" in cfg and cfg["batch_pairs"] < P:
            assert st["n_batches"] > 1
        lo, lv = _canon(b, c, v)
        if ref is None:
            ref = lv
        assert np.array_equal(lv, ref)


def test_host_budget_enomem(torch_cuda):
    xy = datagen.subsample(datagen.tec_like(), 20_000, seed=6)
    with pytest.raises(hdb.HdbError) as e:
        lib_table(xy, 0.8, host_budget_bytes=1000)
    assert e.value.status == hdb.HDB_ENOMEM


def test_estimate_and_plan_stats(torch_cuda):
    """The sampled estimate a_b and the Eq. 1 plan of the batched host-table path (a5);
    dense device tables skip the sample (test_single_pass_selection_and_exact_bound)."""
    xy = datagen.subsample(datagen.tec_like(), 200_000, seed=8)
    b, c, v, view, st = lib_table(xy, 0.45)
    assert st["sample_size"] == math.ceil(xy.shape[0] / 100)
    assert st["est_pairs"] == st["sample_pairs"] * 100
    bb, nb = hdb.hdb_plan_batches(st["est_pairs"], 0.05, 3)
    assert st["planned_batches"] == nb
    # the strided sample of the cell-sorted order is a decent estimator
    assert abs(st["est_pairs"] - view.npairs) / view.npairs < 0.25
    assert st["candidate_tests"] >= view.npairs


def test_virtual_devices_in_one_context(torch_cuda):
    """Several 'devices' mapped to GPU 0: exercises the multi-device shard
    driver (sampled cuts, per-shard count/scan, gather of counts, per-shard
    D2H at global bases, host scatter of T) on one GPU."""
    xy = datagen.subsample(datagen.dense_skew(2_000_000, seed=5), 60_000, seed=1)
    eps = 3.0
    ref = lib_table(xy, eps)
    for devs in ([0, 0], [0, 0, 0, 0]):
        b, c, v, view, st = lib_table(xy, eps, devices=devs, batch_pairs=100_000)
        assert st["n_devices"] == len(devs)
        assert np.array_equal(c, ref[1])
        assert np.array_equal(_canon(b, c, v)[1], _canon(*ref[:3])[1])
    assert_table_equal(xy, eps, *ref[:3])


@pytest.mark.parametrize("R", [2, 3, 8])
def test_process_shards_partition_the_table(torch_cuda, R):
    """shard_rank/shard_count (torchrun mode): the R partial tables cover
    disjoint, contiguous ranges of the cell-sorted queries, their pair
    counts sum to P, and together they are the full table."""
    xy = datagen.subsample(datagen.sdss_like(), 50_000, seed=3)
    eps = 0.5
    full = lib_table(xy, eps, device=True)
    n = xy.shape[0]
    count = np.zeros(n, np.int64)
    rows_seen = np.zeros(n, np.int64)
    total = 0
    ranges = []
    for r in range(R):
        for device in (True, False):
            b, c, v, view, st = lib_table(xy, eps, device=device, shard_rank=r, shard_count=R)
            if device:
                ranges.append((view.first_query, view.end_query))
                total += view.npairs
                mine = c > 0
                rows_seen += mine
                count[mine] = c[mine]
                # each present row equals the full table's row
                fb, fc, fv = full[:3]
                for p in np.nonzero(mine)[0][:200]:
                    a = np.sort(v[b[p]:b[p] + c[p]])
                    bref = np.sort(fv[fb[p]:fb[p] + fc[p]])
                    assert np.array_equal(a, bref)
    assert ranges[0][0] == 0 and ranges[-1][1] == n
    assert all(ranges[i][1] == ranges[i + 1][0] for i in range(R - 1))
    assert total == full[3].npairs
    assert np.all(rows_seen == 1)
    assert np.array_equal(count, full[1].astype(np.int64))


def test_single_pass_device_table_and_fallback(torch_cuda):
    """search_kernel=4 builds device-resident tables in one pass (count + reserve
    + emit per group) into a table sized from the sampled estimate; an estimate
    that is far too low must fall back to the exact two-pass path, with the
    same table."""
    xy = datagen.subsample(datagen.tec_like(), 30_000, seed=4)
    for eps in (0.15, 0.45, 1.0):
        b, c, v, view, st = lib_table(xy, eps, device=True, search_kernel=4)
        assert st["single_pass"] == 1
        assert view.npairs == int(c.astype(np.int64).sum())
        assert_table_equal(xy, eps, b, c, v)
    # one sample (stride > n) on a sparse point: a_b ~ 1e6 << P ~ 9e6
    rng = np.random.default_rng(3)
    sparse = rng.uniform(0, 100, size=(17_000, 2))
    sparse[0] = (-50.0, -50.0)           # sorted position 0: an isolated point
    xy2 = np.concatenate([sparse, np.full((3_000, 2), 50.0)])
    b, c, v, view, st = lib_table(xy2, 0.5, device=True, sample_fraction=1e-6, search_kernel=4)
    assert st["single_pass"] == 0
    assert st["est_pairs"] < view.npairs
    assert_table_equal(xy2, 0.5, b, c, v)


def test_single_pass_selection_and_exact_bound(torch_cuda):
    """search_kernel 0 on device-resident tables: dense data (>= 150 candidate tests
    per query) takes the single pass sized by the exact bound P <= tests without a
    sampled estimate (est_pairs 0); moderately dense data the single pass sized from
    the sample; sparse data the two passes.  Every table equals the oracle, including
    the degenerate all-in-one-cell case (P = n^2) and f32 input."""
    rng = np.random.default_rng(22)
    dense = rng.uniform(0, 10, size=(40_000, 2))   # ~310 pairs, >= 400 candidate tests per query
    b, c, v, view, st = lib_table(dense, 0.5, device=True)
    assert st["single_pass"] == 1 and st["est_pairs"] == 0
    assert_table_equal(dense, 0.5, b, c, v)
    xf = dense.astype(np.float32)
    b, c, v, view, st = lib_table(xf, 0.5, device=True)
    assert st["single_pass"] == 1
    assert_table_equal(xf, 0.5, b, c, v, dtype="f32")
    mid = rng.uniform(0, 40, size=(40_000, 2))   # ~38 pairs, ~110 tests per query: the sample decides
    b, c, v, view, st = lib_table(mid, 0.7, device=True)
    assert st["single_pass"] == 1 and st["est_pairs"] > 0
    assert_table_equal(mid, 0.7, b, c, v)
    same = np.repeat(rng.uniform(0, 1, size=(1, 2)), 3_000, axis=0)   # one cell, every pair a neighbour
    b, c, v, view, st = lib_table(same, 0.5, device=True)
    assert st["single_pass"] == 1 and view.npairs == 3_000 ** 2
    assert_table_equal(same, 0.5, b, c, v)
    uni = rng.uniform(0, 100, size=(20_000, 2))   # ~3 pairs per query: the dense/sparse split,
    b, c, v, view, st = lib_table(uni, 0.5, device=True)   # single pass on both kinds of group
    assert st["single_pass"] == 1 and st["n_sparse_queries"] > 0 and st["est_pairs"] == 0
    assert_table_equal(uni, 0.5, b, c, v)
    b, c, v, view, st = lib_table(uni, 0.5, device=True, search_kernel=3)   # no split: two passes
    assert st["single_pass"] == 0 and st["n_sparse_queries"] == 0
    assert_table_equal(uni, 0.5, b, c, v)


def test_deterministic(torch_cuda):
    xy = datagen.subsample(datagen.tec_like(), 30_000, seed=9)
    a = lib_table(xy, 0.45)
    b = lib_table(xy, 0.45)
    for x, y in zip(a[:3], b[:3]):
        assert np.array_equal(x, y)


def test_sort_lists_option(torch_cuda):
    xy = datagen.subsample(datagen.tec_like(), 10_000, seed=2)
    b, c, v, _, _ = lib_table(xy, 0.6, sort_lists=1)
    for p in range(0, 10_000, 97):
        lst = v[b[p]:b[p] + c[p]]
        assert np.all(np.diff(lst.astype(np.int64)) > 0)


# ------------------------------------------------------------------ DBSCAN end to end
@pytest.mark.parametrize("threads", [1, 8])
def test_dbscan_end_to_end(torch_cuda, threads):
    for xy, eps, minpts in ((datagen.c1(), 0.5, 4),
                            (datagen.subsample(datagen.tec_like(), 30_000, seed=1), 0.45, 4),
                            (datagen.subsample(datagen.sdss_like(), 30_000, seed=1), 0.3, 8),
                            (datagen.subsample(datagen.tec_like(), 20_000, seed=2), 0.3, 1)):
        want = oracle.dbscan(*oracle.eps_join(xy, eps), minpts)
        ctx = _ctx()
        try:
            g = hdb.hdb_grid_build(ctx, xy, eps)
            t = hdb.hdb_neighbor_table(ctx, g)
            hdb.hdb_grid_free(g)
            lab, core, k = hdb.hdb_dbscan(t, minpts, n_threads=threads)
            hdb.hdb_table_free(t)
        finally:
            hdb.hdb_ctx_destroy(ctx)
        assert k == want[2]
        assert np.array_equal(core, want[1])
        assert np.array_equal(lab, want[0])


@pytest.mark.parametrize("on_device", [0, 1])
def test_sweep_matches_oracle(torch_cuda, on_device):
    xy = datagen.subsample(datagen.tec_like(), 20_000, seed=11)
    eps_list = (0.15, 0.3, 0.45, 1.0)
    mp = (4, 8, 16)
    ctx = _ctx(sweep_on_device=on_device)
    try:
        labels, k = hdb.hdb_sweep(ctx, xy, eps_list, mp)
    finally:
        hdb.hdb_ctx_destroy(ctx)
    for i, eps in enumerate(eps_list):
        off, nbr = oracle.eps_join(xy, eps)
        for j, m in enumerate(mp):
            want = oracle.dbscan(off, nbr, m)
            assert k[i, j] == want[2]
            assert np.array_equal(labels[i, j], want[0])


@pytest.mark.parametrize("case", ["sparse_split", "query_lanes", "f32"])
def test_device_sweep_position_space(torch_cuda, monkeypatch, case):
    """The device sweep clusters in position space (tables of sorted positions, T by
    position, union-find over positions with roots hooked by original id): through
    the single pass's three kernels -- k_fused with k_sparse_fused on SDSS-like
    sparse groups, with k_qlanes (forced) on dense-skew small groups, and f32 input
    -- the labels equal the oracle's canonical labelling (and the host sweep's)."""
    if case == "sparse_split":
        xy, eps_list = datagen.subsample(datagen.sdss_like(), 25_000, seed=12), (0.2, 0.6)
    elif case == "query_lanes":
        monkeypatch.setenv("HDB_QLANES", "1")
        xy, eps_list = datagen.dense_skew(25_000, seed=13), (4.0, 9.0)
    else:
        xy, eps_list = datagen.subsample(datagen.tec_like(), 20_000, seed=14).astype(np.float32), (0.3, 0.9)
    mp = (4, 12)
    ctx = _ctx(sweep_on_device=1)
    try:
        labels, k = hdb.hdb_sweep(ctx, xy, eps_list, mp)
        st = hdb.hdb_stats_get(ctx)
    finally:
        hdb.hdb_ctx_destroy(ctx)
    if case == "sparse_split":
        assert st["n_sparse_queries"] > 0 and not st["query_lanes"]
    if case == "query_lanes":
        assert st["n_sparse_queries"] > 0 and st["query_lanes"]
    dt = "f32" if case == "f32" else "f64"
    for i, eps in enumerate(eps_list):
        off, nbr = oracle.eps_join(xy, eps, dtype=dt)
        for j, m in enumerate(mp):
            want = oracle.dbscan(off, nbr, m)
            assert k[i, j] == want[2]
            assert np.array_equal(labels[i, j], want[0])


# ------------------------------------------------------------------ full-size sampled rows
def _sampled_rows_check(xy, eps, m_rows=1500, seed=0, dtype="f64", **opts):
    b, c, v, view, st = lib_table(xy, eps, device=True, **opts)
    n = xy.shape[0]
    assert view.npairs == c.astype(np.int64).sum()
    rng = np.random.default_rng(seed)
    rows = rng.choice(n, size=m_rows, replace=False)
    # plus the rows with the largest lists (dense-cell stress)
    rows = np.unique(np.concatenate([rows, np.argsort(c)[-50:]]))
    roff, rnbr = oracle.eps_join_rows(xy, eps, rows, dtype=dtype)
    for i, p in enumerate(rows):
        got = np.sort(v[b[p]:b[p] + c[p]])
        assert np.array_equal(got, rnbr[roff[i]:roff[i + 1]]), p
    # symmetry on the sampled rows
    for p in rows[:300]:
        for q in v[b[p]:b[p] + c[p]][:50]:
            lst = v[b[q]:b[q] + c[q]]
            assert p in lst
    return view, st


def test_c2_full_size_sampled_rows(torch_cuda):
    xy = datagen.tec_like()
    view, st = _sampled_rows_check(xy, 0.45)
    assert 1.0e9 < view.npairs < 2.0e9


@pytest.mark.parametrize("eps,lo,hi", [(0.15, 1.0e8, 3.0e8), (1.40, 7.0e9, 1.0e10)])
def test_c2_other_eps_full_size_sampled_rows(torch_cuda, eps, lo, hi):
    """The other C2 bench workloads at full size (the auto cell split picks
    k = 1 at eps 0.15 and k = 6 at eps 1.40; 1.40 is a 34 GB device table)."""
    xy = datagen.tec_like()
    view, st = _sampled_rows_check(xy, eps, m_rows=600, seed=int(eps * 100))
    assert lo < view.npairs < hi


def test_c2_full_size_f32_sampled_rows(torch_cuda):
    """bench.py --dtype f32 at full size: the predicate in f32 (reading R1/R2)."""
    xy = datagen.tec_like().astype(np.float32)
    view, st = _sampled_rows_check(xy, 0.45, m_rows=800, seed=32, dtype="f32")
    assert 1.0e9 < view.npairs < 2.0e9


def test_c3l_full_size_sampled_rows(torch_cuda):
    """C3L (5M SDSS-like) bench workloads at full size: eps 0.07 takes the
    dense/sparse split (single pass: warp-per-group k_fused on the dense groups,
    thread-per-query k_sparse_fused on the sparse queries), eps 0.20 the single
    pass without the split."""
    xy = datagen.sdss_like(datagen.C3_N_LARGE, seed=4)
    view, st = _sampled_rows_check(xy, 0.07, m_rows=800, seed=7)
    assert st["n_sparse_queries"] > 0 and st["single_pass"] == 1
    view, st = _sampled_rows_check(xy, 0.20, m_rows=800, seed=20)
    assert st["single_pass"] == 1


def test_c3_full_size_sampled_rows(torch_cuda):
    xy = datagen.sdss_like()
    for eps in datagen.C3_EPS:
        _sampled_rows_check(xy, eps, m_rows=800, seed=int(eps * 100))


def test_single_pass_natural_order_large_point_set(torch_cuda):
    """C5's recipe at 14M points (> 256 MB of coordinates + ids): the single
    pass visits the groups in cell-sorted order instead of the cost order
    ("C5 in the single pass") -- only point sets of C5's
    scale take this branch, so it is checked here on sampled rows."""
    xy = datagen.dense_skew(n=14_000_000, seed=15)
    assert xy.shape[0] * (16 + 4) > (256 << 20)
    view, st = _sampled_rows_check(xy, 0.7, m_rows=1000, seed=15)
    assert st["single_pass"] == 1
    assert 3e8 < view.npairs < 1e9


def test_c5_full_size_sampled_rows(torch_cuda):
    """C5 at the size and launch configuration bench.py times (50M points,
    eps 0.5, single pass in the natural order; a 15.8 GB device table)."""
    xy = datagen.dense_skew()
    view, st = _sampled_rows_check(xy, datagen.C5_EPS[0], m_rows=600, seed=5)
    assert st["single_pass"] == 1
    assert 3.5e9 < view.npairs < 4.5e9


def test_c5_eps1_full_size_sampled_rows(torch_cuda):
    """C5's stretch point, eps 1.0 (~4x the pairs of eps 0.5: a ~63 GB device table;
    the cells are 4x as full, so the groups are dense and take k_fused): sampled rows
    (plus the longest lists) against the oracle."""
    xy = datagen.dense_skew()
    view, st = _sampled_rows_check(xy, datagen.C5_EPS[1], m_rows=300, seed=6)
    assert st["single_pass"] == 1
    assert 1.4e10 < view.npairs < 1.8e10


def test_exact_f64_kernel_variant(torch_cuda):
    """search_kernel=1 forces the exact-f64-only kernel, 2 the write pass that
    recomputes the tests instead of replaying stored hit masks; all must equal
    the oracle, host- and device-resident."""
    xy = datagen.subsample(datagen.tec_like(), 30_000, seed=12)
    for eps in (0.15, 0.45):
        for k in (0, 1, 2):
            b, c, v, _, _ = lib_table(xy, eps, search_kernel=k)
            assert_table_equal(xy, eps, b, c, v)


def test_filter_disabled_for_huge_extent(torch_cuda):
    """Extent/eps so large that the f32 filter bound is useless: the library
    falls back to exact f64 and stays exact."""
    rng = np.random.default_rng(8)
    base = rng.uniform(-1e7, 1e7, (300, 2))
    xy = np.concatenate([base, base + rng.normal(0, 0.02, base.shape)])
    b, c, v, _, _ = lib_table(xy, 0.05)
    assert_table_equal(xy, 0.05, b, c, v)


@pytest.mark.parametrize("k", [2, 3, 4, 6])
def test_cell_split_parity(torch_cuda, k):
    """cell_split = k: cells of width eps/k and a (2k+1)^2 stencil (rows trimmed to the
    eps-disc for k >= 4; the lattice cases put exact ties on the disc); same table."""
    cases = [(datagen.subsample(datagen.tec_like(), 40_000, seed=1), (0.15, 0.45, 1.40)),
             (datagen.subsample(datagen.sdss_like(), 40_000, seed=2), (0.07, 0.6)),
             (datagen.near_ties(3000, 0.45, seed=3), (0.45,)),
             (datagen.lattice(30, origin=(-3.0, 7.0)), (1.0, math.sqrt(2.0)))]
    for xy, eps_list in cases:
        for eps in eps_list:
            for device in (True, False):
                b, c, v, view, st = lib_table(xy, eps, device=device, cell_split=k)
                assert_table_equal(xy, eps, b, c, v)
    xy = datagen.c1().astype(np.float32)
    b, c, v, _, _ = lib_table(xy, 0.5, cell_split=k)
    assert_table_equal(xy, 0.5, b, c, v, "f32")


@pytest.mark.parametrize("split", [0, 1])
def test_device_dbscan_matches_oracle(torch_cuda, split):
    """NEXT-4: DBSCAN on the device-resident table gives the canonical labels."""
    torch = torch_cuda
    cases = [(datagen.c1(), 0.5, 4), (datagen.c1(), 2.0, 1),
             (datagen.subsample(datagen.tec_like(), 40_000, seed=1), 0.45, 4),
             (datagen.subsample(datagen.tec_like(), 40_000, seed=1), 0.15, 8),
             (datagen.subsample(datagen.sdss_like(), 40_000, seed=2), 0.3, 4),
             (datagen.lattice(12), 1.0, 5)]
    for xy, eps, minpts in cases:
        want = oracle.dbscan(*oracle.eps_join(xy, eps), minpts)
        ctx = _ctx(cell_split=split)
        try:
            g = hdb.hdb_grid_build(ctx, xy, eps)
            t = hdb.hdb_neighbor_table_device(ctx, g)
            hdb.hdb_grid_free(g)
            lab, core, k = hdb.hdb_dbscan(t, minpts)                 # host output buffers
            dlab = torch.empty(xy.shape[0], dtype=torch.int32, device="cuda")
            _, _, k2 = hdb.hdb_dbscan(t, minpts, labels=dlab)        # device output buffer
            for _ in range(4):                                        # lock-free union-find: repeatable
                again, _, k3 = hdb.hdb_dbscan(t, minpts)
                assert k3 == k and np.array_equal(again, lab)
            hdb.hdb_table_free(t)
        finally:
            hdb.hdb_ctx_destroy(ctx)
        assert k == want[2] == k2
        assert np.array_equal(core, want[1])
        assert np.array_equal(lab, want[0])
        assert np.array_equal(dlab.cpu().numpy(), want[0])


@pytest.mark.parametrize("bridge", [False, True])
def test_device_dbscan_giant_components(torch_cuda, bridge):
    """Exercises the giant-component skip rule of k_union: rows in A skip, rows in
    B take only edges into A, other rows take edges into A/B and v < u."""
    xy = datagen.giants(5, bridge)
    for eps, minpts in ((0.25, 4), (0.25, 12), (0.5, 30)):
        want = oracle.dbscan(*oracle.eps_join(xy, eps), minpts)
        ctx = _ctx()
        try:
            g = hdb.hdb_grid_build(ctx, xy, eps)
            t = hdb.hdb_neighbor_table_device(ctx, g)
            hdb.hdb_grid_free(g)
            for _ in range(3):
                lab, core, k = hdb.hdb_dbscan(t, minpts)
                assert k == want[2]
                assert np.array_equal(core, want[1])
                assert np.array_equal(lab, want[0])
            hdb.hdb_table_free(t)
        finally:
            hdb.hdb_ctx_destroy(ctx)


def test_device_dbscan_shared_border_orders(torch_cuda):
    import json
    import os
    with open(os.path.join(os.path.dirname(__file__), "golden", "border_orders.json")) as f:
        g = json.load(f)
    for o in g["orders"]:
        xy = np.stack([np.array(o["x"], float), np.zeros(len(o["x"]))], axis=1)
        ctx = _ctx()
        try:
            gr = hdb.hdb_grid_build(ctx, xy, g["eps"])
            t = hdb.hdb_neighbor_table_device(ctx, gr)
            hdb.hdb_grid_free(gr)
            lab, core, k = hdb.hdb_dbscan(t, g["minpts"])
            hdb.hdb_table_free(t)
        finally:
            hdb.hdb_ctx_destroy(ctx)
        assert lab.tolist() == o["labels"] and core.tolist() == o["core"] and k == o["n_clusters"]


# ------------------------------------------------- the paper's kernels (NEXT-3)
@pytest.mark.parametrize("kernel", [7, 8])
@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_paper_kernels_match_oracle(torch_cuda, kernel, dtype):
    """search_kernel 7 / 8 = GPUCalcGlobal (Alg. 2) / GPUCalcShared (Alg. 3):
    atomic key/value result set, sorted by key, T read off the keys -- the same
    table as the oracle on the paper's eps cells (cell_split 1) and on split
    grids, for uniform, banded and clustered data."""
    cases = [(datagen.c1(), (datagen.C1_EPS,)),
             (datagen.subsample(datagen.tec_like(), 30_000, seed=1), (0.15, 0.45)),
             (datagen.subsample(datagen.sdss_like(), 30_000, seed=2), (0.07, 0.6))]
    for xy, eps_list in cases:
        if dtype == "f32":
            xy = xy.astype(np.float32)
        for eps in eps_list:
            for split in (1, 2):
                b, c, v, view, st = lib_table(xy, eps, device=True, search_kernel=kernel, cell_split=split)
                assert view.npairs == int(c.astype(np.int64).sum()) == st["npairs"]
                assert st["ms_sort"] > 0
                assert_table_equal(xy, eps, b, c, v, dtype)


@pytest.mark.parametrize("kernel", [7, 8])
def test_paper_kernels_dense_cell_and_overflow(torch_cuda, kernel):
    """A cell of 5,000 points (> blockDim = 256: Alg. 3's "additional loop",
    P:518-521) and an estimate far below |R| (one sample on an isolated point):
    the append counter reports the exact |R| and the kernel reruns once."""
    rng = np.random.default_rng(5)
    xy = np.concatenate([rng.normal(0, 0.05, (5000, 2)), rng.uniform(-5, 5, (3000, 2))])
    b, c, v, _, st = lib_table(xy, 0.3, device=True, search_kernel=kernel, cell_split=1)
    assert_table_equal(xy, 0.3, b, c, v)
    sparse = rng.uniform(0, 100, size=(17_000, 2))
    sparse[0] = (-50.0, -50.0)
    xy2 = np.concatenate([sparse, np.full((3_000, 2), 50.0)])
    b, c, v, view, st = lib_table(xy2, 0.5, device=True, sample_fraction=1e-6, search_kernel=kernel)
    assert st["est_pairs"] < view.npairs and st["pool_grows"] >= 1
    assert_table_equal(xy2, 0.5, b, c, v)


def test_paper_kernels_need_device_tables(torch_cuda):
    xy = datagen.c1()
    with pytest.raises(hdb.HdbError):
        lib_table(xy, datagen.C1_EPS, device=False, search_kernel=7)


# ------------------------------------------- dense/sparse hybrid (NEXT-1)
def test_sparse_dense_hybrid(torch_cuda):
    """Groups with few tests go to the thread-per-query kernel, the rest to the
    warp-per-group kernels, in one call: sparse-dominated (SDSS-like at small
    eps), mixed (dense square in sparse background) and dense-dominated data
    give the oracle's table, host- and device-resident, f64 and f32, the same
    as with the split disabled (search_kernel 3)."""
    cases = [(datagen.subsample(datagen.sdss_like(datagen.C3_N_LARGE, seed=4), 60_000, seed=3), 0.07 * 4),
             (datagen.dense_skew(40_000, seed=9), 2.0),
             (datagen.subsample(datagen.tec_like(), 40_000, seed=5), 0.45)]
    saw_mixed = False
    for xy, eps in cases:
        for dtype in ("f64", "f32"):
            x = xy.astype(np.float32) if dtype == "f32" else xy
            for device in (False, True):
                b, c, v, view, st = lib_table(x, eps, device=device)
                assert_table_equal(x, eps, b, c, v, dtype)
                saw_mixed |= 0 < st["n_sparse_queries"] < x.shape[0]
            b3, c3, v3, _, st3 = lib_table(x, eps, device=True, search_kernel=3)
            assert st3["n_sparse_queries"] == 0
            assert np.array_equal(c3, c)
    assert saw_mixed


def test_sparse_single_pass_many_hits(torch_cuda):
    """A sparse query (one query x <= 256 candidates) with more hits than the
    single-pass sparse kernel buffers (32): it re-scans its candidates to write
    them; the table still equals the oracle, f64 and f32, next to dense groups
    and isolated points."""
    rng = np.random.default_rng(8)
    lone = np.array([[0.99, 0.5]])                                        # alone in its cell
    clump = np.stack([rng.uniform(1.0, 1.3, 100), rng.uniform(0.4, 0.6, 100)], 1)   # all within eps of it
    far = rng.uniform(10, 400, size=(400, 2))                             # isolated: sparse groups
    xy = np.concatenate([lone, clump, far])
    for dtype in ("f64", "f32"):
        x = xy.astype(np.float32) if dtype == "f32" else xy
        b, c, v, view, st = lib_table(x, 1.0, device=True)
        assert st["single_pass"] == 1 and st["n_sparse_queries"] > 0
        assert c[0] == 101
        assert_table_equal(x, 1.0, b, c, v, dtype)


@pytest.mark.parametrize("R", [2, 4, 7])
def test_process_shard_bands_assemble_to_the_oracle_table(torch_cuda, R):
    """Process shards build only their band of cell rows plus the k halo rows
    (DESIGN.md sec. 7): each shard's grid holds fewer points than
    the input, the bands are consecutive ranges of the global cell-sorted
    order, and the shards' tables (single pass on device, two passes into host
    memory) assemble into exactly the oracle's table -- also with a skewed
    load (C5's dense square) and a cell split."""
    from paper_conf_ipps_gowanlockrblp17_b200 import dist as hdist
    xy = datagen.dense_skew(40_000, seed=21)
    n = xy.shape[0]
    for eps, split in ((3.0, 0), (5.0, 3)):
        for device in (True, False):
            parts, ranges = [], []
            for r in range(R):
                ctx = _ctx(shard_rank=r, shard_count=R, cell_split=split)
                try:
                    g = hdb.hdb_grid_build(ctx, xy, eps)
                    gv = hdb.hdb_grid_view_get(g)
                    assert gv.n < n
                    t = (hdb.hdb_neighbor_table_device if device else hdb.hdb_neighbor_table)(ctx, g)
                    hdb.hdb_grid_free(g)
                    v = hdb.hdb_table_view_get(t)
                    ranges.append((v.first_query, v.end_query))
                    parts.append(hdb.hdb_table_copy_to_host(t))
                    hdb.hdb_table_free(t)
                finally:
                    hdb.hdb_ctx_destroy(ctx)
            assert ranges[0][0] == 0 and ranges[-1][1] == n
            assert all(ranges[i][1] == ranges[i + 1][0] for i in range(R - 1))
            b, c, v = hdist.assemble(parts, n)
            assert_table_equal(xy, eps, b, c, v)


def test_process_shard_bands_empty_and_tiny(torch_cuda):
    """More shards than populated cell rows: some bands hold no queries (their
    tables are empty, P = 0) and the rest still assemble into the oracle's
    table; a single point and an all-identical set behave the same way."""
    from paper_conf_ipps_gowanlockrblp17_b200 import dist as hdist
    rng = np.random.default_rng(3)
    sets = [(np.stack([rng.uniform(0, 50, 300), rng.choice([0.1, 0.2, 3.9], 300)], 1), 0.5),
            (np.array([[1.5, -2.0]]), 1.0),
            (np.tile([[0.25, 0.75]], (70, 1)), 0.1)]
    for xy, eps in sets:
        n = xy.shape[0]
        for device in (True, False):
            parts, ranges, empty = [], [], 0
            for r in range(8):
                ctx = _ctx(shard_rank=r, shard_count=8)
                try:
                    g = hdb.hdb_grid_build(ctx, xy, eps)
                    t = (hdb.hdb_neighbor_table_device if device else hdb.hdb_neighbor_table)(ctx, g)
                    hdb.hdb_grid_free(g)
                    v = hdb.hdb_table_view_get(t)
                    ranges.append((v.first_query, v.end_query))
                    empty += v.npairs == 0
                    parts.append(hdb.hdb_table_copy_to_host(t))
                    hdb.hdb_table_free(t)
                finally:
                    hdb.hdb_ctx_destroy(ctx)
            assert empty >= 1
            assert ranges[0][0] == 0 and ranges[-1][1] == n
            assert all(ranges[i][1] == ranges[i + 1][0] for i in range(7))
            b, c, v = hdist.assemble(parts, n)
            assert_table_equal(xy, eps, b, c, v)


def test_sparse_batches_and_shards(torch_cuda):
    """The sparse queries of a group range follow the range: many small batches
    (host table) and process shards give the oracle's table."""
    xy = datagen.dense_skew(40_000, seed=9)
    P = int(oracle.eps_join(xy, 2.0)[0][-1])
    b, c, v, view, st = lib_table(xy, 2.0, batch_pairs=P // 40 + 1, n_streams=3)
    assert st["n_batches"] > 10 and st["n_sparse_queries"] > 0
    assert_table_equal(xy, 2.0, b, c, v)
    off, nbr = oracle.eps_join(xy, 2.0)
    want = np.diff(off.astype(np.int64))
    got = np.zeros(xy.shape[0], np.int64)
    for r in range(3):
        b, c, v, view, st = lib_table(xy, 2.0, device=True, shard_rank=r, shard_count=3)
        got += c.astype(np.int64)
    assert np.array_equal(got, want)


def test_c3_large_bucketed_row_scatter(torch_cuda):
    """5,000,000 points (C3L, SDSS2-size): the by-id row scatter takes the
    bucketed path (>= 2^22 rows) -- rows must tile the value array exactly and
    sampled rows equal the oracle's, device- and host-resident."""
    xy = datagen.sdss_like(datagen.C3_N_LARGE, seed=4)
    for device in (True, False):
        b, c, v, view, st = lib_table(xy, 0.07, device=device)
        order = np.argsort(b)
        bs, cs = b[order].astype(np.int64), c[order].astype(np.int64)
        assert bs[0] == 0 and np.array_equal(bs[1:], bs[:-1] + cs[:-1]) and bs[-1] + cs[-1] == view.npairs
        rng = np.random.default_rng(17)
        rows = np.unique(np.concatenate([rng.choice(xy.shape[0], 1000, replace=False), np.argsort(c)[-20:]]))
        roff, rnbr = oracle.eps_join_rows(xy, 0.07, rows)
        for i, p in enumerate(rows):
            assert np.array_equal(np.sort(v[b[p]:b[p] + c[p]]), rnbr[roff[i]:roff[i + 1]]), p


# ------------------------------------------------------------------ query-lane blocks (opt-in)
@pytest.fixture
def qlanes(monkeypatch):
    """HDB_QLANES=1: small groups take the query-per-lane single pass (k_qlanes)."""
    monkeypatch.setenv("HDB_QLANES", "1")


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_query_lane_blocks_heavy_and_ragged(torch_cuda, qlanes, dtype):
    """Small groups take the query-per-lane single pass (k_qlanes): blocks of up to
    32 queries of one cell row whose output overflows the kernel's shared output
    stage (uniform ~20 points per eps-cell: ~63 hits per query, ~2,000 ids per
    block -> several emission rounds), next to dense groups (a clump), isolated
    points (empty rows) and points on the grid's last row / column; the table is
    the oracle's, and with HDB_QLANES-style classification off (search_kernel 3:
    no split) the counts agree."""
    rng = np.random.default_rng(21)
    side = 1000 ** 0.5
    uni = rng.uniform(0.0, side, size=(20_000, 2))
    clump = rng.uniform(5.0, 5.5, size=(600, 2))
    lone = np.array([[side + 40.0, 3.0], [side + 40.0, side + 40.0], [-30.0, side + 40.0]])
    xy = np.concatenate([uni, clump, lone])
    x = xy.astype(np.float32) if dtype == "f32" else xy
    b, c, v, view, st = lib_table(x, 1.0, device=True)
    assert st["single_pass"] == 1 and 0 < st["n_sparse_queries"] < x.shape[0]
    assert_table_equal(x, 1.0, b, c, v, dtype)
    b3, c3, v3, _, st3 = lib_table(x, 1.0, device=True, search_kernel=3)
    assert st3["n_sparse_queries"] == 0
    assert np.array_equal(c3, c)


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_query_lane_blocks_workloads(torch_cuda, qlanes, dtype):
    """The query-lane single pass on the workload shapes (TEC bands, SDSS clumps,
    dense skew) at several eps -- block formation across cell rows, ragged blocks,
    dense groups next to small ones -- adversarial near-ties (the block-local f32
    filter's band replay) and exact lattice ties: every table is the oracle's."""
    cases = [(datagen.subsample(datagen.tec_like(), 30_000, seed=1), (0.15, 0.45)),
             (datagen.subsample(datagen.sdss_like(), 30_000, seed=2), (0.07, 0.2, 0.6)),
             (datagen.dense_skew(30_000, seed=7), (0.5, 4.0)),
             (datagen.near_ties(3_000, 0.35), (0.35,)),
             (datagen.lattice(60, spacing=0.25), (0.5, 0.75))]
    saw = False
    for xy, eps_list in cases:
        x = xy.astype(np.float32) if dtype == "f32" else xy
        for eps in eps_list:
            b, c, v, view, st = lib_table(x, eps, device=True)
            assert_table_equal(x, eps, b, c, v, dtype)
            saw |= st["n_sparse_queries"] > 0
    assert saw


def test_query_lane_blocks_in_shard_bands(torch_cuda, qlanes):
    """Process-shard bands with the query-lane split: each band's small queries
    are its share of the list (the kernel reads the range from the prefix), and
    the shards assemble into the oracle's table."""
    xy = datagen.dense_skew(40_000, seed=11)
    eps = 2.0
    off, nbr = oracle.eps_join(xy, eps)
    want = np.diff(off.astype(np.int64))
    got = np.zeros(xy.shape[0], np.int64)
    for r in range(3):
        b, c, v, view, st = lib_table(xy, eps, device=True, shard_rank=r, shard_count=3)
        got += c.astype(np.int64)
        rows = np.nonzero(c)[0]
        for p in rows[:: max(1, rows.size // 200)]:
            lst = np.sort(v[int(b[p]):int(b[p]) + int(c[p])])
            assert np.array_equal(lst, np.sort(nbr[int(off[p]):int(off[p + 1])]))
    assert np.array_equal(got, want)
