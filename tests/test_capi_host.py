"""CPU-only tests of the C-ABI library: it loads, exports every symbol the
header declares, and its host-side logic (Sec. VI planning helpers, host
DBSCAN on a table, canonicalisation, validation) is correct.  No GPU compute."""
import json
import os
import re

import numpy as np
import pytest

import datagen
import oracle
from paper_conf_ipps_gowanlockrblp17_b200 import hdb

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLD = os.path.join(ROOT, "tests", "golden")


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def test_header_symbols_exported():
    with open(os.path.join(ROOT, "include", "hdb.h")) as f:
        src = f.read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    declared = set(re.findall(r"\b(hdb_[a-z0-9_]+)\s*\(", src))
    assert len(declared) >= 20
    for name in sorted(declared):
        assert hasattr(hdb.lib, name), f"{name} declared in hdb.h but not exported"
    assert declared == set(hdb.EXPORTED), declared ^ set(hdb.EXPORTED)


def test_version_and_struct_sizes():
    assert "sm_100a" in hdb.hdb_version()
    o = hdb.hdb_opts_default()
    assert o.sample_fraction == 0.01 and o.alpha == 0.05 and o.n_streams == 3


def test_eq1_and_buffer_rule_golden():
    g = _gold("eq1_buffer.json")
    for c in g["cases"]:
        bb, nb = hdb.hdb_plan_batches(c["a_b"], g["alpha"], 3)
        assert nb == c["n_b"], c
        if "b_b" in c:
            assert bb == pytest.approx(c["b_b"], rel=1e-12)


def test_fig2_strided_assignment_golden():
    g = _gold("fig2_batches.json")
    nb = g["n_b"]
    for p1, b1, gid in zip(g["point_1based"], g["batch_1based"], g["gid"]):
        assert hdb.hdb_strided_point(gid, b1 - 1, nb) == p1 - 1


def test_balanced_cuts():
    w = np.array([5, 1, 1, 1, 10, 1, 1, 1, 1, 1], np.uint64)
    pre = np.concatenate([[0], np.cumsum(w)]).astype(np.uint64)
    for parts in (1, 2, 3, 7, 10, 15):
        cuts = hdb.hdb_balanced_cuts(pre, parts)
        assert cuts[0] == 0 and cuts[-1] == w.size
        assert np.all(np.diff(cuts.astype(np.int64)) >= 0)
    cuts = hdb.hdb_balanced_cuts(pre, 2)
    # total 23, half 11.5 -> cut at the first prefix >= 11 (before item 4)
    assert cuts.tolist() == [0, 4, 10]


def _lib_table(off, nbr, seed=0):
    """library table from a CSR, with rows stored in a shuffled order so that
    begin[] indirection is exercised."""
    n = off.size - 1
    cnt = np.diff(off.astype(np.int64)).astype(np.uint32)
    order = np.random.default_rng(seed).permutation(n)
    begin = np.empty(n, np.uint64)
    parts = []
    pos = 0
    for p in order:
        begin[p] = pos
        lst = nbr[off[p]:off[p + 1]][::-1]   # reversed: lists need not be sorted
        parts.append(lst)
        pos += lst.size
    flat = np.concatenate(parts) if parts else np.zeros(0, np.uint32)
    return hdb.hdb_table_from_host(begin, cnt, flat)


@pytest.mark.parametrize("threads", [1, 4])
def test_host_dbscan_matches_oracle(threads):
    cases = [(datagen.subsample(datagen.tec_like(200_000, seed=2), 6000, seed=s), eps, m)
             for s, eps, m in ((1, 0.4, 4), (2, 0.8, 8), (3, 0.25, 3))]
    cases.append((datagen.lattice(9), 1.0, 5))
    cases.append((datagen.uniform(5000, (0, 0), (30, 30), seed=9), 0.6, 1))
    for xy, eps, minpts in cases:
        off, nbr = oracle.eps_join(xy, eps)
        want_lab, want_core, want_k = oracle.dbscan(off, nbr, minpts)
        t = _lib_table(off, nbr)
        try:
            lab, core, k = hdb.hdb_dbscan(t, minpts, n_threads=threads)
        finally:
            hdb.hdb_table_free(t)
        assert k == want_k
        assert np.array_equal(core, want_core)
        assert np.array_equal(lab, want_lab)


@pytest.mark.parametrize("bridge", [False, True])
def test_host_dbscan_giant_components(bridge):
    """Exercises the parallel host DBSCAN's giant-component skip rule (two dense
    squares -> giants A and B; optional bridge -> A-B edges through other rows)."""
    xy = datagen.giants(5, bridge)
    for eps, minpts in ((0.25, 4), (0.25, 12), (0.5, 30)):
        off, nbr = oracle.eps_join(xy, eps)
        want = oracle.dbscan(off, nbr, minpts)
        t = _lib_table(off, nbr)
        try:
            for threads in (4, 16):
                lab, core, k = hdb.hdb_dbscan(t, minpts, n_threads=threads)
                assert k == want[2]
                assert np.array_equal(core, want[1])
                assert np.array_equal(lab, want[0])
        finally:
            hdb.hdb_table_free(t)


def test_host_dbscan_shared_border_golden():
    g = _gold("border_orders.json")
    for o in g["orders"]:
        xy = np.stack([np.array(o["x"], float), np.zeros(len(o["x"]))], axis=1)
        off, nbr = oracle.eps_join(xy, g["eps"])
        for threads in (1, 3):
            t = _lib_table(off, nbr, seed=threads)
            lab, core, k = hdb.hdb_dbscan(t, g["minpts"], n_threads=threads)
            hdb.hdb_table_free(t)
            assert lab.tolist() == o["labels"] and core.tolist() == o["core"] and k == o["n_clusters"]


def test_parallel_dbscan_large_equals_sequential():
    xy = datagen.subsample(datagen.sdss_like(400_000, seed=3), 60_000, seed=1)
    off, nbr = oracle.eps_join(xy, 0.25)
    t = _lib_table(off, nbr)
    a = hdb.hdb_dbscan(t, 4, n_threads=1)
    b = hdb.hdb_dbscan(t, 4, n_threads=8)
    hdb.hdb_table_free(t)
    assert a[2] == b[2] and np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])


def test_canonicalize_host_table():
    xy = datagen.subsample(datagen.c1(), 2000, seed=2)
    off, nbr = oracle.eps_join(xy, 2.0)
    t = _lib_table(off, nbr, seed=5)
    hdb.hdb_table_canonicalize(t)
    b, c, v = hdb.hdb_table_copy_to_host(t)
    hdb.hdb_table_free(t)
    assert np.array_equal(b, off[:-1]) and np.array_equal(v, nbr)
    assert np.array_equal(c.astype(np.uint64), np.diff(off))


def test_validation_errors():
    t = hdb.hdb_table_from_host(np.zeros(1, np.uint64), np.ones(1, np.uint32), np.zeros(1, np.uint32))
    with pytest.raises(hdb.HdbError) as e:
        hdb.hdb_dbscan(t, 0)
    assert e.value.status == hdb.HDB_EINVAL
    hdb.hdb_table_free(t)
    with pytest.raises(hdb.HdbError) as e:   # row outside nbrs
        hdb.hdb_table_from_host(np.array([1], np.uint64), np.array([1], np.uint32), np.zeros(1, np.uint32))
    assert e.value.status == hdb.HDB_EINVAL
    with pytest.raises(hdb.HdbError) as e:   # id >= n
        hdb.hdb_table_from_host(np.array([0], np.uint64), np.array([1], np.uint32), np.array([3], np.uint32))
    assert e.value.status == hdb.HDB_EINVAL
    with pytest.raises(hdb.HdbError):
        hdb.hdb_plan_batches(-1.0, 0.05, 3)


def test_empty_table_dbscan():
    t = hdb.hdb_table_from_host(np.zeros(0, np.uint64), np.zeros(0, np.uint32), np.zeros(0, np.uint32))
    lab, core, k = hdb.hdb_dbscan(t, 4)
    hdb.hdb_table_free(t)
    assert lab.size == 0 and k == 0


def test_ctx_create_without_gpu_fails_loudly():
    from conftest import cuda_available
    if cuda_available():
        pytest.skip("GPU present")
    with pytest.raises(hdb.HdbError) as e:
        hdb.hdb_ctx_create()
    assert e.value.status == hdb.HDB_ECUDA


@pytest.mark.parametrize("bad", [dict(sweep_on_device=2), dict(cell_split=9), dict(cell_split=7), dict(n_streams=0),
                                 dict(sample_fraction=0.0), dict(alpha=-1.0), dict(shard_count=2, shard_rank=2)])
def test_opts_validation_before_device(bad):
    """Option errors are reported as HDB_EINVAL before any device is touched."""
    with pytest.raises(hdb.HdbError) as e:
        hdb.hdb_ctx_create(**bad)
    assert e.value.status == hdb.HDB_EINVAL
