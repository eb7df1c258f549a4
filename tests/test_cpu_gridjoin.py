"""The CPU grid-join comparator (cpu_baseline/, timed by bench.py beside the
GPU path) must compute the same table as the oracle, so that its pairs/s is a
like-for-like number."""
import math

import numpy as np
import pytest

import cpu_baseline
import datagen
import oracle


def _same_table(xy, eps, dtype, rows=None):
    off, nbr = cpu_baseline.gridjoin_rows(xy, eps, rows, dtype=dtype)
    o2, n2 = oracle.eps_join_rows(xy, eps, rows, dtype=dtype)
    np.testing.assert_array_equal(off, o2)
    for r in range(off.shape[0] - 1):
        np.testing.assert_array_equal(np.sort(nbr[off[r]:off[r + 1]]), n2[o2[r]:o2[r + 1]])


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_gridjoin_equals_oracle(dtype):
    _same_table(datagen.uniform(3000, (0, 0), (30, 30), seed=21), 0.7, dtype)
    _same_table(datagen.near_ties(2500, 0.45, seed=12, extent=40.0), 0.45, dtype)
    _same_table(datagen.lattice(9), math.sqrt(2.0), dtype)
    _same_table(datagen.lattice(9), 1.0, dtype)


def test_gridjoin_sampled_rows_clustered():
    xy = datagen.tec_like(200_000, seed=2)
    rows = np.linspace(0, xy.shape[0] - 1, 300).astype(np.int64)
    _same_table(xy, 0.45, "f64", rows)


def test_gridjoin_edge_cases():
    off, nbr = cpu_baseline.gridjoin_rows(np.zeros((0, 2)), 0.5)
    assert off.tolist() == [0] and nbr.size == 0
    off, nbr = cpu_baseline.gridjoin_rows(np.array([[1.0, 2.0]]), 0.5)
    assert off.tolist() == [0, 1] and nbr.tolist() == [0]
    same = np.ones((50, 2))
    off, _ = cpu_baseline.gridjoin_rows(same, 0.1, threads=4)
    assert int(off[-1]) == 2500


def test_gridjoin_threads_same_output():
    xy = datagen.uniform(5000, (0, 0), (40, 40), seed=9)
    a = cpu_baseline.gridjoin_rows(xy, 0.8, threads=1)
    b = cpu_baseline.gridjoin_rows(xy, 0.8, threads=4)
    np.testing.assert_array_equal(a[0], b[0])
    np.testing.assert_array_equal(a[1], b[1])
