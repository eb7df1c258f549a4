"""CPU pin of the test helper tests/_rowhash.py (the library-side row hash of
the full-size parity tests): its mix64 equals an independent numpy SplitMix64
finaliser, and its per-row (count, hash) of a table read through the C-ABI's
table view equals the oracle's eps_join_rowhash -- with rows placed out of
order and batched, as the library's device tables are."""
import numpy as np
import torch

import datagen
import oracle
from paper_conf_ipps_gowanlockrblp17_b200 import hdb
import _rowhash


def _np_mix(x):
    x = x.astype(np.uint64)
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def test_mix64_torch_equals_numpy():
    v = np.concatenate([np.array([0, 1, 2**31, 2**32 - 1], np.uint64),
                        np.random.default_rng(1).integers(0, 2**32, 5000, dtype=np.uint64)])
    got = _rowhash.mix64(torch, torch.from_numpy(v.astype(np.int64))).numpy().view(np.uint64)
    np.testing.assert_array_equal(got, _np_mix(v))


def test_table_rowhash_through_view_equals_oracle():
    xy = datagen.subsample(datagen.tec_like(), 3000, seed=5)
    eps = 0.9
    off, nbr = oracle.eps_join(xy, eps)
    n = xy.shape[0]
    cnt = np.diff(off).astype(np.uint32)
    # rows stored in a shuffled order with gaps (as a device table's reservation order)
    perm = np.random.default_rng(2).permutation(n)
    begin = np.zeros(n, np.uint64)
    vals = []
    pos = 0
    for p in perm:
        lst = nbr[off[p]:off[p + 1]][::-1]          # list order is free
        begin[p] = pos
        vals.append(lst)
        vals.append(np.zeros(3, np.uint32))   # padding between rows (not part of any row)
        pos += lst.size + 3
    t = hdb.hdb_table_from_host(begin, cnt, np.concatenate(vals))
    try:
        view = hdb.hdb_table_view_get(t)
        b, c, v = _rowhash.view_tensors(torch, view)
        got_c, got_h = _rowhash.table_rowhash(torch, b, c, v, max_entries=5000)
    finally:
        hdb.hdb_table_free(t)
    want_c, want_h = oracle.eps_join_rowhash(xy, eps)
    np.testing.assert_array_equal(got_c, want_c)
    np.testing.assert_array_equal(got_h, want_h)
