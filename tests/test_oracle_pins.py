"""Pins for the oracle (CPU only): each oracle function is checked against
something other than itself -- hand-worked fixtures from the paper's
definitions, closed forms, exact rational arithmetic, scipy/sklearn library
routines on tie-free data, and invariants.  A plausible mistake (dropped term,
wrong sign, '<' for '<=', FMA contraction, lost self-pair, Alg. 1 line-21
nesting) fails at least one test here.
"""
import json
import math
import os
from fractions import Fraction

import numpy as np
import pytest

import datagen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


# --------------------------------------------------------------------------
# exact IEEE rounding of rationals (independent of the oracle's arithmetic)
# --------------------------------------------------------------------------
def _round_rne(fr: Fraction, p: int) -> Fraction:
    """Round a rational to the nearest p-bit-significand binary float, ties to even."""
    if fr == 0:
        return Fraction(0)
    s = -1 if fr < 0 else 1
    a = abs(fr)
    e = a.numerator.bit_length() - a.denominator.bit_length()
    if Fraction(2) ** e > a:
        e -= 1
    while Fraction(2) ** (e + 1) <= a:
        e += 1
    scale = Fraction(2) ** (p - 1 - e)
    m = a * scale
    fl = m.numerator // m.denominator
    rem = m - fl
    if rem > Fraction(1, 2) or (rem == Fraction(1, 2) and fl % 2 == 1):
        fl += 1
    return s * Fraction(fl) / scale


def _ieee_pred(xp, yp, xq, yq, eps, p, fma=False):
    r = lambda v: _round_rne(v, p)
    X = [Fraction(v) for v in (xp, yp, xq, yq, eps)]
    dx = r(X[0] - X[2])
    dy = r(X[1] - X[3])
    e2 = r(X[4] * X[4])
    if fma:
        d2 = r(dx * dx + r(dy * dy))
    else:
        d2 = r(r(dx * dx) + r(dy * dy))
    return d2 <= e2


# --------------------------------------------------------------------------
# O1 -- predicate
# --------------------------------------------------------------------------
def test_predicate_inclusive_exact_tie():
    # dist = eps exactly representable: inclusive <=
    assert oracle.predicate((0.0, 0.0), (0.5, 0.0), 0.5)
    assert oracle.predicate((0.0, 0.0), (0.0, -0.5), 0.5)
    assert oracle.predicate((0.0, 0.0), (0.3, 0.4), 0.5) == (
        _ieee_pred(0.0, 0.0, 0.3, 0.4, 0.5, 53))
    assert not oracle.predicate((0.0, 0.0), (0.5000000000000001, 0.0), 0.5)
    assert oracle.predicate((0.0, 0.0), (0.5, 0.0), 0.5, dtype="f32")
    assert not oracle.predicate((0.0, 0.0), (0.50000006, 0.0), 0.5, dtype="f32")


def test_predicate_reflexive():
    rng = np.random.default_rng(0)
    for x, y in rng.uniform(-1e6, 1e6, (200, 2)):
        assert oracle.predicate((x, y), (x, y), 1e-300)
        assert oracle.predicate((x, y), (x, y), 1e-30, dtype="f32")


def test_predicate_decimal_near_tie_closed_form():
    # SURVEY 8(c) O1 pin: 0.3-0.2 = 0.09999999999999998, its square
    # 0.009999999999999995 <= fl(0.1^2) = 0.010000000000000002.
    assert 0.3 - 0.2 == 0.09999999999999998
    assert oracle.predicate((0.3, 0.0), (0.2, 0.0), 0.1)
    assert oracle.predicate((0.0, 0.3), (0.0, 0.2), 0.1)


@pytest.mark.parametrize("p,dtype", [(53, "f64"), (24, "f32")])
def test_predicate_matches_exact_ieee_rational(p, dtype):
    """Near-ties: the oracle equals the correctly rounded no-FMA evaluation
    computed in exact rational arithmetic; and at least one sampled case is
    FMA-sensitive, so a contracted build would fail here."""
    rng = np.random.default_rng(7 + p)
    npdt = np.float64 if dtype == "f64" else np.float32
    n_fma_sensitive = 0
    for _ in range(3000):
        eps = float(npdt(rng.uniform(0.05, 2.0)))
        ang = rng.uniform(0, 2 * np.pi)
        xp, yp = (float(npdt(v)) for v in rng.uniform(-200, 200, 2))
        xq = float(npdt(xp + eps * math.cos(ang)))
        yq = float(npdt(yp + eps * math.sin(ang)))
        want = _ieee_pred(xp, yp, xq, yq, eps, p)
        if want != _ieee_pred(xp, yp, xq, yq, eps, p, fma=True):
            n_fma_sensitive += 1
        assert oracle.predicate((xp, yp), (xq, yq), eps, dtype=dtype) == want
    assert n_fma_sensitive > 0


def test_predicate_far_from_tie_matches_real_distance():
    # away from ties the rounding cannot matter: compare with exact reals
    rng = np.random.default_rng(3)
    pts = rng.uniform(-50, 50, (2000, 4))
    for xp, yp, xq, yq in pts:
        eps = 10.0
        d2 = Fraction(xp - 0) * 0  # placeholder to keep Fraction imported
        d2 = (Fraction(xp) - Fraction(xq)) ** 2 + (Fraction(yp) - Fraction(yq)) ** 2
        if abs(d2 - 100) < Fraction(1, 10 ** 6):
            continue
        assert oracle.predicate((xp, yp), (xq, yq), eps) == (d2 <= 100)


# --------------------------------------------------------------------------
# O2 -- neighbour table
# --------------------------------------------------------------------------
def _counts(off):
    return np.diff(off.astype(np.int64))


def test_lattice_counts_eps1_and_sqrt2():
    g = _gold("lattice5.json")
    k = g["k"]
    xy = datagen.lattice(k)
    corner = {0, k - 1, k * (k - 1), k * k - 1}
    for key in ("eps1", "eps_sqrt2"):
        eps = g[key]["eps"]
        assert eps * eps == g[key].get("eps_sq", eps * eps)
        off, nbr = oracle.eps_join(xy, eps)
        c = _counts(off)
        for pid in range(k * k):
            iy, ix = divmod(pid, k)
            if pid in corner:
                want = g[key]["count_corner"]
            elif ix in (0, k - 1) or iy in (0, k - 1):
                want = g[key]["count_edge"]
            else:
                want = g[key]["count_interior"]
            assert c[pid] == want, (key, pid)


def test_join_lists_ascending_and_self_included():
    xy = datagen.uniform(800, (0, 0), (20, 20), seed=5)
    off, nbr = oracle.eps_join(xy, 0.9)
    for p in range(xy.shape[0]):
        lst = nbr[off[p]:off[p + 1]]
        assert np.all(np.diff(lst.astype(np.int64)) > 0)
        assert p in lst


def _tie_free(xy, eps, tol=1e-9):
    from scipy.spatial import cKDTree
    t = cKDTree(xy)
    a = t.query_pairs(eps * (1 + tol), output_type="ndarray")
    if a.size == 0:
        return True
    d = np.hypot(*(xy[a[:, 0]] - xy[a[:, 1]]).T)
    return not np.any(np.abs(d - eps) < eps * tol)


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_join_matches_ckdtree(dtype):
    from scipy.spatial import cKDTree
    xy = datagen.subsample(datagen.sdss_like(200_000, seed=3), 3000, seed=1)
    xy[:, 0] *= 0.2   # squeeze to get dense neighbourhoods
    if dtype == "f32":
        xy = xy.astype(np.float32).astype(np.float64)
    for eps in (0.05, 0.3, 1.1):
        assert _tie_free(xy, eps)
        off, nbr = oracle.eps_join(xy, eps, dtype=dtype)
        lists = cKDTree(xy).query_ball_point(xy, r=eps)
        for p in range(xy.shape[0]):
            assert sorted(lists[p]) == nbr[off[p]:off[p + 1]].tolist()


def test_join_matches_sklearn_radius_neighbors():
    from sklearn.neighbors import NearestNeighbors
    xy = datagen.subsample(datagen.tec_like(100_000, seed=2), 2000, seed=3)
    eps = 2.5
    assert _tie_free(xy, eps)
    off, nbr = oracle.eps_join(xy, eps)
    nn = NearestNeighbors(radius=eps, algorithm="brute").fit(xy)
    lists = nn.radius_neighbors(xy, return_distance=False)
    for p in range(xy.shape[0]):
        assert np.array_equal(np.sort(lists[p]), nbr[off[p]:off[p + 1]])


def test_join_invariants_symmetry_parity_monotone():
    xy = datagen.subsample(datagen.tec_like(200_000, seed=2), 1500, seed=2)
    prev = None
    for eps in (0.2, 0.5, 1.0, 3.0):
        off, nbr = oracle.eps_join(xy, eps)
        n = xy.shape[0]
        rows = np.repeat(np.arange(n), _counts(off))
        pairs = set(zip(rows.tolist(), nbr.tolist()))
        assert all((q, p) in pairs for p, q in pairs)            # symmetric
        assert all((p, p) in pairs for p in range(n))            # reflexive
        assert (len(pairs) - n) % 2 == 0                          # P - n even
        if prev is not None:
            assert prev <= pairs                                  # monotone in eps
        prev = pairs


def test_rows_and_rowhash_agree_with_full_table():
    xy = datagen.subsample(datagen.c1(), 1200, seed=4)
    eps = 3.0
    off, nbr = oracle.eps_join(xy, eps)
    rows = np.array([0, 5, 17, 1199, 600, 5])
    roff, rnbr = oracle.eps_join_rows(xy, eps, rows)
    for i, p in enumerate(rows):
        assert np.array_equal(rnbr[roff[i]:roff[i + 1]], nbr[off[p]:off[p + 1]])
    cnt, h = oracle.eps_join_rowhash(xy, eps, rows)
    # independent numpy SplitMix64 finaliser
    def mix(x):
        x = x.astype(np.uint64)
        with np.errstate(over="ignore"):
            z = x + np.uint64(0x9E3779B97F4A7C15)
            z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
            z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
            return z ^ (z >> np.uint64(31))
    for i, p in enumerate(rows):
        lst = nbr[off[p]:off[p + 1]]
        assert cnt[i] == lst.size
        with np.errstate(over="ignore"):
            assert h[i] == np.sum(mix(lst), dtype=np.uint64)


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_plane_sweep_equals_brute_force(dtype):
    """The R-tree-free scan the north star names: an x-sorted plane sweep (a
    different search order and pruning rule) must reproduce the brute-force
    rows exactly, including near-ties, duplicates and the lattice ties."""
    sets = [
        (datagen.uniform(3000, (0, 0), (30, 30), seed=21), 0.7),
        (datagen.subsample(datagen.tec_like(200_000, seed=2), 6000, seed=3), 0.45),
        (datagen.near_ties(2500, 0.45, seed=12, extent=40.0), 0.45),
        (datagen.lattice(9), 1.0),
        (datagen.lattice(9), math.sqrt(2.0)),
        (np.repeat(datagen.uniform(200, (0, 0), (5, 5), seed=4), 3, axis=0), 0.3),
    ]
    for xy, eps in sets:
        c0, h0 = oracle.eps_join_rowhash(xy, eps, dtype=dtype)
        c1, h1 = oracle.sweep_rowhash(xy, eps, dtype=dtype)
        np.testing.assert_array_equal(c0, c1)
        np.testing.assert_array_equal(h0, h1)
        c2, h2 = oracle.strip_rowhash(xy, eps, dtype=dtype)
        np.testing.assert_array_equal(c0, c2)
        np.testing.assert_array_equal(h0, h2)
        off0, nbr0 = oracle.eps_join(xy, eps, dtype=dtype)
        off1, nbr1 = oracle.strip_join(xy, eps, dtype=dtype)
        np.testing.assert_array_equal(off0, off1)
        np.testing.assert_array_equal(nbr0, nbr1)


@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_strip_sweep_equals_brute_force_on_strip_edges(dtype):
    """The strip sweep (the plane sweep inside horizontal strips of width ~2 eps,
    used for the 50M-point rows of C5) against brute force where the strips
    matter: neighbours straddling strip boundaries, points exactly on the
    boundaries y = ymin + t * 2 eps, a single column (one strip per point
    pair), a domain tall enough to cap the strip count, dense skew."""
    rng = np.random.default_rng(5)
    eps = 0.25
    on_edges = np.stack([rng.uniform(0, 6, 2000), np.floor(rng.uniform(0, 12, 2000)) * 2 * eps], 1)
    near_edges = on_edges + np.stack([np.zeros(2000), rng.choice([-1, 1], 2000) * rng.uniform(0, 1e-9, 2000)], 1)
    column = np.stack([np.full(1500, 3.0), np.sort(rng.uniform(0, 40, 1500))], 1)
    tall = np.stack([rng.uniform(0, 1, 1200), rng.uniform(-5e6, 5e6, 1200)], 1)
    tall[:600, 1] = rng.uniform(0, 2, 600)   # plus a dense patch
    sets = [(on_edges, eps), (near_edges, eps), (np.concatenate([on_edges, near_edges]), 2 * eps),
            (column, eps), (tall, 0.05), (datagen.dense_skew(20_000, seed=9), 4.0),
            (datagen.near_ties(2500, 0.45, seed=13, extent=20.0), 0.45)]
    for xy, e in sets:
        c0, h0 = oracle.eps_join_rowhash(xy, e, dtype=dtype)
        c1, h1 = oracle.strip_rowhash(xy, e, dtype=dtype)
        np.testing.assert_array_equal(c0, c1)
        np.testing.assert_array_equal(h0, h1)
        off0, nbr0 = oracle.eps_join(xy, e, dtype=dtype)
        off1, nbr1 = oracle.strip_join(xy, e, dtype=dtype)
        np.testing.assert_array_equal(off0, off1)
        np.testing.assert_array_equal(nbr0, nbr1)


@pytest.mark.parametrize("fn", ["sweep_rowhash", "strip_rowhash"])
def test_plane_sweep_lattice_golden(fn):
    g = _gold("lattice5.json")
    xy = datagen.lattice(g["k"])
    c, _ = getattr(oracle, fn)(xy, g["eps_sqrt2"]["eps"])
    assert sorted(set(c.tolist())) == sorted({g["eps_sqrt2"]["count_corner"], g["eps_sqrt2"]["count_edge"],
                                              g["eps_sqrt2"]["count_interior"]})
    assert int(c.sum()) == 4 * g["eps_sqrt2"]["count_corner"] + 12 * g["eps_sqrt2"]["count_edge"] \
        + 9 * g["eps_sqrt2"]["count_interior"]


def test_identical_points_give_n_squared():
    xy = np.tile([[1.25, -3.5]], (37, 1))
    off, nbr = oracle.eps_join(xy, 1e-9)
    assert int(off[-1]) == 37 * 37
    assert np.all(_counts(off) == 37)


def test_empty_and_single():
    off, nbr = oracle.eps_join(np.zeros((0, 2)), 1.0)
    assert off.tolist() == [0] and nbr.size == 0
    off, nbr = oracle.eps_join(np.array([[2.0, 3.0]]), 1.0)
    assert off.tolist() == [0, 1] and nbr.tolist() == [0]
    lab, core, k = oracle.dbscan(off, nbr, 1)
    assert lab.tolist() == [0] and core.tolist() == [1] and k == 1
    lab, core, k = oracle.dbscan(off, nbr, 2)
    assert lab.tolist() == [-1] and core.tolist() == [0] and k == 0
    lab, core, k = oracle.dbscan(np.zeros(1, np.uint64), np.zeros(0, np.uint32), 4)
    assert lab.size == 0 and k == 0


def test_c1_statistical_smoke():
    # Not a pin: C1 is Poisson rho=1, E[P] ~ n(1 + pi eps^2 rho) = 17,854 less edge loss.
    xy = datagen.c1()
    off, _ = oracle.eps_join(xy, 0.5)
    P = int(off[-1])
    assert 17_000 < P < 18_200


# --------------------------------------------------------------------------
# O3 -- DBSCAN (Algorithm 1 on T)
# --------------------------------------------------------------------------
def test_lattice_dbscan_core_border_noise():
    g = _gold("lattice5.json")
    xy = datagen.lattice(g["k"])
    off, nbr = oracle.eps_join(xy, 1.0)
    lab, core, k = oracle.dbscan(off, nbr, 5)
    w = g["eps1"]["minpts5"]
    assert int(core.sum()) == w["n_core"]
    assert int(((lab >= 0) & (core == 0)).sum()) == w["n_border"]
    assert int((lab < 0).sum()) == w["n_noise"]
    assert k == w["n_clusters"]


def test_shared_border_three_orders():
    g = _gold("border_orders.json")
    for o in g["orders"]:
        xy = np.stack([np.array(o["x"], float), np.zeros(len(o["x"]))], axis=1)
        off, nbr = oracle.eps_join(xy, g["eps"])
        lab, core, k = oracle.dbscan(off, nbr, g["minpts"])
        assert lab.tolist() == o["labels"]
        assert core.tolist() == o["core"]
        assert k == o["n_clusters"]


def test_minpts1_equals_connected_components():
    from scipy.sparse import csr_matrix
    from scipy.sparse.csgraph import connected_components
    xy = datagen.subsample(datagen.tec_like(100_000, seed=2), 2500, seed=9)
    for eps in (0.3, 0.8):
        off, nbr = oracle.eps_join(xy, eps)
        n = xy.shape[0]
        A = csr_matrix((np.ones(nbr.size), nbr.astype(np.int64), off.astype(np.int64)), shape=(n, n))
        ncc, cc = connected_components(A, directed=False)
        lab, core, k = oracle.dbscan(off, nbr, 1)
        assert k == ncc and np.all(core == 1) and np.all(lab >= 0)
        # same partition, and clusters numbered by increasing minimum id
        first = {}
        for p in range(n):
            first.setdefault(cc[p], len(first))
        assert np.array_equal(lab, np.array([first[c] for c in cc]))


@pytest.mark.parametrize("seed", range(6))
def test_dbscan_equals_sklearn(seed):
    from sklearn.cluster import DBSCAN
    base = datagen.sdss_like(150_000, seed=20 + seed)
    xy = datagen.subsample(base, 1800, seed=seed)
    xy[:, 0] *= 0.15
    xy[:, 1] *= 0.5
    for eps, minpts in ((0.4, 4), (0.8, 8), (0.25, 3)):
        assert _tie_free(xy, eps)
        off, nbr = oracle.eps_join(xy, eps)
        lab, core, k = oracle.dbscan(off, nbr, minpts)
        sk = DBSCAN(eps=eps, min_samples=minpts, algorithm="kd_tree").fit(xy)
        skcore = np.zeros(xy.shape[0], np.uint8)
        skcore[sk.core_sample_indices_] = 1
        assert np.array_equal(core, skcore)
        assert np.array_equal(lab, sk.labels_)
        assert k == (sk.labels_.max() + 1 if sk.labels_.size else 0)


def test_dbscan_degenerate_cases():
    xy = datagen.subsample(datagen.c1(), 500, seed=1)
    off, nbr = oracle.eps_join(xy, 2.0)
    # minpts above every count -> all noise
    lab, core, k = oracle.dbscan(off, nbr, int(np.diff(off.astype(np.int64)).max()) + 1)
    assert k == 0 and np.all(lab == -1) and core.sum() == 0
    # eps >= bbox diagonal -> one cluster of everything
    off, nbr = oracle.eps_join(xy, 200.0)
    lab, core, k = oracle.dbscan(off, nbr, 4)
    assert k == 1 and np.all(lab == 0) and np.all(core == 1)
    # identical points: all core iff n >= minpts
    same = np.tile([[5.0, 5.0]], (6, 1))
    off, nbr = oracle.eps_join(same, 0.1)
    assert oracle.dbscan(off, nbr, 6)[2] == 1
    lab, core, k = oracle.dbscan(off, nbr, 7)
    assert k == 0 and np.all(lab == -1)


def test_dbscan_invariants_monotone():
    xy = datagen.subsample(datagen.tec_like(100_000, seed=2), 2000, seed=5)
    cores = {}
    for eps in (0.3, 0.6):
        off, nbr = oracle.eps_join(xy, eps)
        for m in (4, 8):
            lab, core, k = oracle.dbscan(off, nbr, m)
            cores[(eps, m)] = core.astype(bool)
            noise = lab < 0
            # noise is exactly: non-core with no core neighbour
            cnt = np.diff(off.astype(np.int64))
            rows = np.repeat(np.arange(xy.shape[0]), cnt)
            has_core_nb = np.zeros(xy.shape[0], bool)
            np.logical_or.at(has_core_nb, rows, core[nbr].astype(bool))
            assert np.array_equal(noise, ~has_core_nb)
    assert np.all(cores[(0.3, 4)] <= cores[(0.6, 4)])   # grows with eps
    assert np.all(cores[(0.3, 8)] <= cores[(0.3, 4)])   # shrinks with minpts
