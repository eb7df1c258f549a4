"""Seeded synthetic inputs shaped like the paper's workloads.

This module holds NONE of the method's arithmetic: it only draws 2-D points.
It is the one module shared by the oracle side (tests) and the CUDA side
(tests, bench.py, smoke); see DESIGN.md "Input recipe".

The real datasets (SW1/SW4 ionospheric TEC, SDSS DR12 galaxies; P:826-841,
Sec. VII-A) are not available, so each config is a calibrated stand-in
(SURVEY.md 8(d)):

* C1 -- n=10,000 uniform in [0,100)^2 (seed 1), eps=0.5, minpts=4.
* C2 -- TEC-like, n=1,864,620 (SW1's size), lon in [-180,180),
  lat clipped to [-90,90] (seed 2): 60% two receiver-network latitude bands,
  38% Pareto-weighted hotspots, 2% global background ("many overdense
  regions").
* C3 -- SDSS-like, n=2,000,000 (seed 3) or 5,000,000 (seed 4) in
  [0,250)x[0,70): 85% uniform + 15% Neyman-Scott clumps ("more uniformly
  distributed").
* C5 -- dense-skew, n=50,000,000 in [0,1000)^2: 45M uniform + 5M uniform in
  [450,550)^2 (seed 5).

All generators return a C-contiguous float64 array of shape (n, 2) holding
interleaved (x, y) rows.  Deterministic: numpy PCG64 with the fixed seed.
"""
from __future__ import annotations

import numpy as np

C2_N = 1_864_620
C3_N_SMALL = 2_000_000
C3_N_LARGE = 5_000_000
C5_N = 50_000_000

C1_EPS = 0.5
C2_EPS = (0.15, 0.45, 1.40)
C3_EPS = (0.07, 0.12, 0.20)
C4_EPS = (0.15, 0.20, 0.30, 0.45, 0.60, 0.80, 1.00, 1.40)
C4_MINPTS = (4, 8, 16)
C5_EPS = (0.5, 1.0)
MINPTS = 4


def _rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def uniform(n: int, lo=(0.0, 0.0), hi=(100.0, 100.0), seed: int = 1) -> np.ndarray:
    rng = _rng(seed)
    out = np.empty((n, 2), dtype=np.float64)
    out[:, 0] = rng.uniform(lo[0], hi[0], n)
    out[:, 1] = rng.uniform(lo[1], hi[1], n)
    return out


def c1(seed: int = 1) -> np.ndarray:
    """C1: 10,000 uniform points in [0,100)^2."""
    return uniform(10_000, (0.0, 0.0), (100.0, 100.0), seed)


def _band_points(rng, m):
    """m points from the two receiver-network bands, split equally."""
    out = np.empty((m, 2))
    na = rng.random(m) < 0.5
    k = int(na.sum())
    out[na, 0] = rng.uniform(-130.0, -60.0, k)
    out[na, 1] = rng.normal(40.0, 7.0, k)
    out[~na, 0] = rng.uniform(-15.0, 45.0, m - k)
    out[~na, 1] = rng.normal(50.0, 6.0, m - k)
    return out


def tec_like(n: int = C2_N, seed: int = 2, n_sites: int = 2000) -> np.ndarray:
    """C2: TEC-like lon/lat set (banded density with Pareto hotspots)."""
    rng = _rng(seed)
    n_band = int(round(0.60 * n))
    n_hot = int(round(0.38 * n))
    n_bg = n - n_band - n_hot
    band = _band_points(rng, n_band)
    sites = _band_points(rng, n_sites)
    w = (1.0 - rng.random(n_sites)) ** (-1.0 / 1.5)     # Pareto shape 1.5
    w /= w.sum()
    site_of = rng.choice(n_sites, size=n_hot, p=w)
    hot = sites[site_of] + rng.normal(0.0, 0.3, (n_hot, 2))
    bg = np.empty((n_bg, 2))
    bg[:, 0] = rng.uniform(-180.0, 180.0, n_bg)
    bg[:, 1] = rng.uniform(-60.0, 75.0, n_bg)
    pts = np.concatenate([band, hot, bg], axis=0)
    pts[:, 1] = np.clip(pts[:, 1], -90.0, 90.0)
    # longitudes stay inside [-180, 180): sites lie in [-130, 45]; wrap defensively
    pts[:, 0] = (pts[:, 0] + 180.0) % 360.0 - 180.0
    perm = rng.permutation(n)
    return np.ascontiguousarray(pts[perm])


def sdss_like(n: int = C3_N_SMALL, seed: int = 3, width: float = 250.0,
              height: float = 70.0) -> np.ndarray:
    """C3: SDSS-like footprint: 85% uniform + 15% Neyman-Scott clumps."""
    rng = _rng(seed)
    n_clump = int(round(0.15 * n))
    n_uni = n - n_clump
    uni = np.empty((n_uni, 2))
    uni[:, 0] = rng.uniform(0.0, width, n_uni)
    uni[:, 1] = rng.uniform(0.0, height, n_uni)
    got = []
    have = 0
    while have < n_clump:
        n_par = max(1024, (n_clump - have) // 8)
        par = np.empty((n_par, 2))
        par[:, 0] = rng.uniform(0.0, width, n_par)
        par[:, 1] = rng.uniform(0.0, height, n_par)
        members = np.floor(5.0 * (1.0 - rng.random(n_par)) ** (-1.0 / 1.5)).astype(np.int64)
        sigma = rng.uniform(0.02, 0.3, n_par)
        idx = np.repeat(np.arange(n_par), members)
        pts = par[idx] + rng.normal(0.0, 1.0, (idx.size, 2)) * sigma[idx, None]
        keep = (pts[:, 0] >= 0.0) & (pts[:, 0] < width) & (pts[:, 1] >= 0.0) & (pts[:, 1] < height)
        pts = pts[keep]      # resample the clipped points: draw more clumps
        got.append(pts)
        have += pts.shape[0]
    clump = np.concatenate(got, axis=0)[:n_clump]
    pts = np.concatenate([uni, clump], axis=0)
    perm = rng.permutation(n)
    return np.ascontiguousarray(pts[perm])


def dense_skew(n: int = C5_N, seed: int = 5, dense_frac: float = 0.10) -> np.ndarray:
    """C5: 90% uniform over [0,1000)^2 + 10% uniform in [450,550)^2."""
    rng = _rng(seed)
    nd = int(round(dense_frac * n))
    ns = n - nd
    out = np.empty((n, 2), dtype=np.float64)
    out[:ns, 0] = rng.uniform(0.0, 1000.0, ns)
    out[:ns, 1] = rng.uniform(0.0, 1000.0, ns)
    out[ns:, 0] = rng.uniform(450.0, 550.0, nd)
    out[ns:, 1] = rng.uniform(450.0, 550.0, nd)
    perm = rng.permutation(n)
    return np.ascontiguousarray(out[perm])


def subsample(xy: np.ndarray, m: int, seed: int = 0) -> np.ndarray:
    """A seeded random subset of m rows (keeps the spatial structure)."""
    rng = _rng(seed)
    idx = np.sort(rng.choice(xy.shape[0], size=m, replace=False))
    return np.ascontiguousarray(xy[idx])


def lattice(k: int, spacing: float = 1.0, origin=(0.0, 0.0)) -> np.ndarray:
    """k x k lattice, row-major: point id = iy*k + ix."""
    iy, ix = np.divmod(np.arange(k * k), k)
    return np.ascontiguousarray(np.stack([origin[0] + ix * spacing, origin[1] + iy * spacing], axis=1),
                                dtype=np.float64)


def giants(seed: int = 5, bridge: bool = False) -> np.ndarray:
    """Two dense squares (12,000 and 9,000 points; the giant components of the
    union-find pre-pass) + 2,000 background points, optionally joined by a
    thin chain of points (spacing 0.2) -- test input for the DBSCAN skip rules."""
    rng = _rng(seed)
    a = rng.uniform((0, 0), (10, 10), size=(12_000, 2))
    b = rng.uniform((20, 0), (30, 10), size=(9_000, 2))
    c = rng.uniform((-5, -5), (35, 15), size=(2_000, 2))
    parts = [a, b, c]
    if bridge:
        x = np.arange(10.0, 20.0001, 0.2)
        parts.append(np.stack([x, np.full_like(x, 5.0)], axis=1))
    xy = np.concatenate(parts)
    return xy[rng.permutation(xy.shape[0])]


def near_ties(m: int, eps: float, seed: int = 11, extent: float = 400.0) -> np.ndarray:
    """Adversarial near-tie set: pairs of points whose distance is eps up to
    a few ulps, at random offsets inside a large extent so that cell
    boundaries fall between them (stress for the grid's cell width)."""
    rng = _rng(seed)
    base = rng.uniform(-extent / 2, extent / 2, (m, 2))
    ang = rng.uniform(0.0, 2 * np.pi, m)
    jitter = 1.0 + rng.integers(-4, 5, m) * np.finfo(np.float64).eps
    other = base + np.stack([np.cos(ang), np.sin(ang)], axis=1) * (eps * jitter)[:, None]
    axis = rng.random(m) < 0.3          # also exactly axis-aligned pairs
    other[axis, 0] = base[axis, 0] + eps * jitter[axis]
    other[axis, 1] = base[axis, 1]
    out = np.empty((2 * m, 2))
    out[0::2] = base
    out[1::2] = other
    return np.ascontiguousarray(out)


CONFIGS = {
    "C1": dict(gen=c1, eps=(C1_EPS,), minpts=(MINPTS,)),
    "C2": dict(gen=tec_like, eps=C2_EPS, minpts=(MINPTS,)),
    "C3": dict(gen=sdss_like, eps=C3_EPS, minpts=(MINPTS,)),
    "C3L": dict(gen=lambda: sdss_like(C3_N_LARGE, seed=4), eps=C3_EPS, minpts=(MINPTS,)),
    "C4": dict(gen=tec_like, eps=C4_EPS, minpts=C4_MINPTS),
    "C5": dict(gen=dense_skew, eps=C5_EPS, minpts=(MINPTS,)),
}
