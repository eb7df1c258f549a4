"""Oracle -- TEST INFRASTRUCTURE ONLY (see oracle/oracle.c header).

Plain CPU implementation of what the HYBRID-DBSCAN hot path computes
(Gowanlock et al., IPDPSW 2017; PAPER.md cited as P:n):

* ``predicate``       -- O1, dist(p,q) <= eps, exact no-FMA arithmetic.
* ``eps_join``        -- O2, the neighbour table T by brute force.
* ``eps_join_rows``   -- O2 restricted to sampled query rows (each vs all n).
* ``eps_join_rowhash``-- O2 streamed as per-row (count, order-free hash).
* ``sweep_rowhash``   -- O2 by an x-sorted plane sweep (the R-tree-free scan).
* ``strip_rowhash``   -- the same sweep inside horizontal strips (50M points).
* ``strip_join``      -- O2 as a full CSR table by the strip sweep.
* ``dbscan``          -- O3, Algorithm 1 on T.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  It shares no code with the
CUDA path and never imports it.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
# -ffp-contract=off is part of the arithmetic contract (O1): gcc would
# otherwise fuse dx*dx+dy*dy into an FMA.  No -ffast-math.
CFLAGS = ["-O3", "-march=x86-64-v3", "-ffp-contract=off", "-fno-fast-math",
          "-DORACLE_FP_CONTRACT_OFF", "-fopenmp", "-fPIC", "-shared", "-std=c11",
          "-Wall", "-Wextra"]

_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so (gcc) if missing or stale; return its path."""
    if (not force and os.path.exists(_LIB)
            and os.path.getmtime(_LIB) >= os.path.getmtime(_SRC)):
        return _LIB
    tmp = _LIB + f".tmp{os.getpid()}"
    subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp])
    os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        i64, u64, d, f = ctypes.c_int64, ctypes.c_uint64, ctypes.c_double, ctypes.c_float
        lib.oracle_predicate_f64.argtypes = [d, d, d, d, d]
        lib.oracle_predicate_f64.restype = ctypes.c_int
        lib.oracle_predicate_f32.argtypes = [f, f, f, f, f]
        lib.oracle_predicate_f32.restype = ctypes.c_int
        lib.oracle_threads.restype = ctypes.c_int
        for t, et in (("f64", d), ("f32", f)):
            getattr(lib, f"oracle_join_count_{t}").argtypes = [P, i64, et, P, i64, P]
            getattr(lib, f"oracle_join_fill_{t}").argtypes = [P, i64, et, P, i64, P, P]
            getattr(lib, f"oracle_join_rowhash_{t}").argtypes = [P, i64, et, P, i64, P, P]
            getattr(lib, f"oracle_sweep_rowhash_{t}").argtypes = [P, i64, et, P, P]
            getattr(lib, f"oracle_sweep_rowhash_{t}").restype = ctypes.c_int
            getattr(lib, f"oracle_strip_rowhash_{t}").argtypes = [P, i64, et, P, P]
            getattr(lib, f"oracle_strip_rowhash_{t}").restype = ctypes.c_int
            getattr(lib, f"oracle_strip_join_{t}").argtypes = [P, i64, et, P, P]
            getattr(lib, f"oracle_strip_join_{t}").restype = ctypes.c_int
        lib.oracle_dbscan.argtypes = [P, P, i64, u64, P, P]
        lib.oracle_dbscan.restype = i64
        _lib = lib
        return lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _prep(xy, dtype):
    if dtype not in ("f64", "f32"):
        raise ValueError(f"dtype must be 'f64' or 'f32', got {dtype!r}")
    npdt = np.float64 if dtype == "f64" else np.float32
    xy = np.ascontiguousarray(xy, dtype=npdt).reshape(-1, 2)
    return xy, npdt


def threads() -> int:
    """OpenMP threads the oracle's join loops use."""
    return int(_load().oracle_threads())


def predicate(p, q, eps, dtype="f64") -> bool:
    """O1: q in N_eps(p) in the given precision, no FMA."""
    lib = _load()
    if dtype == "f64":
        return bool(lib.oracle_predicate_f64(float(p[0]), float(p[1]), float(q[0]), float(q[1]), float(eps)))
    e = float(np.float32(eps))
    return bool(lib.oracle_predicate_f32(float(np.float32(p[0])), float(np.float32(p[1])),
                                         float(np.float32(q[0])), float(np.float32(q[1])), e))


def eps_join_rows(xy, eps, rows=None, dtype="f64"):
    """O2 for the query rows ``rows`` (None = all): CSR (off[len+1], nbr) with
    each row's list ascending and including the row itself."""
    lib = _load()
    xy, npdt = _prep(xy, dtype)
    n = xy.shape[0]
    if rows is None:
        nrows, rptr = n, None
    else:
        rows = np.ascontiguousarray(rows, dtype=np.int64)
        nrows, rptr = rows.shape[0], rows
    cnt = np.zeros(nrows, dtype=np.uint64)
    e = float(npdt(eps))
    getattr(lib, f"oracle_join_count_{dtype}")(_ptr(xy), n, e, _ptr(rptr), nrows, _ptr(cnt))
    off = np.zeros(nrows + 1, dtype=np.uint64)
    np.cumsum(cnt, out=off[1:])
    nbr = np.empty(int(off[-1]), dtype=np.uint32)
    getattr(lib, f"oracle_join_fill_{dtype}")(_ptr(xy), n, e, _ptr(rptr), nrows, _ptr(off), _ptr(nbr))
    return off, nbr


def eps_join(xy, eps, dtype="f64"):
    """O2: the full neighbour table T of all n points (brute force, n^2 tests)."""
    return eps_join_rows(xy, eps, None, dtype)


def eps_join_rowhash(xy, eps, rows=None, dtype="f64"):
    """Per-row (count, sum of mix64(q) mod 2^64) of N_eps(row), streamed."""
    lib = _load()
    xy, npdt = _prep(xy, dtype)
    n = xy.shape[0]
    if rows is None:
        nrows, rptr = n, None
    else:
        rows = np.ascontiguousarray(rows, dtype=np.int64)
        nrows, rptr = rows.shape[0], rows
    cnt = np.zeros(nrows, dtype=np.uint64)
    h = np.zeros(nrows, dtype=np.uint64)
    getattr(lib, f"oracle_join_rowhash_{dtype}")(_ptr(xy), n, float(npdt(eps)), _ptr(rptr), nrows,
                                                 _ptr(cnt), _ptr(h))
    return cnt, h


def sweep_rowhash(xy, eps, dtype="f64"):
    """O2 by the x-sorted plane sweep (no cells): per-row (count, hash) for all
    rows, equal to ``eps_join_rowhash`` by construction (see oracle.c)."""
    lib = _load()
    xy, npdt = _prep(xy, dtype)
    n = xy.shape[0]
    cnt = np.zeros(n, dtype=np.uint64)
    h = np.zeros(n, dtype=np.uint64)
    if getattr(lib, f"oracle_sweep_rowhash_{dtype}")(_ptr(xy), n, float(npdt(eps)), _ptr(cnt), _ptr(h)) != 0:
        raise MemoryError("oracle_sweep_rowhash: allocation failed")
    return cnt, h


def strip_rowhash(xy, eps, dtype="f64"):
    """O2 by the plane sweep inside horizontal strips of width ~2 eps (the
    scale-out of ``sweep_rowhash`` for 50M points): per-row (count, hash) for
    all rows, equal to ``sweep_rowhash`` / ``eps_join_rowhash`` (see oracle.c
    for the exactness argument; the strip widths are checked at run time)."""
    lib = _load()
    xy, npdt = _prep(xy, dtype)
    n = xy.shape[0]
    cnt = np.zeros(n, dtype=np.uint64)
    h = np.zeros(n, dtype=np.uint64)
    rc = getattr(lib, f"oracle_strip_rowhash_{dtype}")(_ptr(xy), n, float(npdt(eps)), _ptr(cnt), _ptr(h))
    if rc == -1:
        raise MemoryError("oracle_strip_rowhash: allocation failed")
    if rc != 0:
        raise ValueError("oracle_strip_rowhash: a strip is not wider than eps (exactness check failed)")
    return cnt, h


def strip_join(xy, eps, dtype="f64"):
    """O2 as a full CSR table (off[n+1], nbr) with ascending lists, built by the
    strip sweep -- equal to ``eps_join`` (pinned), in seconds at millions of
    points (the full-size DBSCAN partitions of the GPU parity tests)."""
    lib = _load()
    xy, npdt = _prep(xy, dtype)
    n = xy.shape[0]
    off = np.zeros(n + 1, dtype=np.uint64)
    fn = getattr(lib, f"oracle_strip_join_{dtype}")
    e = float(npdt(eps))
    for rc in (fn(_ptr(xy), n, e, _ptr(off), None),):
        if rc == -1:
            raise MemoryError("oracle_strip_join: allocation failed")
        if rc != 0:
            raise ValueError("oracle_strip_join: a strip is not wider than eps")
    nbr = np.empty(int(off[-1]), dtype=np.uint32)
    rc = fn(_ptr(xy), n, e, _ptr(off), _ptr(nbr) if nbr.size else _ptr(np.empty(1, np.uint32)))
    if rc != 0:
        raise MemoryError("oracle_strip_join: fill pass failed")
    return off, nbr


def dbscan(off, nbr, minpts):
    """O3: Algorithm 1 on T.  Returns (labels int32[n], is_core uint8[n], n_clusters)."""
    lib = _load()
    off = np.ascontiguousarray(off, dtype=np.uint64)
    nbr = np.ascontiguousarray(nbr, dtype=np.uint32)
    n = off.shape[0] - 1
    if minpts < 0:
        raise ValueError("minpts must be >= 0")
    labels = np.empty(max(n, 0), dtype=np.int32)
    core = np.empty(max(n, 0), dtype=np.uint8)
    k = lib.oracle_dbscan(_ptr(off), _ptr(nbr), n, int(minpts), _ptr(labels), _ptr(core))
    if k < 0:
        raise MemoryError("oracle_dbscan: allocation failed")
    return labels, core, int(k)
