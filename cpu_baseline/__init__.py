"""CPU grid-join comparator -- BENCHMARK / TEST INFRASTRUCTURE ONLY.

The single-thread (and, with ``threads > 1``, OpenMP) CPU epsilon grid-join
that the north star times beside the GPU path (CPU baselines 2/3).
See gridjoin.c for the method and citations.  Used by ``bench.py``'s
``cpu_baseline`` leg and by ``tests/`` (which check it against ``oracle/``);
never by the library.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading
import time

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gridjoin.c")
_LIB = os.path.join(_HERE, "libgridjoin.so")
CFLAGS = ["-O3", "-march=x86-64-v3", "-ffp-contract=off", "-fno-fast-math", "-DGJ_FP_CONTRACT_OFF",
          "-fopenmp", "-fPIC", "-shared", "-std=c11", "-Wall", "-Wextra"]
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    if (not force and os.path.exists(_LIB)
            and os.path.getmtime(_LIB) >= os.path.getmtime(_SRC)):
        return _LIB
    tmp = _LIB + f".tmp{os.getpid()}"
    subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp, "-lm"])
    os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            P, i64, d, i = ctypes.c_void_p, ctypes.c_int64, ctypes.c_double, ctypes.c_int
            lib.gj_prepare.argtypes = [P, i64, i, d, ctypes.POINTER(ctypes.c_int)]
            lib.gj_prepare.restype = P
            lib.gj_release.argtypes = [P]
            lib.gj_count.argtypes = [P, P, i, d, P, i64, i, P]
            lib.gj_fill.argtypes = [P, P, i, d, P, i64, i, P, P]
            _lib = lib
        return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def gridjoin_rows(xy, eps, rows=None, dtype="f64", threads=1, timings=None):
    """Neighbour lists of the query ``rows`` (None = all) as CSR (off, nbr),
    lists in candidate order.  ``timings`` (dict) receives the seconds spent in
    the grid build and in the join (count + fill)."""
    lib = _load()
    npdt = np.float64 if dtype == "f64" else np.float32
    xy = np.ascontiguousarray(xy, dtype=npdt).reshape(-1, 2)
    n = xy.shape[0]
    is32 = 1 if dtype == "f32" else 0
    if rows is None:
        nrows, rp = n, None
    else:
        rp = np.ascontiguousarray(rows, dtype=np.int64)
        nrows = rp.shape[0]
    t0 = time.perf_counter()
    st = ctypes.c_int(0)
    h = lib.gj_prepare(_p(xy), n, is32, float(eps), ctypes.byref(st))
    if st.value != 0:
        raise RuntimeError(f"gj_prepare failed ({st.value})")
    t1 = time.perf_counter()
    try:
        cnt = np.zeros(nrows, dtype=np.uint64)
        lib.gj_count(h, _p(xy), is32, float(eps), _p(rp), nrows, int(threads), _p(cnt))
        off = np.zeros(nrows + 1, dtype=np.uint64)
        np.cumsum(cnt, out=off[1:])
        nbr = np.empty(int(off[-1]), dtype=np.uint32)
        lib.gj_fill(h, _p(xy), is32, float(eps), _p(rp), nrows, int(threads), _p(off), _p(nbr))
    finally:
        lib.gj_release(h)
    t2 = time.perf_counter()
    if timings is not None:
        timings["build_s"] = t1 - t0
        timings["join_s"] = t2 - t1
    return off, nbr
