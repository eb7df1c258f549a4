"""Thin ctypes binding of libhdb (include/hdb.h) -- argument marshalling only.

Every function keeps the C name and signature shape; statuses other than
HDB_OK raise :class:`HdbError` carrying ``hdb_last_error()``.  Buffers may be
numpy arrays (host), torch tensors (host or CUDA) or raw integer pointers.
There is no CPU fallback: if ``libhdb.so`` is missing, importing this module
raises ImportError (run ``__graft_entry__.build()``).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("HDB_LIB") or os.path.join(_HERE, "libhdb.so")   # HDB_LIB: A/B builds (tools/ab.sh)

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} not built: run `python -c 'import __graft_entry__ as g; g.build()'`")

lib = ctypes.CDLL(LIB_PATH)

HDB_OK, HDB_EINVAL, HDB_ERANGE, HDB_ENOMEM, HDB_ECUDA, HDB_EINTERNAL = 0, -1, -2, -3, -4, -5
HDB_F64, HDB_F32 = 0, 1
STATUS_NAMES = {0: "HDB_OK", -1: "HDB_EINVAL", -2: "HDB_ERANGE", -3: "HDB_ENOMEM", -4: "HDB_ECUDA",
                -5: "HDB_EINTERNAL"}

_u64, _u32, _i32, _dbl, _vp = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int32, ctypes.c_double, ctypes.c_void_p
_int = ctypes.c_int


class hdb_opts(ctypes.Structure):
    _fields_ = [("devices", ctypes.POINTER(_int)), ("n_devices", _int), ("sample_fraction", _dbl),
                ("alpha", _dbl), ("n_streams", _int), ("batch_pairs", _u64), ("sort_lists", _int),
                ("host_budget_bytes", _u64), ("shard_rank", _int), ("shard_count", _int),
                ("search_kernel", _int), ("host_threads", _int), ("cell_split", _int),
                ("sweep_on_device", _int)]


class hdb_table_view(ctypes.Structure):
    _fields_ = [("n", _u64), ("npairs", _u64), ("begin", _vp), ("count", _vp), ("nbrs", _vp),
                ("on_device", _int), ("device", _int), ("first_query", _u64), ("end_query", _u64),
                ("eps", _dbl), ("dtype", _int)]


class hdb_grid_view(ctypes.Structure):
    _fields_ = [("n", _u64), ("eps", _dbl), ("dtype", _int), ("xmin", _dbl), ("ymin", _dbl), ("xmax", _dbl),
                ("ymax", _dbl), ("cell_w", _dbl), ("nx", _u32), ("ny", _u32), ("n_cells", _u64),
                ("n_nonempty", _u64), ("n_groups", _u64), ("device", _int), ("xy_sorted", _vp), ("ids", _vp),
                ("cell_keys", _vp), ("cell_start", _vp)]


class hdb_stats(ctypes.Structure):
    _fields_ = [(k, _u64) for k in ("n", "npairs", "n_cells", "n_nonempty", "n_groups", "sample_size",
                                    "sample_pairs", "est_pairs", "planned_batch_pairs", "planned_batches",
                                    "n_batches", "max_batch_pairs", "candidate_tests", "bytes_h2d",
                                    "bytes_d2h", "pool_grows")] + \
        [("n_streams", _int), ("n_devices", _int), ("kernel_launches", _u32), ("write_launches", _u32)] + \
        [(k, _dbl) for k in ("ms_grid", "ms_sample", "ms_count", "ms_scan", "ms_write_kernel", "ms_table_wall")] + \
        [("single_pass", _int), ("ms_sort", _dbl), ("n_sparse_queries", _u64), ("query_lanes", _int)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


_PP = ctypes.POINTER(_vp)
_sig = {
    "hdb_opts_default": (None, [ctypes.POINTER(hdb_opts)]),
    "hdb_ctx_create": (_int, [ctypes.POINTER(hdb_opts), _PP]),
    "hdb_ctx_destroy": (None, [_vp]),
    "hdb_ctx_set_stream": (_int, [_vp, _vp]),
    "hdb_stats_get": (_int, [_vp, ctypes.POINTER(hdb_stats)]),
    "hdb_grid_build": (_int, [_vp, _vp, _u64, _int, _dbl, _PP]),
    "hdb_grid_free": (None, [_vp]),
    "hdb_grid_view_get": (_int, [_vp, ctypes.POINTER(hdb_grid_view)]),
    "hdb_grid_copy_to_host": (_int, [_vp, _vp, _vp, _vp, _vp]),
    "hdb_neighbor_table": (_int, [_vp, _vp, _PP]),
    "hdb_neighbor_table_device": (_int, [_vp, _vp, _PP]),
    "hdb_table_from_host": (_int, [_u64, _vp, _vp, _vp, _u64, _PP]),
    "hdb_table_view_get": (_int, [_vp, ctypes.POINTER(hdb_table_view)]),
    "hdb_table_copy_to_host": (_int, [_vp, _vp, _vp, _vp]),
    "hdb_table_canonicalize": (_int, [_vp]),
    "hdb_table_free": (None, [_vp]),
    "hdb_dbscan": (_int, [_vp, _u32, _vp, _vp, _vp]),
    "hdb_dbscan_ex": (_int, [_vp, _u32, _int, _vp, _vp, _vp]),
    "hdb_sweep": (_int, [_vp, _vp, _u64, _int, _vp, _u32, _vp, _u32, _vp, _vp]),
    "hdb_plan_batches": (_int, [_dbl, _dbl, _int, ctypes.POINTER(_dbl), ctypes.POINTER(_u64)]),
    "hdb_strided_point": (_u64, [_u64, _u64, _u64]),
    "hdb_balanced_cuts": (_int, [_vp, _u64, _u32, _vp]),
    "hdb_last_error": (ctypes.c_char_p, []),
    "hdb_version": (ctypes.c_char_p, []),
    "hdb_kernel_launches": (_u64, []),
}
for _name, (_res, _args) in _sig.items():
    _f = getattr(lib, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED = tuple(_sig)


class HdbError(RuntimeError):
    def __init__(self, status, where):
        self.status = status
        msg = lib.hdb_last_error().decode(errors="replace")
        super().__init__(f"{where}: {STATUS_NAMES.get(status, status)}: {msg}")


def _check(st, where):
    if st != HDB_OK:
        raise HdbError(st, where)


def _ptr(buf):
    """Pointer of a numpy array / torch tensor / int / None."""
    if buf is None:
        return None
    if isinstance(buf, int):
        return buf
    if isinstance(buf, np.ndarray):
        if not buf.flags["C_CONTIGUOUS"]:
            raise ValueError("buffer must be C-contiguous")
        return buf.ctypes.data
    if hasattr(buf, "data_ptr"):
        if not buf.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return buf.data_ptr()
    raise TypeError(f"unsupported buffer type {type(buf)}")


def _dtype_of(xy):
    dt = getattr(xy, "dtype", None)
    s = str(dt)
    if s in ("float64", "torch.float64"):
        return HDB_F64
    if s in ("float32", "torch.float32"):
        return HDB_F32
    raise TypeError(f"xy must be float64 or float32, got {dt}")


def _nrows(xy):
    shape = tuple(xy.shape)
    if len(shape) == 2 and shape[1] == 2:
        return shape[0]
    if len(shape) == 1 and shape[0] % 2 == 0:
        return shape[0] // 2
    raise ValueError(f"xy must have shape (n, 2), got {shape}")


# ------------------------------------------------------------------ functions
def hdb_opts_default(**over) -> hdb_opts:
    o = hdb_opts()
    lib.hdb_opts_default(ctypes.byref(o))
    devices = over.pop("devices", None)
    for k, v in over.items():
        setattr(o, k, v)
    if devices:
        arr = (_int * len(devices))(*devices)
        o.devices = ctypes.cast(arr, ctypes.POINTER(_int))
        o.n_devices = len(devices)
        o._keep = arr
    return o


def hdb_ctx_create(opts: hdb_opts | None = None, **over):
    if opts is None:
        opts = hdb_opts_default(**over)
    out = _vp()
    _check(lib.hdb_ctx_create(ctypes.byref(opts), ctypes.byref(out)), "hdb_ctx_create")
    return out.value


def hdb_ctx_destroy(ctx):
    lib.hdb_ctx_destroy(ctx)


def hdb_ctx_set_stream(ctx, stream):
    _check(lib.hdb_ctx_set_stream(ctx, stream), "hdb_ctx_set_stream")


def hdb_stats_get(ctx) -> dict:
    s = hdb_stats()
    _check(lib.hdb_stats_get(ctx, ctypes.byref(s)), "hdb_stats_get")
    return s.as_dict()


def hdb_grid_build(ctx, xy, eps: float, dtype: int | None = None):
    """xy: (n,2) float64/float32 numpy array or torch tensor (host or CUDA)."""
    n = _nrows(xy)
    dt = _dtype_of(xy) if dtype is None else dtype
    out = _vp()
    _check(lib.hdb_grid_build(ctx, _ptr(xy), n, dt, float(eps), ctypes.byref(out)), "hdb_grid_build")
    return out.value


def hdb_grid_free(grid):
    lib.hdb_grid_free(grid)


def hdb_grid_view_get(grid) -> hdb_grid_view:
    v = hdb_grid_view()
    _check(lib.hdb_grid_view_get(grid, ctypes.byref(v)), "hdb_grid_view_get")
    return v


def hdb_grid_copy_to_host(grid):
    v = hdb_grid_view_get(grid)
    ids = np.empty(v.n, np.uint32)
    keys = np.empty(v.n_nonempty, np.uint64)
    start = np.empty(v.n_nonempty + 1, np.uint32)
    xy = np.empty((v.n, 2), np.float64 if v.dtype == HDB_F64 else np.float32)
    _check(lib.hdb_grid_copy_to_host(grid, _ptr(ids), _ptr(keys), _ptr(start), _ptr(xy)), "hdb_grid_copy_to_host")
    return dict(ids=ids, cell_keys=keys, cell_start=start, xy_sorted=xy, view=v)


def hdb_neighbor_table(ctx, grid):
    out = _vp()
    _check(lib.hdb_neighbor_table(ctx, grid, ctypes.byref(out)), "hdb_neighbor_table")
    return out.value


def hdb_neighbor_table_device(ctx, grid):
    out = _vp()
    _check(lib.hdb_neighbor_table_device(ctx, grid, ctypes.byref(out)), "hdb_neighbor_table_device")
    return out.value


def hdb_table_from_host(begin, count, nbrs):
    begin = np.ascontiguousarray(begin, np.uint64)
    count = np.ascontiguousarray(count, np.uint32)
    nbrs = np.ascontiguousarray(nbrs, np.uint32)
    out = _vp()
    _check(lib.hdb_table_from_host(begin.size, _ptr(begin), _ptr(count), _ptr(nbrs), nbrs.size, ctypes.byref(out)),
           "hdb_table_from_host")
    return out.value


def hdb_table_view_get(table) -> hdb_table_view:
    v = hdb_table_view()
    _check(lib.hdb_table_view_get(table, ctypes.byref(v)), "hdb_table_view_get")
    return v


def hdb_table_copy_to_host(table):
    """(begin uint64[n], count uint32[n], nbrs uint32[npairs]) copies."""
    v = hdb_table_view_get(table)
    begin = np.empty(v.n, np.uint64)
    count = np.empty(v.n, np.uint32)
    nbrs = np.empty(v.npairs, np.uint32)
    _check(lib.hdb_table_copy_to_host(table, _ptr(begin), _ptr(count), _ptr(nbrs)), "hdb_table_copy_to_host")
    return begin, count, nbrs


def hdb_table_canonicalize(table):
    _check(lib.hdb_table_canonicalize(table), "hdb_table_canonicalize")


def hdb_table_free(table):
    lib.hdb_table_free(table)


def hdb_dbscan(table, minpts: int, n_threads: int = 0, labels=None, is_core=None):
    """DBSCAN on a host table (host threads) or a device table (GPU, NEXT-4).
    labels / is_core: numpy (host) or torch CUDA tensors; allocated on the host if None."""
    v = hdb_table_view_get(table)
    if labels is None:
        labels = np.empty(v.n, np.int32)
    if is_core is None:
        is_core = np.empty(v.n, np.uint8)
    k = _u32(0)
    _check(lib.hdb_dbscan_ex(table, int(minpts), int(n_threads), _ptr(labels), _ptr(is_core), ctypes.byref(k)),
           "hdb_dbscan")
    return labels, is_core, int(k.value)


def hdb_sweep(ctx, xy, eps_list, minpts_list, dtype: int | None = None, labels=None):
    """labels: optional preallocated int32 [n_eps, n_minpts, n] (numpy, or a CUDA
    tensor when the context was created with sweep_on_device=1)."""
    n = _nrows(xy)
    dt = _dtype_of(xy) if dtype is None else dtype
    eps = np.ascontiguousarray(eps_list, np.float64)
    mp = np.ascontiguousarray(minpts_list, np.uint32)
    if labels is None:
        labels = np.empty((eps.size, mp.size, n), np.int32)
    k = np.empty((eps.size, mp.size), np.uint32)
    _check(lib.hdb_sweep(ctx, _ptr(xy), n, dt, _ptr(eps), eps.size, _ptr(mp), mp.size, _ptr(labels), _ptr(k)),
           "hdb_sweep")
    return labels, k


def hdb_plan_batches(est_pairs: float, alpha: float, n_streams: int):
    bb = _dbl(0)
    nb = _u64(0)
    _check(lib.hdb_plan_batches(float(est_pairs), float(alpha), int(n_streams), ctypes.byref(bb), ctypes.byref(nb)),
           "hdb_plan_batches")
    return bb.value, int(nb.value)


def hdb_strided_point(gid: int, l: int, n_b: int) -> int:
    return int(lib.hdb_strided_point(gid, l, n_b))


def hdb_balanced_cuts(prefix, parts: int):
    prefix = np.ascontiguousarray(prefix, np.uint64)
    cuts = np.empty(parts + 1, np.uint64)
    _check(lib.hdb_balanced_cuts(_ptr(prefix), prefix.size - 1, int(parts), _ptr(cuts)), "hdb_balanced_cuts")
    return cuts


def hdb_last_error() -> str:
    return lib.hdb_last_error().decode(errors="replace")


def hdb_version() -> str:
    return lib.hdb_version().decode()


def hdb_kernel_launches() -> int:
    return int(lib.hdb_kernel_launches())
