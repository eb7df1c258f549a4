"""Test helper: per-row (count, order-free hash) of a LIBRARY table, to compare
with the oracle's ``sweep_rowhash`` / ``strip_rowhash`` / ``eps_join_rowhash``
row by row at sizes where the two tables cannot both be held on the host
(SURVEY.md 8(c) O4).  hash(row) = sum of mix64(q) over the row's list, mod 2^64,
mix64 = the SplitMix64 finaliser (the oracle's definition, re-typed here in
torch int64 arithmetic; pinned against the oracle by tests/test_rowhash.py).

This is test code: it reads the library's output through the table view
(device pointers for device tables) and never calls the oracle.
"""
from __future__ import annotations

import numpy as np

_M64 = (1 << 64)


def _s64(v: int) -> int:
    """uint64 constant -> the int64 with the same bits."""
    return v - _M64 if v >= (1 << 63) else v


C1, C2, C3 = _s64(0x9E3779B97F4A7C15), _s64(0xBF58476D1CE4E5B9), _s64(0x94D049BB133111EB)


def mix64(torch, x):
    """SplitMix64 finaliser on an int64 tensor (bits of the uint64 value), wrapping."""
    def lsr(z, k):
        return (z >> k) & ((1 << (64 - k)) - 1)
    z = x + C1
    z = (z ^ lsr(z, 30)) * C2
    z = (z ^ lsr(z, 27)) * C3
    return z ^ lsr(z, 31)


class _CAI:
    """__cuda_array_interface__ wrapper of a raw device pointer (borrowed)."""

    def __init__(self, ptr, n, typestr):
        self.__cuda_array_interface__ = {"shape": (int(n),), "typestr": typestr, "data": (int(ptr), False),
                                         "version": 3, "strides": None}


def view_tensors(torch, view):
    """(begin int64, count int64, nbrs int32) tensors of a table view; device
    tables are wrapped in place (no copy), host tables copied from the view."""
    n, P = int(view.n), int(view.npairs)
    if view.on_device:
        dev = torch.device("cuda", int(view.device))
        begin = torch.as_tensor(_CAI(view.begin, n, "<i8"), device=dev) if n else torch.zeros(0, dtype=torch.int64, device=dev)
        count = torch.as_tensor(_CAI(view.count, n, "<i4"), device=dev).to(torch.int64) if n else torch.zeros(0, dtype=torch.int64, device=dev)
        nbrs = torch.as_tensor(_CAI(view.nbrs, P, "<i4"), device=dev) if P else torch.zeros(0, dtype=torch.int32, device=dev)
        return begin, count, nbrs
    import ctypes
    b = np.ctypeslib.as_array(ctypes.cast(view.begin, ctypes.POINTER(ctypes.c_int64)), (n,)) if n else np.zeros(0, np.int64)
    c = np.ctypeslib.as_array(ctypes.cast(view.count, ctypes.POINTER(ctypes.c_int32)), (n,)) if n else np.zeros(0, np.int32)
    v = np.ctypeslib.as_array(ctypes.cast(view.nbrs, ctypes.POINTER(ctypes.c_int32)), (P,)) if P else np.zeros(0, np.int32)
    return torch.from_numpy(b.copy()), torch.from_numpy(c.astype(np.int64)), torch.from_numpy(v)


def table_rowhash(torch, begin, count, nbrs, max_entries=1 << 28):
    """Per-row (count uint64[n], hash uint64[n]) of the table (begin, count, nbrs)
    given as torch tensors (any device).  Rows are visited in begin order in
    batches of <= max_entries entries (bounded memory at 34 GB tables)."""
    n = begin.numel()
    dev = begin.device
    h = torch.zeros(n, dtype=torch.int64, device=dev)
    if n == 0:
        return np.zeros(0, np.uint64), np.zeros(0, np.uint64)
    order = torch.argsort(begin)
    b_s, c_s = begin[order], count[order]
    e_s = b_s + c_s
    # batch cuts: rows [r0, r1) with e_s[r1-1] - b_s[r0] <= max_entries (a single
    # longer row forms its own batch)
    starts = b_s.cpu().numpy()
    ends = e_s.cpu().numpy()
    r0 = 0
    while r0 < n:
        lim = starts[r0] + max_entries
        r1 = int(np.searchsorted(ends, lim, side="right"))
        r1 = max(r1, r0 + 1)
        a, z = int(starts[r0]), int(ends[r1 - 1])
        if z > a:
            vals = nbrs[a:z].to(torch.int64) & 0xFFFFFFFF
            cs = torch.zeros(z - a + 1, dtype=torch.int64, device=dev)
            torch.cumsum(mix64(torch, vals), 0, out=cs[1:])
            del vals
            lb = b_s[r0:r1] - a
            le = e_s[r0:r1] - a
            h[order[r0:r1]] = cs[le] - cs[lb]
            del cs
        r0 = r1
    return count.cpu().numpy().astype(np.uint64), h.cpu().numpy().view(np.uint64)
