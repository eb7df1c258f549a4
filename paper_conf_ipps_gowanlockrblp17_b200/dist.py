"""Process-level query sharding helpers (torchrun mode).

Every rank builds the full grid and computes the table of its shard of the
cell-sorted queries (``hdb_opts.shard_rank/shard_count``).  The one exchange
of the path is the gather of per-shard pair counts, which gives each shard its
base offset in the single table (``gather_pair_counts``); ``assemble`` builds
that table on one rank from the shards' host tables.  Plumbing only -- the
tables themselves come from libhdb.
"""
from __future__ import annotations

import numpy as np


def gather_pair_counts(pairs: int, device=None):
    """all_gather of this rank's pair count -> (bases[world], total)."""
    import torch
    import torch.distributed as dist
    ws = dist.get_world_size()
    t = torch.tensor([int(pairs)], dtype=torch.int64, device=device)
    out = [torch.zeros_like(t) for _ in range(ws)]
    dist.all_gather(out, t)
    counts = [int(x.item()) for x in out]
    bases = np.concatenate([[0], np.cumsum(counts)[:-1]]).astype(np.uint64)
    return bases, int(sum(counts))


def assemble(parts, n):
    """Merge shard host tables [(begin, count, nbrs), ...] in shard order into
    one table (begin by original id into the concatenated nbrs).  Rows absent
    from a shard have count 0 there; every row must be present in exactly one
    shard."""
    begin = np.zeros(n, np.uint64)
    count = np.zeros(n, np.uint32)
    seen = np.zeros(n, np.int32)
    base = 0
    flats = []
    for b, c, v in parts:
        mine = c > 0
        begin[mine] = b[mine] + np.uint64(base)
        count[mine] = c[mine]
        seen += mine
        flats.append(v)
        base += v.size
    if n and not np.all(seen == 1):
        raise ValueError("shards do not partition the rows")
    nbrs = np.concatenate(flats) if flats else np.zeros(0, np.uint32)
    return begin, count, nbrs
