"""Multi-process (world size 2, gloo, CPU) test of the shard plumbing: the
gather of per-shard pair counts and the assembly of the shards' tables into
one table.  The shards here are row ranges of an oracle table (no GPU)."""
import os
import socket

import numpy as np
import pytest

import datagen
import oracle


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, ws, port, q):
    import torch.distributed as dist
    from paper_conf_ipps_gowanlockrblp17_b200 import dist as hd
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    try:
        xy = datagen.subsample(datagen.tec_like(100_000, seed=2), 3000, seed=rank * 0 + 7)
        off, nbr = oracle.eps_join(xy, 0.8)
        n = xy.shape[0]
        # shard = contiguous row range; its table stores only its rows, with
        # begin relative to its own nbrs (what libhdb returns per shard)
        lo, hi = (n * rank) // ws, (n * (rank + 1)) // ws
        cnt = np.zeros(n, np.uint32)
        beg = np.zeros(n, np.uint64)
        cnt[lo:hi] = np.diff(off[lo:hi + 1].astype(np.int64))
        beg[lo:hi] = off[lo:hi] - off[lo]
        mine = nbr[off[lo]:off[hi]]
        bases, total = hd.gather_pair_counts(mine.size)
        parts = [None] * ws
        obj = [(beg, cnt, mine)]
        gathered = [None] * ws
        dist.all_gather_object(gathered, obj[0])
        if rank == 0:
            b, c, v = hd.assemble(gathered, n)
            ok = (total == int(off[-1]) and int(bases[1]) == int(off[(n * 1) // ws])
                  and np.array_equal(c.astype(np.uint64), np.diff(off))
                  and all(np.array_equal(v[b[p]:b[p] + c[p]], nbr[off[p]:off[p + 1]]) for p in range(n)))
            q.put(bool(ok))
    finally:
        dist.destroy_process_group()


def test_gather_and_assemble_world2():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=240)
        assert p.exitcode == 0
    assert q.get(timeout=10) is True


def test_assemble_rejects_overlap():
    from paper_conf_ipps_gowanlockrblp17_b200 import dist as hd
    b = np.zeros(2, np.uint64)
    c = np.ones(2, np.uint32)
    v = np.array([0, 1], np.uint32)
    with pytest.raises(ValueError):
        hd.assemble([(b, c, v), (b, c, v)], 2)
