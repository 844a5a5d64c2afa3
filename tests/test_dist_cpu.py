"""Multi-process host logic of the sharded MSM on CPU (`-m "not gpu"`),
world_size 2 over gloo:

* shard_range partitions [0, n) exactly, contiguous and in rank order;
* the NCCL unique id made by rank 0 reaches every rank unchanged;
* the sharding maths: per-rank partial sums folded in rank order equal the
  full MSM (partials from the oracle here, standing in for the GPU partial);
* the bench's max-over-ranks timing reduction.
"""

import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_shard_range_partitions():
    import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
    for n in (0, 1, 2, 7, 8, 1000, 1 << 20, (1 << 22) + 3):
        for G in range(1, 9):
            spans = [gz.shard_range(n, G, r) for r in range(G)]
            assert spans[0][0] == 0 and spans[-1][1] == n
            for (a, b), (c, d) in zip(spans, spans[1:]):
                assert b == c and a <= b
            assert sum(b - a for a, b in spans) == n


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, ROOT)
    import torch
    import torch.distributed as dist

    import oracle
    import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
    import synth
    try:
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", world_size=world, rank=rank)
        # 1. unique id broadcast
        uid = gz.broadcast_unique_id(rank)
        ids = [None] * world
        dist.all_gather_object(ids, uid)
        # 2. sharded MSM maths with a rank-order fold
        curve, n = "bn254", 37
        d = synth.dlogs(curve, n, 5)
        pts = oracle.points_from_dlogs(curve, d, nthreads=1)
        k = synth.scalars(curve, n, 6)
        lo, hi = gz.shard_range(n, world, rank)
        part = oracle.msm(curve, pts[lo:hi], k[lo:hi], nthreads=1)
        parts = [None] * world
        dist.all_gather_object(parts, part)
        acc = np.zeros_like(part)
        for p in parts:
            acc = oracle.ec_add(curve, acc, p)
        full = oracle.msm(curve, pts, k, nthreads=1)
        # 3. max over ranks of a per-rank time (bench.py)
        t = torch.tensor([10.0 + rank], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        q.put((rank, len(set(ids)) == 1 and len(ids[0]) == 128, bool(np.array_equal(acc, full)),
               float(t.item())))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover - surfaced by the assert below
        q.put((rank, repr(e), None, None))


def test_two_rank_gloo_sharded_logic():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, ids_ok, fold_ok, tmax in res:
        assert ids_ok is True, (rank, ids_ok)
        assert fold_ok is True, rank
        assert tmax == 10.0 + world - 1
