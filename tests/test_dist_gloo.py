"""World-size-2 gloo tests on CPU for the N > 1 path's host logic:
the CSP exchange protocol (count notification, then ids, then rows)
with each rank holding only its own shard, seed co-partitioning and the
steps-per-epoch agreement, and bench.py's max-over-ranks timing reduction."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import sys
    here = os.path.dirname(os.path.abspath(__file__))
    sys.path[:0] = [os.path.dirname(here), here]
    import datagen
    import oracle
    from csp_replay import replay_distributed
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        cfg = datagen.CONFIGS["tiny"]
        ip, ix = datagen.make_graph(cfg)
        bnds = datagen.bounds(cfg.num_nodes, world)
        my_ip, my_ix = datagen.shard(ip, ix, int(bnds[rank]), int(bnds[rank + 1]))
        train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
        steps = datagen.steps_per_epoch(train, bnds, cfg.batch)
        t = torch.tensor([steps])
        dist.all_reduce(t, op=dist.ReduceOp.MIN)
        assert int(t) == steps                         # every rank computes the same count
        batches = datagen.rank_seed_batches(train, bnds, rank, cfg.batch, 0)
        ok = True
        for step in range(2):
            seeds = batches[step]
            blocks = replay_distributed(my_ip, my_ix, bnds, seeds, cfg.fanouts, 0x5EED + step,
                                        cfg.num_nodes)
            ref = oracle.sample(ip, ix, seeds, cfg.fanouts, 0x5EED + step)
            for b, e in zip(blocks, ref):
                for key in ("indptr", "indices", "src_ids"):
                    ok &= bool(np.array_equal(b[key], e[key]))
        # bench.py reduction: every rank contributes its device time, rank 0 reports the max
        from bench import reduce_max_over_ranks
        m = reduce_max_over_ranks(float(rank + 1) * 1.5)
        ok &= (m == 1.5 * world)
        q.put((rank, ok, steps))
    finally:
        dist.destroy_process_group()


def test_csp_protocol_gloo_world2():
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
        assert p.exitcode == 0
    assert all(ok for _, ok, _ in res), res
    assert len({s for _, _, s in res}) == 1
