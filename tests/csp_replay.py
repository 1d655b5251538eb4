"""CPU replay of CSP's three stages (Sec. 4.1) on oracle pieces.

Test infrastructure: per layer, every rank groups its frontier by owner
(contiguous id ranges), ships the ids to the owners ("shuffle"), each
owner runs ``oracle.sample_rows`` on ITS OWN CSR shard ("sample"), the rows go
back to the requester in request order ("reshuffle") and the requester builds
its block with ``oracle.build_block``.  Two transports: in-process lists, or
``torch.distributed`` all_to_all over gloo (world_size >= 2 on CPU).  Used to
pin the oracle's partition invariance (R8, R16) and the Fig. 5
message pattern.
"""
from __future__ import annotations

import numpy as np

import oracle


def owner_of(ids, bounds) -> np.ndarray:
    return np.searchsorted(np.asarray(bounds), np.asarray(ids, np.int64), side="right") - 1


def _shard(indptr, indices, lo, hi, weights=None):
    ip = indptr[lo: hi + 1]
    w = None if weights is None else weights[ip[0]: ip[-1]]
    return ip - ip[0], indices[ip[0]: ip[-1]], w


def replay_inprocess(indptr, indices, bounds, rank_seeds, fanouts, rng_seed, log=None, weights=None):
    """All P ranks in one process.  Returns blocks[r][l] (oracle dicts).
    ``weights`` (fp32 per edge) selects biased sampling; each owner uses its
    own shard of them."""
    N = len(indptr) - 1
    P = len(bounds) - 1
    shards = [_shard(indptr, indices, int(bounds[o]), int(bounds[o + 1]), weights) for o in range(P)]
    frontier = [np.asarray(s, np.int32) for s in rank_seeds]
    blocks = [[] for _ in range(P)]
    for l, k in enumerate(fanouts):
        # shuffle: requests[r][o] = (frontier positions, ids) that r sends to o
        own = [owner_of(f, bounds) for f in frontier]
        req = [[np.nonzero(own[r] == o)[0] for o in range(P)] for r in range(P)]
        if log is not None:
            log.append({"layer": l, "shuffle": {f"{r}->{o}": frontier[r][req[r][o]].tolist()
                                                for r in range(P) for o in range(P)}})
        # sample at the owner on its shard
        res = [[None] * P for _ in range(P)]
        for o in range(P):
            ip, ix, w = shards[o]
            for r in range(P):
                ids = frontier[r][req[r][o]]
                res[r][o] = oracle.sample_rows(ip, ix, ids, k, l, rng_seed, id_offset=int(bounds[o]), weights=w)
        # reshuffle back to request order, then build the block
        for r in range(P):
            F = len(frontier[r])
            cnt = np.zeros(F, np.int32)
            rows = np.full((F, k), -1, np.int32)
            for o in range(P):
                c, rw = res[r][o]
                cnt[req[r][o]] = c
                rows[req[r][o]] = rw
            if log is not None:
                log[-1].setdefault("reshuffle_rows", {}).update(
                    {f"{o}->{r}": {int(frontier[r][i]): rows[i, :cnt[i]].tolist() for i in req[r][o]}
                     for o in range(P) if o != r and len(req[r][o])})
            b = oracle.build_block(N, frontier[r], cnt, rows)
            blocks[r].append(b)
            frontier[r] = b["src_ids"]
    return blocks


def replay_distributed(indptr_shard, indices_shard, bounds, seeds, fanouts, rng_seed, num_nodes):
    """One rank of the replay over torch.distributed (gloo).  Each rank holds
    ONLY its own CSR shard.  Returns this rank's blocks."""
    import torch
    import torch.distributed as dist
    P = dist.get_world_size()
    r = dist.get_rank()
    frontier = np.asarray(seeds, np.int32)
    blocks = []
    for l, k in enumerate(fanouts):
        own = owner_of(frontier, bounds)
        order = np.argsort(own, kind="stable")
        send_counts = np.bincount(own, minlength=P).astype(np.int64)
        # count notification first, then the ids
        recv_counts = torch.zeros(P, dtype=torch.int64)
        dist.all_to_all_single(recv_counts, torch.from_numpy(send_counts))
        recv_counts = recv_counts.numpy()
        recv_ids = torch.zeros(int(recv_counts.sum()), dtype=torch.int32)
        dist.all_to_all_single(recv_ids, torch.from_numpy(frontier[order].copy()),
                               output_split_sizes=recv_counts.tolist(),
                               input_split_sizes=send_counts.tolist())
        cnt, rows = oracle.sample_rows(indptr_shard, indices_shard, recv_ids.numpy(), k, l, rng_seed,
                                       id_offset=int(bounds[r]))
        packed = np.concatenate([cnt[:, None], rows], axis=1).astype(np.int32)   # [n, 1 + k]
        back = torch.zeros((len(frontier), 1 + k), dtype=torch.int32)
        dist.all_to_all_single(back, torch.from_numpy(packed),
                               output_split_sizes=send_counts.tolist(),
                               input_split_sizes=recv_counts.tolist())
        back = back.numpy()
        cnt_f = np.zeros(len(frontier), np.int32)
        rows_f = np.zeros((len(frontier), k), np.int32)
        cnt_f[order] = back[:, 0]
        rows_f[order] = back[:, 1:]
        b = oracle.build_block(num_nodes, frontier, cnt_f, rows_f)
        blocks.append(b)
        frontier = b["src_ids"]
    return blocks


def replay_layerwise_inprocess(indptr, indices, bounds, rank_seeds, sizes, rng_seed):
    """Layer-wise CSP replayed on P in-process ranks: per layer a
    requester asks the owners for its frontier's degrees (W_u, shuffle), draws
    the Eq. 2 allocation itself (``oracle.layer_alloc``), pushes (u, c_u) to
    the owners, which sample c_u neighbours on their own shard
    (``oracle.node_positions``), and builds its block from the returned rows."""
    N = len(indptr) - 1
    P = len(bounds) - 1
    shards = [_shard(indptr, indices, int(bounds[o]), int(bounds[o + 1])) for o in range(P)]
    frontier = [np.asarray(s, np.int32) for s in rank_seeds]
    g0 = [int(s[0]) if len(s) else 0 for s in rank_seeds]
    blocks = [[] for _ in range(P)]
    for l, n in enumerate(sizes):
        for r in range(P):
            f = frontier[r]
            own = owner_of(f, bounds)
            # degree query at the owners
            W = np.zeros(len(f), np.uint64)
            for i, (v, o) in enumerate(zip(f.tolist(), own.tolist())):
                ip, _, _ = shards[o]
                lv = v - int(bounds[o])
                W[i] = ip[lv + 1] - ip[lv]
            c = oracle.layer_alloc(rng_seed, g0[r], l, W, n)
            # sampling tasks pushed to the owners; rows come back in request order
            width = max(1, int(c.max()) if len(c) else 1)
            cnt = np.zeros(len(f), np.int32)
            rows = np.full((len(f), width), -1, np.int32)
            for i, (v, o) in enumerate(zip(f.tolist(), own.tolist())):
                if c[i] == 0:
                    continue
                ip, ix, _ = shards[o]
                lv = v - int(bounds[o])
                s0, d = int(ip[lv]), int(ip[lv + 1] - ip[lv])
                pos = oracle.node_positions(rng_seed, v, l, d, int(c[i]))
                cnt[i] = len(pos)
                rows[i, :len(pos)] = ix[s0 + pos]
            b = oracle.build_block(N, f, cnt, rows)
            blocks[r].append(b)
            frontier[r] = b["src_ids"]
    return blocks
