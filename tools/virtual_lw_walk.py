"""Multi-rank layer-wise sampling and random walks as P virtual ranks on one GPU
(products graph): time per synchronous group call, one cooperative launch per
rank.
python tools/virtual_lw_walk.py"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import datagen
import paper_conf_ppopp_caiz0zszck23_b200 as pkg

cfg = datagen.CONFIGS["products"]
ip, ix = datagen.make_graph(cfg)
train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
mode = "persistent"
for P in (2, 4):
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, datagen.features(lo, hi, 4)))
    # layer-wise, Table 7 sizes
    grp = pkg.LocalGroup(bnds, shards, (1000, 1000), cfg.batch, devices=[0] * P, scheme="layer")
    per = [datagen.rank_seed_batches(train, bnds, r, cfg.batch, 0) for r in range(P)]
    for it in range(25):
        if it == 5:
            torch.cuda.synchronize()
            t0 = time.perf_counter()
        grp.sample([torch.from_numpy(per[r][it % len(per[r])]).cuda() for r in range(P)], 7 + it)
    torch.cuda.synchronize()
    print(f"layer-wise ({mode}) P={P}: {(time.perf_counter() - t0) / 20 * 1e6:.0f} us per group call")
    grp.close()
    # random walks: 16384 walks x 80 steps per rank
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, cfg.batch, devices=[0] * P, max_walks=16384, max_walk_length=80)
    rng = np.random.default_rng(0)
    st = [torch.from_numpy(rng.integers(int(bnds[r]), int(bnds[r + 1]), 16384).astype(np.int32)).cuda()
          for r in range(P)]
    for it in range(8):
        if it == 3:
            torch.cuda.synchronize()
            t0 = time.perf_counter()
        grp.random_walk(st, 80, 5 + it)
    torch.cuda.synchronize()
    print(f"random walks ({mode}) P={P}: {(time.perf_counter() - t0) / 5 * 1e3:.2f} ms per group call "
          f"(16384 walks x 80 steps per rank)")
    grp.close()
