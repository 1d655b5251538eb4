"""Per-warp cycle breakdown of the biased sampling phase of one layer
(DSP_BPROF=<layer> experiment build, DSP_LIB=...): python tools/bprof.py"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import datagen
import paper_conf_ppopp_caiz0zszck23_b200 as pkg

cfg = datagen.CONFIGS["products"]
ip, ix = datagen.make_graph(cfg)
feats = datagen.features(0, cfg.num_nodes, cfg.dim)
bnds = datagen.bounds(cfg.num_nodes, 1)
ew = datagen.edge_weights(ix, datagen.node_weights(cfg.num_nodes))
s = pkg.Sampler(bnds, ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2, edge_weights=ew)
train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
batches = datagen.rank_seed_batches(train, bnds, 0, cfg.batch, 0)
for i in range(6):
    s.sample(torch.from_numpy(batches[i]).cuda(), 100 + i, biased=True)
    d = s.workspace[:2048].view(torch.int64)[129:161].cpu().numpy().astype(np.float64)
nw = 148 * 32
names = ["claim fetch", "g8 passes", "g16 passes", "g32 passes", "warp-wide", "g8 nodes", "g16 nodes", "g32 nodes",
         "warp nodes", "claims", "phase total", "g8: ctx+philox", "g8: loads+scans", "g8: rounds", "g8: output", "g8 passes"]
for j, n in enumerate(names):
    v = d[j]
    if j in (0, 1, 2, 3, 4, 10, 11, 12, 13, 14):
        print(f"{n:12s} {v / nw:10.0f} cycles per warp ({v / nw / 1.9e3:6.1f} us)")
    else:
        print(f"{n:12s} {v:10.0f}")
