"""Stage-by-stage (world > 1) path cost on one GPU: P virtual ranks of the
products graph driven by dsp_sample_group on one stream (all ranks' stages
serialised on the device).  Prints per-call time and the per-kernel share
(run under ncu for the launch list).  P=... python tools/virtual_time.py"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import datagen
import paper_conf_ppopp_caiz0zszck23_b200 as pkg

cfg = datagen.CONFIGS[os.environ.get("CFG", "products")]
P = int(os.environ.get("P", "2"))
ip, ix = datagen.make_graph(cfg)
bnds = datagen.bounds(cfg.num_nodes, P)
shards = []
for r in range(P):
    lo, hi = int(bnds[r]), int(bnds[r + 1])
    sip, six = datagen.shard(ip, ix, lo, hi)
    shards.append((sip, six, datagen.features(lo, hi, cfg.dim)))
grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, cfg.batch, devices=[0] * P)
train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
per_rank = [datagen.rank_seed_batches(train, bnds, r, cfg.batch, 0) for r in range(P)]
dev = [[torch.from_numpy(b).cuda() for b in x[:30]] for x in per_rank]
for it in range(25):
    if it == 5:
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        edges = 0
    res = grp.sample([dev[r][it % len(dev[r])] for r in range(P)], 0x5EED + it)
    if it >= 5:
        edges += sum(b.num_edges for rr in res for b in rr)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 20
print(f"P={P} virtual ranks on one GPU: {ms * 1e3:.0f} us per group call ({P} ranks' batches), "
      f"{ms * 1e3 / P:.0f} us per rank-batch, {edges / 20 / P / 1e3:.0f} k edges per rank-batch")
