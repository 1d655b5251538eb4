"""Phase timings of the world > 1 persistent kernel (k_csp_multi) with P
virtual ranks on one GPU (each on 1/P of the SMs): rank 0's globaltimer stamps
at every grid barrier.  P=2 python tools/phases_multi.py [calls]"""
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
    shards.append((sip, six, datagen.features(lo, hi, 4)))
grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, cfg.batch, devices=[0] * P)
train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
per_rank = [datagen.rank_seed_batches(train, bnds, r, cfg.batch, 0) for r in range(P)]
calls = int(sys.argv[1]) if len(sys.argv) > 1 else 12
acc = []
for it in range(calls):
    grp.sample([torch.from_numpy(per_rank[r][it % len(per_rank[r])]).cuda() for r in range(P)], 0x5EED + it)
    torch.cuda.synchronize()
    ws = grp.samplers[0].workspace[:1024].view(torch.int64)
    t = ws[81:105].cpu().numpy()
    nb = sum(1 for g in range(1, 23) if t[g] > t[0])
    stamps = np.array([t[0]] + [t[g] for g in range(1, nb + 1)] + [t[23]], dtype=np.int64)
    acc.append(np.diff(stamps) / 1e3)
n = min(len(a) for a in acc[2:])
a = np.median(np.array([x[:n] for x in acc[2:]]), axis=0)
print(f"P={P}: rank 0 call {a.sum():.1f} us, {n} phases (barrier to barrier):")
print("  " + " ".join(f"{x:.1f}" for x in a))
grp.close()
