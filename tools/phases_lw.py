"""Phase timings of the world-1 layer-wise persistent kernel (k_lw_persistent):
globaltimer stamps at its grid barriers, products, Table 7 sizes (1000, 1000).
python tools/phases_lw.py [calls]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import datagen
import paper_conf_ppopp_caiz0zszck23_b200 as pkg

cfg = datagen.CONFIGS[os.environ.get("CFG", "products")]
ip, ix = datagen.make_graph(cfg)
bnds = datagen.bounds(cfg.num_nodes, 1)
sizes = (1000, 1000)
s = pkg.Sampler(bnds, ip, ix, datagen.features(0, cfg.num_nodes, 4), sizes, cfg.batch, scheme="layer")
train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
batches = datagen.rank_seed_batches(train, bnds, 0, cfg.batch, 0)
calls = int(sys.argv[1]) if len(sys.argv) > 1 else 12
acc = []
for i in range(calls):
    s.sample(torch.from_numpy(batches[i]).cuda(), 100 + i)
    t = s.workspace[:1024].view(torch.int64)[81:105].cpu().numpy()
    nb = sum(1 for g in range(1, 23) if t[g] > t[0])
    if t[0] == 0 or nb == 0:
        print("no stamps (staged path?)"); break
    acc.append(np.diff(np.array([t[0]] + [t[g] for g in range(1, nb + 1)], dtype=np.int64)) / 1e3)
if acc:
    a = np.median(np.array(acc[2:]), axis=0)
    names = [f"{x}{l}" for l in range(len(sizes)) for x in ("alloc", "sample", "big", "collect", "finish")]
    print("total %.1f us" % a.sum())
    for n, v in zip(names, a):
        print(f"   {n:10s} {v:7.1f} us")
dbg = s.workspace[:2048].view(torch.int64)[129 + 16: 129 + 24].cpu().numpy()
if dbg.any():
    for l in range(2):
        d = dbg[4 * l: 4 * l + 4]
        print(f"alloc{l} sub-steps (us): W+scan {(d[1]-d[0])/1e3:.1f}  draws {(d[2]-d[1])/1e3:.1f}  offsets+tasks {(d[3]-d[2])/1e3:.1f}")
