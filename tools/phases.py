"""Phase timings of the persistent kernel (globaltimer stamps in the workspace
header) on the products workload: python tools/phases.py [steps]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import datagen
import paper_conf_ppopp_caiz0zszck23_b200 as pkg

cfg = datagen.CONFIGS[os.environ.get("CFG", "products")]
ip, ix = datagen.make_graph(cfg)
feats = datagen.features(0, cfg.num_nodes, cfg.dim)
bnds = datagen.bounds(cfg.num_nodes, 1)
ew = datagen.edge_weights(ix, datagen.node_weights(cfg.num_nodes)) if "biased" in os.environ.get("MODES", "") else None
s = pkg.Sampler(bnds, ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2, edge_weights=ew)
train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
batches = datagen.rank_seed_batches(train, bnds, 0, cfg.batch, 0)
steps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
rows = []
modes = ["sample", "sample_gather", "pipelined"] if not os.environ.get("MODES") else os.environ["MODES"].split(",")
for mode in modes:
    acc = []
    for i in range(steps):
        seeds = torch.from_numpy(batches[i]).cuda()
        if os.environ.get("EMPTY"):
            seeds = seeds[:0]
        if mode == "sample":
            s.sample(seeds, 100 + i)
        elif mode == "biased":
            s.sample(seeds, 100 + i, biased=True)
        elif mode == "pipelined":
            s.sample_gather(seeds, 100 + i, slot=i % 2, pipelined=True)
            s.sync()
        else:
            s.sample_gather(seeds, 100 + i, slot=i % 2)
        t = s.workspace[:1024].view(torch.int64)[81:105].cpu().numpy()
        ta = s.workspace[:1024].view(torch.int64)[105:129].cpu().numpy()
        nb = sum(1 for g in range(1, 22) if t[g] > t[0])
        if mode == "pipelined" and i == steps - 1:
            hv = s.workspace[:1024].view(torch.int32)
            print("  pipelined: loader warp0/block0 done at %.1f us; chunks loader %d helper %d" % (
                (t[22] - t[0]) / 1e3, int(hv[158]), int(hv[159])))
        stamps = [t[0]] + [t[g] for g in range(1, nb + 1)] + [t[23]]
        work = [ta[g] - (t[g - 1]) for g in range(1, nb + 1)]
        acc.append(np.concatenate([np.diff(np.array(stamps, dtype=np.int64)) / 1e3, np.array(work) / 1e3]))
    a_all = np.median(np.array(acc[2:]), axis=0)
    nph = (len(a_all) + 1) // 2
    a, w0 = a_all[:nph], a_all[nph:]
    L = len(cfg.fanouts)
    names = [f"{x}{l}" for l in range(L) for x in ("sample", "scan-pass1", "scan-pass2")] + ["indices+gather"]
    print(mode, "total %.1f us   (phase = exit-to-exit; block0 = block 0's own work before arriving)" % a.sum())
    for j, (n, v) in enumerate(zip(names, a)):
        extra = f"   block0 {w0[j]:6.1f}" if j < len(w0) else ""
        print(f"   {n:16s} {v:8.1f} us{extra}")
dbg = s.workspace[:2048].view(torch.int64)[129:161].cpu().numpy()
if dbg.any():
    for l in range(len(cfg.fanouts)):
        d = dbg[8 * l: 8 * l + 8]
        if d[0]:
            print(f"layer {l} thread 0 chain (ns from iteration start):", [int(x - d[0]) if x else None for x in d[1:6]])
