"""Phase timings of the persistent kernel in bench.py's exact launch
configuration (K concurrent pipelined step streams, each launch on 1/K of the
SMs): the globaltimer stamps block 0 of the last launch on workspace 0 leaves
at every grid barrier, median over repetitions.
K=4 python tools/phases_bench.py [reps]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import datagen
import paper_conf_ppopp_caiz0zszck23_b200 as pkg

cfg = datagen.CONFIGS[os.environ.get("CFG", "products")]
K = int(os.environ.get("K", "4"))
ip, ix = datagen.make_graph(cfg)
feats = datagen.features(0, cfg.num_nodes, cfg.dim)
bnds = datagen.bounds(cfg.num_nodes, 1)
biased = bool(os.environ.get("BIASED"))
ew = datagen.edge_weights(ix, datagen.node_weights(cfg.num_nodes)) if biased else None
s = pkg.Sampler(bnds, ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2 * K, n_workspaces=K, edge_weights=ew)
sms = torch.cuda.get_device_properties(0).multi_processor_count
pkg.dsp_set_persistent_blocks(s.ctx, sms // K if K > 1 else 0)
train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
batches = torch.from_numpy(datagen.rank_seed_batches(train, bnds, 0, cfg.batch, 0)).cuda()
L = len(cfg.fanouts)
streams = [torch.cuda.Stream() for _ in range(K)]
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 12
sz = torch.zeros((64, 3 * L), dtype=torch.int64).pin_memory()
acc, loader = [], []
i = 0
for rep in range(reps):
    for j in range(4 * K):     # 4 launches per stream, the last on workspace 0 is stamped
        s.sample_gather(batches[i % len(batches)], 100 + i, slot=i % (2 * K), sizes_out=sz[i % 64], pipelined=True,
                        ws=i % K, stream=streams[i % K], biased=biased)
        i += 1
    torch.cuda.synchronize()
    h = s.workspaces[0][:1024].view(torch.int64)
    t = h[81:105].cpu().numpy()
    ta = h[105:129].cpu().numpy()
    nb = sum(1 for g in range(1, 22) if t[g] > t[0])
    st = [t[0]] + [t[g] for g in range(1, nb + 1)] + [t[23]]
    work = [ta[g] - t[g - 1] for g in range(1, nb + 1)]
    if rep >= 2:
        acc.append(np.concatenate([np.diff(np.array(st, dtype=np.int64)) / 1e3, np.array(work) / 1e3]))
        loader.append((t[22] - t[0]) / 1e3)
s.flush()
torch.cuda.synchronize()
n = min(len(a) for a in acc)
a_all = np.median(np.array([a[:n] for a in acc]), axis=0)
nph = (n + 1) // 2
a, w0 = a_all[:nph], a_all[nph:]
print(f"K={K} launch on {sms // K if K > 1 else sms} SMs: total {a.sum():.1f} us, loader warp 0 of block 0 done at "
      f"{np.median(loader):.1f} us; {nph} phases (exit-to-exit, block 0's own work before arriving):")
for j, v in enumerate(a):
    print(f"   phase {j:2d} {v:8.1f} us" + (f"   block0 {w0[j]:6.1f}" if j < len(w0) else ""))
