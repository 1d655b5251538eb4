"""Experiment: K concurrent persistent-kernel steps on K streams (each on
148/K blocks, own workspace + outputs) vs one pipelined stream."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import datagen
import paper_conf_ppopp_caiz0zszck23_b200 as pkg

cfg = datagen.CONFIGS[os.environ.get("CFG", "products")]
ip, ix = datagen.make_graph(cfg)
feats = datagen.features(0, cfg.num_nodes, cfg.dim)
if os.environ.get("DIM"):  # e.g. DIM=4: (almost) no gather, sampling throughput alone
    feats = np.ascontiguousarray(feats[:, : int(os.environ["DIM"])])
bnds = datagen.bounds(cfg.num_nodes, 1)
KMAX = 4
s = pkg.Sampler(bnds, ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2 * KMAX, n_workspaces=KMAX)
train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
batches = torch.from_numpy(datagen.rank_seed_batches(train, bnds, 0, cfg.batch, 0)).cuda()
L = len(cfg.fanouts)
sizes = torch.zeros((4096, 3 * L), dtype=torch.int64).pin_memory()
steps = 60
main = torch.cuda.current_stream()
for K in [int(x) for x in os.environ.get("KS", "1,2,3,4").split(",")]:
    pkg.dsp_set_persistent_blocks(s.ctx, 0 if K == 1 else 148 // K)
    streams = [torch.cuda.Stream() for _ in range(K)]
    for pipelined in (False, True):
        for rep in range(2):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(main)
            for st in streams:
                st.wait_stream(main)
            for i in range(steps):
                j = i % K
                s.sample_gather(batches[i % len(batches)], 7 + i, slot=i % (2 * K), sizes_out=sizes[i],
                                async_=True, pipelined=pipelined, ws=j, stream=streams[j])
            if pipelined:
                for st in streams:
                    with torch.cuda.stream(st):
                        s.flush()
            for st in streams:
                main.wait_stream(st)
            e1.record(main)
            torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        edges = sizes[:steps, 2::3].sum().item()
        print(f"K={K} pipelined={pipelined}: {1e3 * ms / steps:.1f} us/step, {edges / ms / 1e6:.2f} G edges/s")
