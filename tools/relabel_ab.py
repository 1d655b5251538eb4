"""A/B of the relabel map (direct vs hash) on one graph: CFG=papers python tools/relabel_ab.py
Throughput of pipelined steps on K concurrent streams, same seeds, both modes built over one
host copy of the graph."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import datagen
import paper_conf_ppopp_caiz0zszck23_b200 as pkg

cfg = datagen.CONFIGS[os.environ.get("CFG", "papers")]
t0 = time.time()
ip, ix = datagen.make_graph(cfg)
feats = datagen.features(0, cfg.num_nodes, cfg.dim)
print(f"graph {cfg.name}: {time.time() - t0:.0f} s", flush=True)
bnds = datagen.bounds(cfg.num_nodes, 1)
train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
batches = torch.from_numpy(datagen.rank_seed_batches(train, bnds, 0, cfg.batch, 0)[:64]).cuda()
L = len(cfg.fanouts)
steps = 40
for mode in os.environ.get("MODES", "hash,direct").split(","):
    for K in (1, 2):
        s = pkg.Sampler(bnds, ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2 * K, n_workspaces=K,
                        options={pkg.dsp.DSP_OPT_RELABEL_MAP: pkg.dsp.RELABEL_MAPS[mode]})
        if K > 1:
            pkg.dsp_set_persistent_blocks(s.ctx, 148 // K)
        sizes = torch.zeros((256, 3 * L), dtype=torch.int64).pin_memory()
        main = torch.cuda.current_stream()
        streams = [torch.cuda.Stream() for _ in range(K)]
        for rep in range(2):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(main)
            for st in streams:
                st.wait_stream(main)
            for i in range(steps):
                j = i % K
                s.sample_gather(batches[i % len(batches)], 7 + i, slot=i % (2 * K), sizes_out=sizes[i],
                                async_=True, pipelined=True, ws=j, stream=streams[j])
            for st in streams:
                with torch.cuda.stream(st):
                    s.flush()
                main.wait_stream(st)
            e1.record(main)
            torch.cuda.synchronize()
        s.sync()
        ms = e0.elapsed_time(e1)
        edges = sizes[:steps, 2::3].sum().item()
        print(f"{mode} K={K}: {1e3 * ms / steps:.1f} us/step, {edges / ms / 1e6:.2f} G edges/s", flush=True)
        s.close()
        torch.cuda.empty_cache()
