"""Diagnostic: host time of each call in a bench-like timed loop (3 streams,
pipelined), after a warm-up + flush, with and without the NVML clock sampler."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import datagen
import paper_conf_ppopp_caiz0zszck23_b200 as pkg
import bench

cfg = datagen.CONFIGS["products"]
ip, ix = datagen.make_graph(cfg)
feats = datagen.features(0, cfg.num_nodes, cfg.dim)
bnds = datagen.bounds(cfg.num_nodes, 1)
K = 3
s = pkg.Sampler(bnds, ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2 * K, n_workspaces=K)
pkg.dsp_set_persistent_blocks(s.ctx, 148 // K)
train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
batches = torch.from_numpy(datagen.rank_seed_batches(train, bnds, 0, cfg.batch, 0)).cuda()
sizes = torch.zeros((4096, 9), dtype=torch.int64).pin_memory()
main = torch.cuda.current_stream()
streams = [torch.cuda.Stream() for _ in range(K)]


def run(n, tag, clocks):
    torch.cuda.synchronize()
    ts = []
    ctx = bench.ClockSampler(0) if clocks else None
    if ctx: ctx.__enter__()
    t0 = time.perf_counter()
    for st in streams: st.wait_stream(main)
    ts.append(("fork", time.perf_counter()))
    for i in range(n):
        j = i % K
        s.sample_gather(batches[i % len(batches)], 7 + i, slot=i % (2 * K), sizes_out=sizes[i], async_=True,
                        pipelined=True, ws=j, stream=streams[j])
        ts.append((f"step{i}", time.perf_counter()))
    for st in streams:
        with torch.cuda.stream(st):
            s.flush()
        ts.append(("flush", time.perf_counter()))
    for st in streams: main.wait_stream(st)
    ts.append(("join", time.perf_counter()))
    torch.cuda.synchronize()
    ts.append(("sync", time.perf_counter()))
    if ctx: ctx.__exit__()
    prev = t0
    out = []
    for name, t in ts:
        out.append(f"{name}:{1e6 * (t - prev):.0f}")
        prev = t
    print(tag, "clocks" if clocks else "noclk", " ".join(out))


for rep in range(3):
    run(10, f"rep{rep}", False)
    run(10, f"rep{rep}", True)
