"""World > 1 path on one GPU: P virtual ranks of the products graph (one
persistent k_csp_multi launch per rank, exchanges through peer memory of the
same device) driven by dsp_sample_group.  K = exchange channels: K
asynchronous group calls in flight on K streams, each rank's launch on
1/(P*K) of the SMs (DSP_OPT_EXCHANGE_CHANNELS, the paper's concurrent
pipeline stages).  Prints us per rank-batch (sampling only).
P=2 K=4 python tools/virtual_time.py"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import datagen
import paper_conf_ppopp_caiz0zszck23_b200 as pkg

cfg = datagen.CONFIGS[os.environ.get("CFG", "products")]
ip, ix = datagen.make_graph(cfg)
train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
sms = torch.cuda.get_device_properties(0).multi_processor_count
for P in [int(x) for x in os.environ.get("P", "2,4,8").split(",")]:
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, datagen.features(lo, hi, 4)))
    per_rank = [datagen.rank_seed_batches(train, bnds, r, cfg.batch, 0) for r in range(P)]
    dev = [[torch.from_numpy(b).cuda() for b in x[:32]] for x in per_rank]
    for K in [int(x) for x in os.environ.get("K", "1,2,4").split(",")]:
        if P * K > sms:
            continue
        grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, cfg.batch, devices=[0] * P, n_workspaces=K, n_slots=K,
                             options={pkg.dsp.DSP_OPT_EXCHANGE_CHANNELS: K})
        for s in grp.samplers:
            pkg.dsp_set_persistent_blocks(s.ctx, sms // (P * K))
        edges = 0
        for it in range(8):   # sizes of the timed calls (deterministic), synchronous
            res = grp.sample([dev[r][it % 32] for r in range(P)], 0x5EED + it)
            edges += sum(b.num_edges for rr in res for b in rr)
        streams = [torch.cuda.Stream() for _ in range(K)]
        n = 8 * K * 4
        for rep in range(2):
            torch.cuda.synchronize()
            main = torch.cuda.current_stream()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(main)
            for st in streams:
                st.wait_stream(main)
            for it in range(n):
                grp.sample([dev[r][it % 8] for r in range(P)], 0x5EED + it % 8, async_=True, ws=it % K,
                           slot=it % K, stream=streams[it % K])
            for st in streams:
                main.wait_stream(st)
            e1.record(main)
            torch.cuda.synchronize()
        for s in grp.samplers:
            s.sync()
        us = e0.elapsed_time(e1) * 1e3 / n
        print(f"P={P} K={K}: {us:.0f} us per group call ({P} rank-batches), {us / P:.1f} us per rank-batch, "
              f"{edges / 8 / P / 1e3:.0f} k edges per rank-batch, launches on {sms // (P * K)} SMs", flush=True)
        grp.close()
