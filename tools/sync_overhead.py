"""Where the synchronous fused call's time goes (products, one B200): device
time of the call (CUDA events around it on its stream), host wall time per
call, and the binding's own Python time (ctypes call excluded).
python tools/sync_overhead.py"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import datagen
import paper_conf_ppopp_caiz0zszck23_b200 as pkg

cfg = datagen.CONFIGS["products"]
ip, ix = datagen.make_graph(cfg)
feats = datagen.features(0, cfg.num_nodes, cfg.dim)
bnds = datagen.bounds(cfg.num_nodes, 1)
s = pkg.Sampler(bnds, ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2)
train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
batches = torch.from_numpy(datagen.rank_seed_batches(train, bnds, 0, cfg.batch, 0)[:64]).cuda()
st = torch.cuda.current_stream()
for i in range(5):
    s.sample_gather(batches[i], 100 + i, slot=0)
torch.cuda.synchronize()
n = 50
ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n)]
t0 = time.perf_counter()
for i in range(n):
    ev[i][0].record(st)
    blocks, feat = s.sample_gather(batches[i % 64], 200 + i, slot=i % 2)
    ev[i][1].record(st)
wall = (time.perf_counter() - t0) / n * 1e6
torch.cuda.synchronize()
dev = np.mean([a.elapsed_time(b) for a, b in ev]) * 1e3
# the same calls, asynchronous (no host wait), back to back: device throughput of the fused call
t0 = time.perf_counter()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(st)
for i in range(n):
    s.sample_gather(batches[i % 64], 300 + i, slot=i % 2, async_=True)
e1.record(st)
issue = (time.perf_counter() - t0) / n * 1e6
torch.cuda.synchronize()
adev = e0.elapsed_time(e1) / n * 1e3
print(f"synchronous fused call: {wall:.1f} us wall per call, {dev:.1f} us between its events (incl. the host "
      f"round trip inside); asynchronous back to back: {adev:.1f} us device per call, {issue:.1f} us host issue per call")
s.close()
