"""bench.py -- DSP CSP sampling + feature gather throughput on B200.

One step = one pass of the whole hot path over one mini-batch per GPU:
dsp_sample (CSP over all layers: shuffle / sample / reshuffle / relabel,
SURVEY.md 8(a) a1-a7) followed by dsp_gather_features for the sampled nodes
(a8).  Workload at N=1: BASELINE.json configs[1] (ogbn-products-shaped
synthetic R-MAT, fan-out [15,10,5], 1024 seeds/GPU, dim 100); N>1:
configs[2] (the same graph partitioned over N GPUs, weak scaling).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl dsp|reference]

Prints ONE JSON line on rank 0.  `value` = sampled edges/s over all ranks
(sum of every block's num_edges / max-over-ranks device time).  The
reference arm (--impl reference) times the CPU oracle on the host cores on a
bounded sample of the same workload (the paper's system is not available;
see DESIGN.md "Measurement").
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "sampled edges/sec + feature GB/s at 1/2/4/8 B200; % of HBM/NVLink roofline"


def reduce_max_over_ranks(x: float) -> float:
    """Max of a per-rank device time over all ranks (1 rank: identity)."""
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(x)
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def reduce_sum_over_ranks(x: float) -> float:
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(x)
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


def barrier():
    if dist.is_available() and dist.is_initialized():
        dist.barrier()


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self._stop = threading.Event()
        self._t = threading.Thread(target=self._run, daemon=True)

    def _run(self):
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                     timeout=5).stdout.strip()
                if out:
                    self.samples.append([x.strip() for x in out.split(",")])
            except Exception:
                pass
            self._stop.wait(0.1)

    def __enter__(self):
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=10)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if s[2 + i] == "Active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


def ncu_traffic(kernel: str):
    """DRAM bytes per launch of `kernel` from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        d = json.load(open(p))
        v = d.get(kernel)
        if isinstance(v, dict):
            return v.get("dram_bytes_per_launch")
    return None


def setup_dist(n_gpus: int):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != n_gpus:
        if world == 1 and n_gpus > 1:
            raise SystemExit(f"--gpus {n_gpus} needs torchrun with {n_gpus} processes")
        raise SystemExit(f"WORLD_SIZE={world} != --gpus {n_gpus}")
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    return rank, world, local


def load_workload(cfg_name, rank, world):
    import datagen
    cfg = datagen.CONFIGS[cfg_name]
    ip, ix = datagen.make_graph(cfg)
    bnds = datagen.bounds(cfg.num_nodes, world)
    lo, hi = int(bnds[rank]), int(bnds[rank + 1])
    sip, six = datagen.shard(ip, ix, lo, hi)
    feats = datagen.features(lo, hi, cfg.dim)
    train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
    return cfg, ip, ix, bnds, sip, six, feats, train


# --------------------------------------------------------------- reference

def run_reference(args):
    """The CPU oracle, as it stands, on the host cores: each step = one batch
    of the same workload (oracle.sample + oracle.gather), bounded by
    --ref-max-seconds of CPU work."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import datagen
    import oracle
    cfg, ip, ix, bnds, sip, six, feats, train = load_workload(args.config, 0, 1)
    batches = datagen.rank_seed_batches(train, bnds, 0, cfg.batch, 0)
    edges = rows = 0
    steps_done = 0
    t_all = 0.0
    for step in range(args.warmup + args.steps):
        seeds = batches[step % len(batches)]
        t0 = time.perf_counter()
        blocks = oracle.sample(ip, ix, seeds, cfg.fanouts, datagen.BASE_SEED + step)
        out = oracle.gather(feats, blocks[-1]["src_ids"])
        dt = time.perf_counter() - t0
        if step >= args.warmup:
            t_all += dt
            edges += sum(int(b["num_edges"]) for b in blocks)
            rows += out.shape[0]
            steps_done += 1
            if t_all > args.ref_max_seconds:
                break
    value = edges / t_all
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "edges/s", "n_gpus": args.gpus,
        "steps": steps_done, "warmup": args.warmup, "ms_per_step": 1e3 * t_all / steps_done,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32+f32",
        "data": "synthetic", "config": {"workload": cfg.name, "fanouts": list(cfg.fanouts), "batch_per_gpu": cfg.batch,
                                         "num_nodes": cfg.num_nodes, "dim": cfg.dim},
        "cpu_baseline": {"value": value, "unit": "edges/s", "cores": 1, "kind": "oracle",
                         "sample": f"{steps_done} batches of {cfg.batch} seeds (oracle.sample + oracle.gather)"},
        "e2e": {"value": value, "unit": "edges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "feature_GBps": rows * cfg.dim * 4 / t_all / 1e9,
        "seeds_per_s": steps_done * cfg.batch / t_all,
    }
    print(json.dumps(line), flush=True)
    return 0


def cpu_baseline(cfg, ip, ix, feats, batches, seconds: float):
    import datagen
    import oracle
    t_all = 0.0
    edges = 0
    n = 0
    while t_all < seconds and n < len(batches):
        seeds = batches[n]
        t0 = time.perf_counter()
        blocks = oracle.sample(ip, ix, seeds, cfg.fanouts, datagen.BASE_SEED + n)
        oracle.gather(feats, blocks[-1]["src_ids"])
        t_all += time.perf_counter() - t0
        edges += sum(int(b["num_edges"]) for b in blocks)
        n += 1
    return {"value": edges / t_all, "unit": "edges/s", "cores": 1, "kind": "oracle",
            "sample": f"{n} products batches of {cfg.batch} seeds, single host thread "
                      f"(oracle.sample + oracle.gather), {t_all:.1f} s"}


# ----------------------------------------------------------------- product

def run_dsp(args):
    import datagen
    import paper_conf_ppopp_caiz0zszck23_b200 as pkg
    rank, world, local = setup_dist(args.gpus)
    torch.cuda.set_device(local)
    cfg_name = args.config
    cfg, ip, ix, bnds, sip, six, feats, train = load_workload(cfg_name, rank, world)
    ex = pkg.torch_exchange() if world > 1 else None
    s = pkg.Sampler(bnds, sip, six, feats, cfg.fanouts, cfg.batch, rank=rank, world_size=world,
                    device=local, exchange=ex)
    steps_epoch = datagen.steps_per_epoch(train, bnds, cfg.batch)
    batches = datagen.rank_seed_batches(train, bnds, rank, cfg.batch, 0)[:steps_epoch]
    need = args.warmup + args.steps
    dev_batches = torch.from_numpy(np.ascontiguousarray(batches)).cuda()   # inputs resident in HBM
    max_rows = s.max_src[-1]
    out = torch.empty((max_rows, cfg.dim), dtype=torch.float32, device="cuda")
    stream = torch.cuda.current_stream()

    def step(i, timed_gather=None):
        seeds = dev_batches[i % len(batches)]
        blocks = s.sample(seeds, datagen.BASE_SEED + i)
        U = blocks[-1].num_src
        if timed_gather is not None:
            timed_gather[0].record(stream)
        s.gather(blocks[-1].src_ids, out[:U])
        if timed_gather is not None:
            timed_gather[1].record(stream)
        return blocks

    for i in range(args.warmup):
        step(i)
    s.sync()
    barrier()
    torch.cuda.synchronize()

    # ---- timed region: K steps, inputs resident, device time via CUDA events
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    gev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    edges = rows = seeds_n = 0
    with ClockSampler(local) as clk:
        ev0.record(stream)
        for j in range(args.steps):
            blocks = step(args.warmup + j, gev[j])
            edges += sum(b.num_edges for b in blocks)
            rows += blocks[-1].num_src
            seeds_n += blocks[0].num_dst
        ev1.record(stream)
        s.sync()
        torch.cuda.synchronize()
    barrier()
    t_ms = ev0.elapsed_time(ev1)
    g_ms = [a.elapsed_time(b) for a, b in gev]
    t_max = reduce_max_over_ranks(t_ms)
    tot_edges = reduce_sum_over_ranks(edges)
    tot_rows = reduce_sum_over_ranks(rows)
    tot_seeds = reduce_sum_over_ranks(seeds_n)
    g_mean = float(np.mean(g_ms))
    gather_bytes_per_launch = 2.0 * (rows / args.steps) * cfg.dim * 4      # read + write, algorithmic
    achieved = gather_bytes_per_launch / (g_mean * 1e-3) / 1e9
    peak, peak_kind = measured_peaks()

    # ---- e2e: the same steps through the C ABI with HOST buffers: pinned seeds
    # H2D, sample, gather, D2H of the blocks and the gathered features
    h_seeds = torch.from_numpy(np.ascontiguousarray(batches)).pin_memory()
    h_feat = torch.empty((max_rows, cfg.dim), dtype=torch.float32).pin_memory()
    h_blk = [tuple(torch.empty(x.numel(), dtype=torch.int32).pin_memory() for x in bufs) for bufs in s._bufs]
    d_seed = torch.empty(cfg.batch, dtype=torch.int32, device="cuda")
    e2e_steps = max(3, min(args.steps, 20))
    h2d = d2h = 0
    barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e2e_edges = 0
    e0.record(stream)
    for j in range(e2e_steps):
        i = args.warmup + j
        d_seed.copy_(h_seeds[i % len(batches)], non_blocking=True)
        h2d += d_seed.numel() * 4
        blocks = s.sample(d_seed, datagen.BASE_SEED + i)
        U = blocks[-1].num_src
        s.gather(blocks[-1].src_ids, out[:U])
        for b, hb in zip(blocks, h_blk):
            hb[0][: b.num_dst + 1].copy_(b.indptr, non_blocking=True)
            hb[1][: b.num_edges].copy_(b.indices, non_blocking=True)
            hb[2][: b.num_src].copy_(b.src_ids, non_blocking=True)
            d2h += 4 * (b.num_dst + 1 + b.num_edges + b.num_src)
        h_feat[:U].copy_(out[:U], non_blocking=True)
        d2h += U * cfg.dim * 4
        e2e_edges += sum(b.num_edges for b in blocks)
    e1.record(stream)
    torch.cuda.synchronize()
    e2e_ms = reduce_max_over_ranks(e0.elapsed_time(e1))
    e2e_edges = reduce_sum_over_ranks(e2e_edges)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(cfg, ip, ix, feats, batches, args.cpu_seconds)

    kern_per_step = (3 if world == 1 else 5) * len(cfg.fanouts) + 1
    if rank == 0:
        line = {
            "metric": METRIC, "value": tot_edges / (t_max * 1e-3), "unit": "edges/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": t_max / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32+f32",
            "data": "synthetic",
            "config": {"workload": cfg.name if world == 1 else f"{cfg.name}-P{world}",
                       "fanouts": list(cfg.fanouts), "batch_per_gpu": cfg.batch, "num_nodes": cfg.num_nodes,
                       "nnz": int(ip[-1]), "dim": cfg.dim, "parallelism": f"csp{world}",
                       "l2": "inputs larger than L2 (CSR + features >> 126 MB; per-step gather moves ~0.5 GB)"},
            "seeds_per_s": tot_seeds / (t_max * 1e-3),
            "feature_GBps": tot_rows * cfg.dim * 4 / (t_max * 1e-3) / 1e9,
            "gather_kernel_GBps": achieved,
            "edges_per_step": tot_edges / args.steps / world,
            "rows_per_step": tot_rows / args.steps / world,
            "roofline": {"kernel": "k_gather", "bound": "hbm" if world == 1 else "nvlink",
                         "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                         "traffic": ncu_traffic("k_gather"), "peak_kind": peak_kind,
                         "algorithmic_bytes_per_launch": gather_bytes_per_launch,
                         "gather_ms_mean": g_mean, "gather_share_of_step": g_mean / (t_ms / args.steps)},
            "cpu_baseline": cpu,
            "e2e": {"value": e2e_edges / (e2e_ms * 1e-3), "unit": "edges/s",
                    "h2d_bytes_per_step": h2d // e2e_steps, "d2h_bytes_per_step": d2h // e2e_steps,
                    "steps": e2e_steps},
            "gpu_launches": kern_per_step * args.steps,
            "clocks": clk.summary(),
        }
        print(json.dumps(line), flush=True)
    s.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["dsp", "reference"], default="dsp")
    ap.add_argument("--config", default=None)
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--ref-max-seconds", type=float, default=60.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args(argv)
    if args.warmup < 3:
        raise SystemExit("--warmup must be >= 3")
    if args.config is None:
        args.config = "products"
    if args.impl == "reference":
        return run_reference(args)
    return run_dsp(args)


if __name__ == "__main__":
    sys.exit(main())
