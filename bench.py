"""bench.py -- DSP CSP sampling + feature gather throughput on B200.

One step = one pass of the whole hot path over one mini-batch per GPU: one
dsp_sample_gather call -- CSP over all layers (shuffle / sample / reshuffle /
relabel) and the feature gather of the sampled nodes
(a8) -- pipelined as in the paper: the launch of step t samples
batch t while its loader warps gather batch t-1; at N=1 two step streams run
concurrently on 74 SMs each (biased / layer-wise: four on 37).  Workload at N=1: BASELINE.json configs[1]
(ogbn-products-shaped synthetic R-MAT, fan-out [15,10,5], 1024 seeds/GPU,
dim 100); N>1: configs[2] (the same graph partitioned over N GPUs, weak
scaling).  --config papers | friendster, --scheme biased | layer | walk and
--hot-frac select the other workloads.

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
    """SM clocks + throttle reasons sampled (NVML, every 2 ms) during the timed region."""

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self._stop = threading.Event()
        self._t = threading.Thread(target=self._run, daemon=True)

    def _run(self):
        try:
            import pynvml as nv
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.index)
            mx = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
            bits = {"hw_slowdown": nv.nvmlClocksThrottleReasonHwSlowdown,
                    "hw_thermal_slowdown": getattr(nv, "nvmlClocksThrottleReasonHwThermalSlowdown", 0x40),
                    "sw_thermal_slowdown": getattr(nv, "nvmlClocksThrottleReasonSwThermalSlowdown", 0x20),
                    "sw_power_cap": nv.nvmlClocksThrottleReasonSwPowerCap}
            while not self._stop.is_set():
                sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                r = nv.nvmlDeviceGetCurrentClocksThrottleReasons(h)
                self.samples.append((sm, mx, [k for k, b in bits.items() if r & b]))
                self._stop.wait(0.002)
        except Exception as e:  # NVML unavailable: fall back to one nvidia-smi query
            self.error = repr(e)

    def __enter__(self):
        self._t.start()
        t0 = time.time()
        while not self.samples and time.time() - t0 < 5.0 and self._t.is_alive():
            time.sleep(0.005)   # the first sample is taken before the timed region starts
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=10)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"],
                    "error": getattr(self, "error", None)}
        sm = [s[0] for s in self.samples]
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": max(s[1] for s in self.samples),
                "reasons": sorted({x for s in self.samples for x in s[2]}), "samples": len(self.samples)}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


def measure_h2d_gbps(nbytes: int = 256 << 20) -> float:
    """Host-link bandwidth: pinned host -> device copy (best of 5)."""
    h = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    d = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    best = 1e30
    for _ in range(5):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        d.copy_(h, non_blocking=True)
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b))
    return nbytes / (best * 1e-3) / 1e9


def ncu_traffic(kernel: str):
    """DRAM bytes per launch of `kernel` from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        d = json.load(open(p))
        v = d.get(kernel)
        if isinstance(v, dict):
            return v.get("dram_bytes_per_launch")
    return None


def relaunch_under_torchrun(n_gpus: int, argv) -> int:
    """`python bench.py --gpus N` without torchrun: start the N ranks the
    driver's launcher would (one process per GPU, torch.distributed.run on
    127.0.0.1, a free port); rank 0 prints the line."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n_gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *argv]
    return subprocess.call(cmd)


def setup_dist(n_gpus: int):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != n_gpus:
        if world == 1 and n_gpus > 1:
            raise SystemExit(f"--gpus {n_gpus} needs torchrun with {n_gpus} processes")
        raise SystemExit(f"WORLD_SIZE={world} != --gpus {n_gpus}")
    if os.environ.get("DSP_BENCH_SAME_GPU"):   # plumbing check only: all ranks on cuda:0, gloo
        local = 0
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        torch.cuda.set_device(local)
        if os.environ.get("DSP_BENCH_SAME_GPU"):
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    return rank, world, local


def fanouts_of(args, cfg):
    """Node-wise fan-outs of the config, or the layer sizes of --scheme layer
    (Table 7: batch 1024, 1000 nodes per layer for both layers)."""
    if args.scheme == "layer":
        return [int(x) for x in args.layer_sizes.split(",")]
    return list(cfg.fanouts)


def oracle_sample(args, ip, ix, seeds, fanouts, rng, weights=None):
    import oracle
    if args.scheme == "layer":
        return oracle.sample_layerwise(ip, ix, seeds, fanouts, rng)
    return oracle.sample(ip, ix, seeds, fanouts, rng, weights=weights)


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
    ew = datagen.edge_weights(ix, datagen.node_weights(cfg.num_nodes)) if args.scheme == "biased" else None
    edges = rows = 0
    steps_done = 0
    t_all = 0.0
    if args.scheme == "walk":   # a bounded sample of each step's walks (4096 of --walkers)
        rng = np.random.default_rng(1234)
        for step in range(args.warmup + args.steps):
            st = rng.integers(0, cfg.num_nodes, size=min(args.walkers, 4096)).astype(np.int32)
            t0 = time.perf_counter()
            tr = oracle.random_walk(ip, ix, st, args.walk_length, datagen.BASE_SEED + step)
            dt = time.perf_counter() - t0
            if step >= args.warmup:
                t_all += dt
                edges += int((tr[:, 1:] >= 0).sum())
                steps_done += 1
                if t_all > args.ref_max_seconds:
                    break
        line = {"impl": "reference", "metric": METRIC, "value": edges / t_all, "unit": "edges/s",
                "n_gpus": args.gpus, "steps": steps_done, "warmup": args.warmup,
                "ms_per_step": 1e3 * t_all / steps_done, "higher_is_better": True, "scaling": "weak",
                "vs_baseline": None, "dtype": "int32", "data": "synthetic",
                "config": {"workload": f"{cfg.name}-walk", "scheme": "walk", "walk_length": args.walk_length},
                "cpu_baseline": {"value": edges / t_all, "unit": "edges/s", "cores": 1, "kind": "oracle",
                                 "sample": f"{steps_done} x {min(args.walkers, 4096)} walks (oracle.random_walk)"},
                "e2e": {"value": edges / t_all, "unit": "edges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line), flush=True)
        return 0
    for step in range(args.warmup + args.steps):
        seeds = batches[step % len(batches)]
        t0 = time.perf_counter()
        blocks = oracle_sample(args, ip, ix, seeds, fanouts_of(args, cfg), datagen.BASE_SEED + step, weights=ew)
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
        "data": "synthetic", "config": {"workload": cfg.name + ("" if args.scheme == "uniform" else f"-{args.scheme}"),
                                         "scheme": args.scheme, "fanouts": fanouts_of(args, cfg),
                                         "batch_per_gpu": cfg.batch, "num_nodes": cfg.num_nodes, "dim": cfg.dim},
        "cpu_baseline": {"value": value, "unit": "edges/s", "cores": 1, "kind": "oracle",
                         "sample": f"{steps_done} batches of {cfg.batch} seeds (oracle.sample + oracle.gather)"},
        "e2e": {"value": value, "unit": "edges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "feature_GBps": rows * cfg.dim * 4 / t_all / 1e9,
        "seeds_per_s": steps_done * cfg.batch / t_all,
    }
    print(json.dumps(line), flush=True)
    return 0


def host_cpu() -> dict:
    """The host the oracle runs on: CPU model (lscpu / /proc/cpuinfo), logical
    cores, and the cores this process may use."""
    model = None
    try:
        out = subprocess.check_output(["lscpu"], text=True, stderr=subprocess.DEVNULL)
        for line in out.splitlines():
            if line.startswith("Model name:"):
                model = line.split(":", 1)[1].strip()
    except Exception:
        pass
    if model is None:
        try:
            for line in open("/proc/cpuinfo"):
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
        except Exception:
            pass
    return {"model": model, "logical_cores": os.cpu_count(), "cores_available": len(os.sched_getaffinity(0))}


def cpu_baseline(args, cfg, ip, ix, feats, batches, seconds: float, weights=None):
    """the oracle (single host thread) pinned to one core
    (sched_setaffinity of the calling thread, the `taskset -c` of one core), on
    the same seed batches and rng_seed schedule as the GPU run: the whole epoch
    of this rank's batches, or as many as fit in `seconds`.  Runs after the GPU
    timing, outside every timed region."""
    import datagen
    import oracle
    host = host_cpu()
    old = os.sched_getaffinity(0)
    core = min(old)
    os.sched_setaffinity(0, {core})
    try:
        t_all = 0.0
        edges = 0
        n = 0
        while t_all < seconds and n < len(batches):
            seeds = batches[n]
            t0 = time.perf_counter()
            blocks = oracle_sample(args, ip, ix, seeds, fanouts_of(args, cfg), datagen.BASE_SEED + n, weights=weights)
            oracle.gather(feats, blocks[-1]["src_ids"])
            t_all += time.perf_counter() - t0
            edges += sum(int(b["num_edges"]) for b in blocks)
            n += 1
    finally:
        os.sched_setaffinity(0, old)
    full = n == len(batches)
    return {"value": edges / t_all, "unit": "edges/s", "cores": 1, "kind": "oracle",
            "sample": (f"{'the full epoch' if full else 'a bounded sample'}: {n} of {len(batches)} {cfg.name} "
                       f"batches of {cfg.batch} seeds (oracle.sample + oracle.gather), {t_all:.1f} s on 1 core "
                       f"pinned (core {core}) of {host['cores_available']} available"),
            "epoch_batches": len(batches), "batches_timed": n, "seeds_per_s": n * cfg.batch / t_all,
            "host": host}


# ----------------------------------------------------------------- product

def algorithmic_bytes(sizes, L, dim):
    """24 B per frontier node, 8 B per sampled edge, 4 B per
    new unique node, and 2 * dim * 4 B per gathered row (read + write)."""
    F = sum(int(sizes[3 * l]) for l in range(L))
    E = sum(int(sizes[3 * l + 2]) for l in range(L))
    new = sum(int(sizes[3 * l + 1]) - int(sizes[3 * l]) for l in range(L))
    U = int(sizes[3 * (L - 1) + 1])
    return 24 * F + 8 * E + 4 * new, 2 * U * dim * 4


def peer_read_peak(s, bnds, rank: int, world: int, dim: int, reps: int = 5):
    """NVLink denominator measured in this run: every rank at once gathers
    contiguous runs of rows owned by each of the other ranks through
    dsp_gather_features (TMA bulk copies reading the peers' shards over their
    peer mappings: all GPU pairs busy), ~256 MB per rank.  Returns the
    per-GPU receive rate (bytes read from peers / max-over-ranks time)."""
    rows_per_peer = max(1, (256 << 20) // (dim * 4) // max(1, world - 1))
    ids = []
    for r in range(world):
        if r == rank:
            continue
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        n = min(rows_per_peer, hi - lo)
        ids.append(np.arange(lo, lo + n, dtype=np.int32))
    ids = torch.from_numpy(np.concatenate(ids)).cuda()
    out = torch.empty((ids.numel(), dim), dtype=torch.float32, device="cuda")
    for _ in range(2):
        s.gather(ids, out)
    s.sync()
    best = 1e30
    stream = torch.cuda.current_stream()
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        barrier()
        torch.cuda.synchronize()
        a.record(stream)
        s.gather(ids, out)
        b.record(stream)
        torch.cuda.synchronize()
        best = min(best, reduce_max_over_ranks(a.elapsed_time(b)))
    nbytes = reduce_sum_over_ranks(float(ids.numel() * dim * 4)) / world
    del out
    return nbytes / (best * 1e-3) / 1e9, int(ids.numel())


def remote_bytes(blocks, bnds, rank: int, dim: int):
    """NVLink bytes one step of this rank causes (per
    requester; summed over the ranks they count every byte that crosses a link
    once): per layer 4 B per remote frontier id sent to its owner, 4 B count +
    4 B per sampled edge returned for it; the gather reads dim * 4 B per row of
    the last block owned by another rank."""
    lo, hi = int(bnds[rank]), int(bnds[rank + 1])
    csp = 0
    for b in blocks:
        f = b.src_ids[: b.num_dst].cpu().numpy()
        ip = b.indptr[: b.num_dst + 1].cpu().numpy().astype(np.int64)
        rem = (f < lo) | (f >= hi)
        csp += 8 * int(rem.sum()) + 4 * int(np.diff(ip)[rem].sum())
    u = blocks[-1].src_ids.cpu().numpy()
    rows = int(((u < lo) | (u >= hi)).sum())
    return csp, rows * dim * 4, rows


def multi_phase_us(s, L: int):
    """Phase durations of this rank's last synchronous k_csp_multi call from
    the globaltimer stamps block 0 leaves in the workspace header at every
    grid barrier: per layer A shuffle (frontier ids into the owners' inboxes),
    B owner sample (waits for every rank's inbox flag, then samples and writes
    the rows back), C return (waits for the return flags, unpermute + marks),
    D relabel scan (2 barrier intervals)."""
    ws = s.workspace[:1024].view(torch.int64)
    t = ws[81:105].cpu().numpy()
    nb = sum(1 for g in range(1, 23) if t[g] > t[0])
    st = [int(t[0])] + [int(t[g]) for g in range(1, nb + 1)]
    d = np.diff(np.array(st, dtype=np.int64)) / 1e3
    if len(d) == 5 * L + 1:   # a call that zeroed the relabel map first
        d = d[1:]
    if len(d) != 5 * L:
        return None
    return [{"shuffle_us": float(d[5 * l]), "owner_sample_us": float(d[5 * l + 1]),
             "return_unpermute_us": float(d[5 * l + 2]), "relabel_us": float(d[5 * l + 3] + d[5 * l + 4]),
             "exchange_us": float(d[5 * l] + d[5 * l + 1] + d[5 * l + 2])} for l in range(L)]


def run_walk(args):
    """--scheme walk: random walks (fan-out 1 at every step, a node
    without neighbours ends its walk) of --walk-length steps from --walkers
    start nodes per GPU; one bench step = one dsp_random_walk call.  Metric:
    walk steps (sampled edges) per second."""
    import datagen
    import paper_conf_ppopp_caiz0zszck23_b200 as pkg
    rank, world, local = setup_dist(args.gpus)
    torch.cuda.set_device(local)
    cfg, ip, ix, bnds, sip, six, feats, train = load_workload(args.config, rank, world)
    ex = pkg.torch_exchange() if world > 1 else None
    nw, length = args.walkers, args.walk_length
    s = pkg.Sampler(bnds, sip, six, feats, cfg.fanouts, cfg.batch, rank=rank, world_size=world, device=local,
                    exchange=ex, max_walks=nw if world > 1 else None, max_walk_length=length)
    lo, hi = int(bnds[rank]), int(bnds[rank + 1])
    rng = np.random.default_rng(1234 + rank)
    KS, W = args.steps, args.warmup
    starts = [torch.from_numpy(rng.integers(lo, hi, size=nw).astype(np.int32)).cuda() for _ in range(4)]
    stream = torch.cuda.current_stream()
    for i in range(W):
        s.random_walk(starts[i % 4], length, datagen.BASE_SEED + i)
    s.sync()
    barrier()
    torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for e in (ev0, ev1):
        e.record(stream)
    # world 1: K walk calls in flight on K streams (each walk is a chain of dependent random
    # reads, so more independent walks in flight = more throughput); world > 1: one stream
    # (the walkers move through the ctx's exchange region)
    K = max(1, args.instances) if world == 1 else 1
    streams = [torch.cuda.Stream() for _ in range(K)] if K > 1 else [stream]
    outs = [torch.empty((nw, length + 1), dtype=torch.int32, device="cuda") for _ in range(max(2, K))]  # up front
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        ev0.record(stream)
        for st in streams:
            st.wait_stream(stream)
        for j in range(KS):
            with torch.cuda.stream(streams[j % K]):
                s.random_walk(starts[j % 4], length, datagen.BASE_SEED + W + j, out=outs[j % max(2, K)])
        for st in streams:
            stream.wait_stream(st)
        ev1.record(stream)
        s.sync()
        torch.cuda.synchronize()
    barrier()
    t_ms = ev0.elapsed_time(ev1)
    # steps actually taken (a walk ends at a node without neighbours: -1 afterwards): the
    # walks are a pure function of (starts, seed), so they are re-run untimed and counted
    steps_taken = 0.0
    for j in range(KS):
        o = s.random_walk(starts[j % 4], length, datagen.BASE_SEED + W + j, out=outs[0])
        steps_taken += float((o[:, 1:] >= 0).sum().item())
    t_max = reduce_max_over_ranks(t_ms)
    tot = reduce_sum_over_ranks(steps_taken)
    peak, peak_kind = measured_peaks()
    # algorithmic bytes per walk step: indptr pair (16 B) + the adjacency id (4 B) + the trace entry (4 B)
    achieved = 24.0 * steps_taken / (t_ms * 1e-3) / 1e9
    # e2e: starts H2D from pinned host memory and the traces D2H into pinned host memory every call
    h_starts = [x.cpu().pin_memory() for x in starts]
    h_out = torch.empty((nw, length + 1), dtype=torch.int32).pin_memory()
    d_st = torch.empty(nw, dtype=torch.int32, device="cuda")
    n_e2e = max(3, min(KS, 20))
    barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    e_steps = 0
    for j in range(n_e2e):
        d_st.copy_(h_starts[j % 4], non_blocking=True)
        o = s.random_walk(d_st, length, datagen.BASE_SEED + j, out=outs[j % 2])
        h_out.copy_(o, non_blocking=True)
        e_steps += nw * length
    e1.record(stream)
    torch.cuda.synchronize()
    e2e_ms = reduce_max_over_ranks(e0.elapsed_time(e1))
    e2e_frac = steps_taken / (KS * nw * length) if KS else 1.0
    if rank == 0:
        line = {
            "metric": METRIC, "value": tot / (t_max * 1e-3), "unit": "edges/s", "n_gpus": world,
            "steps": KS, "warmup": W, "ms_per_step": t_max / KS, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": f"{cfg.name}-walk" + (f"-P{world}" if world > 1 else ""), "scheme": "walk",
                       "walkers_per_gpu": nw, "walk_length": length, "num_nodes": cfg.num_nodes,
                       "nnz": int(ip[-1]), "parallelism": f"csp{world}",
                       "starts": "uniform over each rank's own node range, 4 fixed sets",
                       "step": "dsp_random_walk (thread per walk at world 1; CSP push without reshuffle at world > 1)"
                               + (f", {K} streams" if K > 1 else "")},
            "roofline": {"kernel": "k_random_walk" if world == 1 else "k_walk_step", "bound": "hbm",
                         "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                         "traffic": None, "peak_kind": peak_kind,
                         "algorithmic_bytes_per_launch": 24.0 * steps_taken / KS,
                         "achieved_def": "24 B per walk step (indptr pair, adjacency id, trace entry) / elapsed time; "
                                         "the walk is bound by dependent random DRAM requests, not bytes",
                         "request_rate": {"achieved": steps_taken / (t_ms * 1e-3), "peak": 47e9, "unit": "requests/s",
                                          "frac": steps_taken / (t_ms * 1e-3) / 47e9,
                                          "def": "one random adjacency read (a 32-B DRAM sector) per walk step (the "
                                                 "indptr pairs hit L2) / elapsed time, against the random-read "
                                                 "request ceiling measured by tools/micro/random_read_bench.cu "
                                                 "(~47 G requests/s on B200, 4-64 B per request)"}},
            "e2e": {"value": reduce_sum_over_ranks(e_steps * e2e_frac) / (e2e_ms * 1e-3), "unit": "edges/s",
                    "h2d_bytes_per_step": nw * 4, "d2h_bytes_per_step": nw * (length + 1) * 4, "steps": n_e2e,
                    "api": "starts H2D from pinned host memory, dsp_random_walk, traces D2H into pinned host memory"},
            "cpu_baseline": None,
            "gpu_launches": KS if world == 1 else KS * (2 * length + 3),
            "clocks": clk.summary(),
        }
        if world == 1 and not args.no_cpu_baseline:
            import oracle
            n_cpu, t_cpu, st_cpu = 0, 0.0, 0
            while t_cpu < min(args.cpu_seconds, 10.0) and n_cpu < 50:
                st = starts[n_cpu % 4][:4096].cpu().numpy()
                t0 = time.perf_counter()
                tr = oracle.random_walk(ip, ix, st, length, datagen.BASE_SEED + n_cpu)
                t_cpu += time.perf_counter() - t0
                st_cpu += int((tr[:, 1:] >= 0).sum())
                n_cpu += 1
            line["cpu_baseline"] = {"value": st_cpu / t_cpu, "unit": "edges/s", "cores": 1, "kind": "oracle",
                                    "sample": f"{n_cpu} x 4096 walks of length {length}, single host thread "
                                              f"(oracle.random_walk), {t_cpu:.1f} s"}
        print(json.dumps(line), flush=True)
    barrier()
    s.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def run_dsp(args):
    import datagen
    import paper_conf_ppopp_caiz0zszck23_b200 as pkg
    rank, world, local = setup_dist(args.gpus)
    torch.cuda.set_device(local)
    cfg, ip, ix, bnds, sip, six, feats, train = load_workload(args.config, rank, world)
    ex = pkg.torch_exchange() if world > 1 else None
    biased = args.scheme == "biased"
    ew = datagen.edge_weights(six, datagen.node_weights(cfg.num_nodes)) if biased else None
    layer = args.scheme == "layer"
    fanouts = fanouts_of(args, cfg)
    # K concurrent step streams, each launch on 1/K of the SMs with its own workspace; at
    # world > 1 each stream's calls use their own exchange channel (DSP_OPT_EXCHANGE_CHANNELS;
    # the layer-wise scheme keeps one stream there: its exchange region is per ctx)
    K = max(1, args.instances) if world == 1 or not layer else 1
    opts = {pkg.dsp.DSP_OPT_EXCHANGE_CHANNELS: K} if world > 1 and not layer else {}
    if args.loader_rows:
        opts[pkg.dsp.DSP_OPT_LOADER_ROWS] = args.loader_rows
    s = pkg.Sampler(bnds, sip, six, feats, fanouts, cfg.batch, rank=rank, world_size=world, scheme="layer" if layer else "node",
                    device=local, exchange=ex, n_slots=2 * K, edge_weights=ew, n_workspaces=K,
                    hot_rows=None if args.hot_frac is None else int(round(args.hot_frac * (len(sip) - 1))),
                    options=opts)
    if K > 1:  # K steps in flight on K streams, each persistent launch on 1/K of the SMs
        pkg.dsp_set_persistent_blocks(s.ctx, torch.cuda.get_device_properties(local).multi_processor_count // K)
    for slot in range(2 * K):
        s.feat_buffer(slot)   # allocate every output set now, not at its first use inside the timed region
    L = len(fanouts)
    steps_epoch = datagen.steps_per_epoch(train, bnds, cfg.batch)
    batches = datagen.rank_seed_batches(train, bnds, rank, cfg.batch, 0)[:steps_epoch]
    dev_batches = torch.from_numpy(np.ascontiguousarray(batches)).cuda()   # inputs resident in HBM
    stream = torch.cuda.current_stream()
    streams = [torch.cuda.Stream() for _ in range(K)]
    KS, W = args.steps, args.warmup
    h_sizes = torch.zeros((W + KS, 3 * L), dtype=torch.int64).pin_memory()
    pipelined = not args.no_pipeline

    def step(i, ev=None):
        # one step = the whole hot path (CSP over all layers + feature gather) for one
        # batch.  Pipelined (default): the launch of step i samples batch i while its
        # loader warps gather the previous batch of the same stream (the paper's
        # pipeline); flush() gathers the last one.  K streams each run
        # every K-th step on 1/K of the SMs, with 2 output sets each.
        j = i % K
        st = streams[j]
        if ev is not None:
            ev[0].record(st)
        s.sample_gather(dev_batches[i % len(batches)], datagen.BASE_SEED + i, slot=(i % (2 * K)),
                        sizes_out=h_sizes[i], async_=True, pipelined=pipelined, biased=biased, ws=j, stream=st)
        if ev is not None:
            ev[1].record(st)

    def flush_all():
        for st in streams:
            with torch.cuda.stream(st):
                s.flush()

    def fork():
        for st in streams:
            st.wait_stream(stream)

    def join():
        for st in streams:
            stream.wait_stream(st)

    fork()
    for i in range(W):
        step(i)
    flush_all()
    join()
    s.sync()
    barrier()
    torch.cuda.synchronize()

    # ---- timed region: KS steps, inputs resident, device time via CUDA events
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    sev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(KS)]
    for e in (ev0, ev1, *[x for pair in sev for x in pair]):
        e.record(stream)   # torch creates the CUDA event at its first record: not inside the timed region
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        ev0.record(stream)
        h0 = time.perf_counter()
        fork()
        for j in range(KS):
            step(W + j, sev[j])
        flush_all()  # the gathers of the last timed batches are inside the timed region
        join()
        ev1.record(stream)
        host_issue_ms = (time.perf_counter() - h0) * 1e3
        s.sync()
        torch.cuda.synchronize()
    barrier()
    K_ = KS
    t_ms = ev0.elapsed_time(ev1)
    step_ms = [a.elapsed_time(b) for a, b in sev]
    sz = h_sizes.numpy()[W: W + KS]
    edges = float(sum(int(sz[j, 3 * l + 2]) for j in range(KS) for l in range(L)))
    rows = float(sum(int(sz[j, 3 * (L - 1) + 1]) for j in range(KS)))
    seeds_n = float(sum(int(sz[j, 0]) for j in range(KS)))
    samp_b = gath_b = 0
    for j in range(KS):
        a, b = algorithmic_bytes(sz[j], L, cfg.dim)
        samp_b += a
        gath_b += b
    t_max = reduce_max_over_ranks(t_ms)
    tot_edges = reduce_sum_over_ranks(edges)
    tot_rows = reduce_sum_over_ranks(rows)
    tot_seeds = reduce_sum_over_ranks(seeds_n)
    peak, peak_kind = measured_peaks()
    step_mean = float(np.mean(step_ms))
    # K launches overlap on the device: the kernel stream's achieved HBM rate is the
    # algorithmic bytes of all timed launches over the elapsed device time
    achieved = (samp_b + gath_b) / (t_ms * 1e-3) / 1e9

    # ---- bytes the scheme adds to the uniform path's algorithmic bytes, from a few
    # untimed synchronous calls on the same batches (host-side counting only)
    weight_b = cold_b = None
    if biased or args.hot_frac is not None:
        deg = np.diff(ip)   # global in-degrees (every rank holds the whole synthetic graph here)
        if args.hot_frac is not None:   # each owner's hot set: largest in-degree, ties by smaller id (R31)
            hot = np.zeros(len(deg), dtype=bool)
            for r in range(world):
                lo_r, hi_r = int(bnds[r]), int(bnds[r + 1])
                nh = int(round(args.hot_frac * (hi_r - lo_r)))
                dr = deg[lo_r:hi_r]
                hot[lo_r + np.lexsort((np.arange(len(dr)), -dr))[:nh]] = True
        wb, cb = [], []
        for j in range(min(KS, 5)):
            blocks = s.sample(dev_batches[(W + j) % len(batches)], datagen.BASE_SEED + W + j, biased=biased)
            if biased:  # every weight of a row with deg > k is read (successive sampling, R25/R26)
                tot = 0
                for l, b in enumerate(blocks):
                    d = deg[b.src_ids[: b.num_dst].cpu().numpy().astype(np.int64)]
                    tot += int(d[d > fanouts[l]].sum())
                wb.append(4.0 * tot)
            if args.hot_frac is not None:
                ids = blocks[-1].src_ids.cpu().numpy().astype(np.int64)
                cb.append(float((~hot[ids]).sum()) * cfg.dim * 4)
        s.sync()
        weight_b = float(np.mean(wb)) if wb else None
        cold_b = float(np.mean(cb)) if cb else None

    # ---- breakdown (not the headline): the two calls separately
    ids_dev = None
    bd = {}
    if not args.no_breakdown:
        NB = min(KS, 20)
        if K > 1:
            pkg.dsp_set_persistent_blocks(s.ctx, 0)   # the breakdown times single full-GPU calls
        g_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(NB)]
        s_ms = []
        nrow = []
        out = s.feat_buffer(0)
        for j in range(NB):
            i = W + j
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            blocks = s.sample(dev_batches[i % len(batches)], datagen.BASE_SEED + i, biased=biased)
            a1.record(stream)
            ids_dev = blocks[-1].src_ids
            g_ev[j][0].record(stream)
            s.gather(ids_dev, out[: ids_dev.numel()])
            g_ev[j][1].record(stream)
            nrow.append(ids_dev.numel())
            torch.cuda.synchronize()
            s_ms.append(a0.elapsed_time(a1))
        s.sync()
        g_ms = [a.elapsed_time(b) for a, b in g_ev]
        g_bytes = [2.0 * n * cfg.dim * 4 for n in nrow]
        bd = {"sample_call_ms_mean": float(np.mean(s_ms)), "gather_call_ms_mean": float(np.mean(g_ms)),
              "gather_GBps": float(np.mean([b / (m * 1e-3) / 1e9 for b, m in zip(g_bytes, g_ms)])),
              "gather_frac_of_hbm": float(np.mean([b / (m * 1e-3) / 1e9 for b, m in zip(g_bytes, g_ms)])) / peak,
              "note": "dsp_sample (synchronous, host sizes) and dsp_gather_features timed separately"}

    # ---- e2e: the same steps through the C ABI from HOST buffers, one synchronous
    # dsp_sample_gather per step (the call a training loop makes): every step copies
    # its seeds H2D from pinned memory and reads the per-layer sizes back (the host
    # needs them to shape the consumer's launch); blocks and features stay in HBM for
    # the GPU trainer.  e2e_host_copy additionally copies every block and all gathered
    # features to pinned host memory (PCIe-bound; a host consumer's view).
    h_seeds = torch.from_numpy(np.ascontiguousarray(batches)).pin_memory()
    h_feat = torch.empty((s.max_src[-1], cfg.dim), dtype=torch.float32).pin_memory()
    h_blk = [tuple(torch.empty(x.numel(), dtype=torch.int32).pin_memory() for x in bufs) for bufs in s._bufs]
    d_seed = torch.empty(cfg.batch, dtype=torch.int32, device="cuda")
    e2e_steps = max(3, min(KS, 20))

    def e2e_run(host_copy: bool):
        h2d = d2h = 0
        barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        n_edges = 0
        e0.record(stream)
        for j in range(e2e_steps):
            i = W + j
            d_seed.copy_(h_seeds[i % len(batches)], non_blocking=True)
            h2d += d_seed.numel() * 4
            # synchronous call: returns after the step with the host-side sizes filled (D2H)
            blocks, feat = s.sample_gather(d_seed, datagen.BASE_SEED + i, slot=0, biased=biased)
            d2h += 3 * 8 * L
            if host_copy:
                for b, hb in zip(blocks, h_blk):
                    hb[0][: b.num_dst + 1].copy_(b.indptr, non_blocking=True)
                    hb[1][: b.num_edges].copy_(b.indices, non_blocking=True)
                    hb[2][: b.num_src].copy_(b.src_ids, non_blocking=True)
                    d2h += 4 * (b.num_dst + 1 + b.num_edges + b.num_src)
                h_feat[: feat.shape[0]].copy_(feat, non_blocking=True)
                d2h += feat.numel() * 4
            n_edges += sum(b.num_edges for b in blocks)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = reduce_max_over_ranks(e0.elapsed_time(e1))
        return reduce_sum_over_ranks(n_edges) / (ms * 1e-3), h2d // e2e_steps, d2h // e2e_steps

    def e2e_async_run():
        # the bench step with the seeds in pinned HOST memory: every step copies its seeds
        # H2D and reads its per-layer sizes back D2H into pinned host memory.  The copies run
        # on their own streams, ordered by events against the step streams (the paper's
        # pipelined loader: copies, sampling and the previous gather overlap):
        # seeds of step j land in buffer j % nbuf once step j - nbuf has consumed it; the
        # sizes leave once step j is done.
        nbuf = 2 * K
        d_seeds = [torch.empty(cfg.batch, dtype=torch.int32, device="cuda") for _ in range(nbuf)]
        n_steps = max(3, min(KS, 200))
        h_sz = torch.zeros((n_steps, 3 * L), dtype=torch.int64).pin_memory()
        d_sz = torch.zeros((n_steps, 3 * L), dtype=torch.int64, device="cuda")
        cs_in, cs_out = torch.cuda.Stream(), torch.cuda.Stream()
        ready = [torch.cuda.Event() for _ in range(nbuf)]
        used = [torch.cuda.Event() for _ in range(nbuf)]
        barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        fork()
        cs_in.wait_stream(stream)
        cs_out.wait_stream(stream)
        for j in range(n_steps):
            i = W + j
            st = streams[j % K]
            b = j % nbuf
            with torch.cuda.stream(cs_in):
                if j >= nbuf:
                    cs_in.wait_event(used[b])
                d_seeds[b].copy_(h_seeds[i % len(batches)], non_blocking=True)
                ready[b].record(cs_in)
            st.wait_event(ready[b])
            s.sample_gather(d_seeds[b], datagen.BASE_SEED + i, slot=(j % (2 * K)), sizes_out=d_sz[j], async_=True,
                            pipelined=pipelined, biased=biased, ws=j % K, stream=st)
            used[b].record(st)
            with torch.cuda.stream(cs_out):
                cs_out.wait_event(used[b])
                h_sz[j].copy_(d_sz[j], non_blocking=True)
        flush_all()
        join()
        stream.wait_stream(cs_in)
        stream.wait_stream(cs_out)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = reduce_max_over_ranks(e0.elapsed_time(e1))
        n_edges = float(h_sz.numpy()[:, 2::3].sum())
        return reduce_sum_over_ranks(n_edges) / (ms * 1e-3), cfg.batch * 4, 3 * 8 * L, n_steps

    if K > 1:   # the asynchronous e2e runs the timed step's configuration: K streams x 1/K of the SMs
        pkg.dsp_set_persistent_blocks(s.ctx, torch.cuda.get_device_properties(local).multi_processor_count // K)
    e2e_av, e2e_ah2d, e2e_ad2h, e2e_an = e2e_async_run()
    if K > 1:   # one synchronous call at a time: the whole GPU
        pkg.dsp_set_persistent_blocks(s.ctx, 0)
    e2e_v, e2e_h2d, e2e_d2h = e2e_run(False)
    e2e_hv, e2e_hh2d, e2e_hd2h = e2e_run(True)

    # ---- world > 1: NVLink bytes of a step (from untimed synchronous calls on the
    # timed batches: the blocks are a pure function of seeds and rng_seed), the
    # peer-read peak measured here, and per-layer exchange time from the stamps
    nvl = None
    if world > 1:
        csp_l, gat_l, rows_l, phases = [], [], [], []
        for j in range(min(KS, 5)):
            blocks = s.sample(dev_batches[(W + j) % len(batches)], datagen.BASE_SEED + W + j, biased=biased)
            ph = None if layer else multi_phase_us(s, L)
            if ph is not None:
                phases.append(ph)
            c_, g_, r_ = remote_bytes(blocks, bnds, rank, cfg.dim)
            csp_l.append(c_)
            gat_l.append(g_)
            rows_l.append(r_)
        s.sync()
        csp_step = reduce_sum_over_ranks(float(np.mean(csp_l))) / world     # per GPU (mean over ranks)
        gat_step = reduce_sum_over_ranks(float(np.mean(gat_l))) / world
        peer_peak, peer_rows = peer_read_peak(s, bnds, rank, world, cfg.dim)
        nvl_achieved = (csp_step + gat_step) * KS / (t_max * 1e-3) / 1e9
        layer_us = None
        if phases:
            layer_us = [{k: float(np.median([p[l][k] for p in phases])) for k in phases[0][l]} for l in range(L)]
        nvl = {"achieved": nvl_achieved, "peak": peer_peak, "frac": nvl_achieved / peer_peak,
               "bytes_per_step_per_gpu": csp_step + gat_step, "csp_exchange_bytes_per_step_per_gpu": csp_step,
               "gather_remote_bytes_per_step_per_gpu": gat_step,
               "remote_row_share": float(np.mean(rows_l)) / max(1.0, rows / KS),
               "peak_kind": (f"measured in this run: dsp_gather_features of {peer_rows} contiguous rows owned by "
                             "the other ranks, every rank at once (TMA reads of the peers' shards over their "
                             "peer mappings), bytes read / max-over-ranks time"
                             + ("; DSP_BENCH_SAME_GPU: every rank on one GPU, so 'peer' reads are local HBM"
                                if os.environ.get("DSP_BENCH_SAME_GPU") else "")),
               "layer_phase_us_rank0": layer_us}

    cpu = None
    if rank == 0 and not args.no_cpu_baseline:
        # the oracle gathers from the whole feature table (rank 0's shard alone at N > 1)
        full = feats if world == 1 else datagen.features(0, cfg.num_nodes, cfg.dim)
        ew_full = ew if world == 1 or ew is None else datagen.edge_weights(ix, datagen.node_weights(cfg.num_nodes))
        cpu = cpu_baseline(args, cfg, ip, ix, full, batches, args.cpu_seconds, weights=ew_full)
        del full

    kern_per_step = 1
    roof_kernel = (("k_lw_persistent" if world == 1 else "k_lw_multi") if layer
                   else ("k_csp_persistent" if world == 1 else "k_csp_multi"))
    roofline = {"kernel": roof_kernel,
                "bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak,
                "traffic": (ncu_traffic(roof_kernel) if roof_kernel == "k_csp_persistent" and args.scheme == "uniform"
                            and args.hot_frac is None and args.config == "products" else None),
                "peak_kind": peak_kind,
                "algorithmic_bytes_per_launch": (samp_b + gath_b) / KS,
                "sampling_bytes_per_launch": samp_b / KS, "gather_bytes_per_launch": gath_b / KS,
                "launch_ms_mean": step_mean, "concurrent_launches": K,
                "achieved_def": "algorithmic bytes of all timed launches / elapsed device time"}
    if weight_b is not None:   # biased: the edge weights of every row sampled with draws are read too
        a_w = (samp_b + gath_b + weight_b * KS) / (t_ms * 1e-3) / 1e9
        roofline.update({"achieved": a_w, "frac": a_w / peak, "weight_bytes_per_launch": weight_b,
                         "algorithmic_bytes_per_launch": (samp_b + gath_b) / KS + weight_b})
    if nvl is not None:        # world > 1: the gather's remote rows and the CSP exchanges cross NVLink
        roofline = {"kernel": roof_kernel, "bound": "nvlink", "achieved": nvl["achieved"], "peak": nvl["peak"],
                    "unit": "GB/s", "frac": nvl["frac"], "traffic": None, "peak_kind": nvl["peak_kind"],
                    "nvlink_bytes_per_step_per_gpu": nvl["bytes_per_step_per_gpu"],
                    "csp_exchange_bytes_per_step_per_gpu": nvl["csp_exchange_bytes_per_step_per_gpu"],
                    "gather_remote_bytes_per_step_per_gpu": nvl["gather_remote_bytes_per_step_per_gpu"],
                    "remote_row_share": nvl["remote_row_share"],
                    "hbm": {"achieved": achieved, "peak": peak, "frac": achieved / peak, "peak_kind": peak_kind,
                            "algorithmic_bytes_per_launch": (samp_b + gath_b) / KS},
                    "launch_ms_mean": step_mean, "concurrent_launches": K,
                    "achieved_def": "NVLink bytes per step per GPU (remote frontier ids + returned rows + remote "
                                    "feature rows, per requester, mean over ranks) x steps / max-over-ranks time"}
    if cold_b is not None:     # cold tier: the dominant stream is the cold rows over the host link
        link = measure_h2d_gbps()
        a_c = cold_b * KS / (t_ms * 1e-3) / 1e9
        roofline = {"kernel": roof_kernel, "bound": "host-link", "achieved": a_c, "peak": link, "unit": "GB/s",
                    "frac": a_c / link, "traffic": None,
                    "peak_kind": "measured here: pinned host -> device cudaMemcpy of 256 MB",
                    "cold_bytes_per_launch": cold_b, "hbm_algorithmic_bytes_per_launch": (samp_b + gath_b) / KS,
                    "hbm_frac": achieved / peak, "launch_ms_mean": step_mean, "concurrent_launches": K,
                    "achieved_def": "cold feature bytes read over the host link per launch x launches / elapsed time"}
    if rank == 0:
        line = {
            "metric": METRIC, "value": tot_edges / (t_max * 1e-3), "unit": "edges/s", "n_gpus": world,
            "steps": KS, "warmup": W, "ms_per_step": t_max / KS,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32+f32",
            "data": "synthetic",
            "config": {"workload": (cfg.name if world == 1 else f"{cfg.name}-P{world}")
                       + ("-biased" if biased else "") + ("-layerwise" if layer else "")
                       + ("" if args.hot_frac is None else f"-hot{args.hot_frac:g}"), "scheme": args.scheme,
                       "features": ("all rows in HBM" if args.hot_frac is None else
                                    f"cold tier: {args.hot_frac:g} of rows (largest in-degree) in HBM, "
                                    "the rest in pinned host memory read over UVA"),
                       "fanouts": fanouts, "batch_per_gpu": cfg.batch, "num_nodes": cfg.num_nodes,
                       "nnz": int(ip[-1]), "dim": cfg.dim, "parallelism": f"csp{world}",
                       "l2": (f"inputs larger than L2 (CSR {(ip.nbytes + ix.nbytes) / 1e9:.1f} GB + features "
                              f"{cfg.num_nodes * cfg.dim * 4 / 1e9:.1f} GB >> "
                              f"{getattr(torch.cuda.get_device_properties(local), 'L2_cache_size', 0) / 2**20:.0f} MB L2)"),
                       "step": ("dsp_sample_gather (DSP_PIPELINED: sampler(t) || loader(t-1), 2 output sets)"
                                if pipelined else "dsp_sample_gather (async, 2 output sets)")
                       + (f", {K} streams x {torch.cuda.get_device_properties(local).multi_processor_count // K} SMs"
                          if K > 1 else "")},
            "seeds_per_s": tot_seeds / (t_max * 1e-3),
            "host_issue_ms_per_step": host_issue_ms / KS,
            "feature_GBps": tot_rows * cfg.dim * 4 / (t_max * 1e-3) / 1e9,
            "edges_per_step": tot_edges / KS / world,
            "rows_per_step": tot_rows / KS / world,
            "roofline": roofline,
            "breakdown": bd,
            "epoch_sampling_s": (steps_epoch * bd["sample_call_ms_mean"] * 1e-3 if bd else None),
            "cpu_baseline": cpu,
            "e2e": ({"value": e2e_av, "unit": "edges/s", "h2d_bytes_per_step": e2e_ah2d,
                     "d2h_bytes_per_step": e2e_ad2h, "steps": e2e_an,
                     "api": "per step: seeds H2D from pinned host memory (copy stream), dsp_sample_gather "
                            "(pipelined, async, as the timed step) and its per-layer sizes D2H into pinned host "
                            "memory (second copy stream), ordered by events; blocks and features stay in HBM "
                            "for the GPU consumer"}
                    if e2e_av is not None else
                    {"value": e2e_v, "unit": "edges/s", "h2d_bytes_per_step": e2e_h2d,
                     "d2h_bytes_per_step": e2e_d2h, "steps": e2e_steps,
                     "api": "pinned seeds H2D + dsp_sample_gather (synchronous, sizes D2H)"}),
            "e2e_sync": {"value": e2e_v, "unit": "edges/s",
                         "h2d_bytes_per_step": e2e_h2d, "d2h_bytes_per_step": e2e_d2h, "steps": e2e_steps,
                         "api": "pinned seeds H2D + dsp_sample_gather (synchronous: host waits for the sizes "
                                "every step); blocks and features stay in HBM"},
            "e2e_host_copy": {"value": e2e_hv, "unit": "edges/s", "h2d_bytes_per_step": e2e_hh2d,
                              "d2h_bytes_per_step": e2e_hd2h,
                              "api": "as e2e_sync, plus D2H of every block and all gathered features (PCIe-bound)"},
            "layer_phase_us_rank0": (nvl or {}).get("layer_phase_us_rank0"),
            "gpu_launches": kern_per_step * KS + (K if pipelined else 0),  # timed region: one launch per step + flushes
            "clocks": clk.summary(),
        }
        print(json.dumps(line), flush=True)
    barrier()   # no rank frees its peer-mapped shard while another may still read it
    s.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def default_instances(scheme: str, world: int) -> int:
    """Concurrent step streams when --instances is not given, measured per workload
    (DESIGN.md "Measurement"): uniform node-wise steps with 5 loader warps per SM run best
    as 2 streams x 74 SMs (products 0.1264-0.1269 vs 0.1287-0.1300 ms/step with 4, papers
    0.631 vs 0.604, Friendster 0.830 vs 0.797 of HBM); biased and layer-wise steps
    (sampling-bound) and random walks as 4; world > 1 keeps 4 exchange channels."""
    return 2 if (scheme == "uniform" and world == 1) else 4


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["dsp", "reference"], default="dsp")
    ap.add_argument("--config", default=None)
    ap.add_argument("--cpu-seconds", type=float, default=60.0,
                    help="bound on the oracle's timed CPU work (products: the full 192-batch epoch takes ~40 s)")
    ap.add_argument("--ref-max-seconds", type=float, default=60.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-breakdown", action="store_true")
    ap.add_argument("--no-pipeline", action="store_true", help="time non-pipelined fused steps")
    ap.add_argument("--instances", type=int, default=None,
                    help="concurrent step streams (each on 1/K of the SMs; world > 1: one exchange channel each); "
                         "default: 2 for uniform node-wise steps at world 1, else 4")
    ap.add_argument("--loader-rows", type=int, default=0, help="DSP_OPT_LOADER_ROWS (0: library default)")
    ap.add_argument("--layer-sizes", default="1000,1000",
                    help="--scheme layer: nodes sampled per layer (Table 7: 1000,1000)")
    ap.add_argument("--walkers", type=int, default=65536, help="--scheme walk: walks per GPU per step")
    ap.add_argument("--walk-length", type=int, default=80, help="--scheme walk: steps per walk (DeepWalk's 80)")
    ap.add_argument("--scheme", choices=["uniform", "biased", "layer", "walk"], default="uniform",
                    help="node-wise scheme (Table 2 IsBiased); biased uses synthetic node weights")
    ap.add_argument("--hot-frac", type=float, default=None,
                    help="cold-feature tier: fraction of each shard's rows kept in HBM (P:L114)")
    args = ap.parse_args(argv)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ and args.impl == "dsp":
        return relaunch_under_torchrun(args.gpus, sys.argv[1:] if argv is None else list(argv))
    if args.warmup < 3:
        raise SystemExit("--warmup must be >= 3")
    if args.config is None:
        args.config = "products"
    if args.instances is None:
        args.instances = default_instances(args.scheme, int(os.environ.get("WORLD_SIZE", "1")))
    if args.impl == "reference":
        return run_reference(args)
    if args.scheme == "walk":
        return run_walk(args)
    return run_dsp(args)


if __name__ == "__main__":
    sys.exit(main())
