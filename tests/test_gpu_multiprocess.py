"""The multi-process CSP path (one process per rank, CUDA IPC peer mapping,
handle all-gather over torch.distributed, flag-synchronised exchange kernels)
run with two processes sharing the one GPU of this environment: the same code
path bench.py --gpus N takes with one process per GPU.  Without MPS the two
processes' kernels time-slice, so this checks correctness, not speed.
Each rank's blocks must equal the oracle on its seeds; the one-sided gather
reads the peer's feature shard through the IPC mapping; random walks move
walkers between the processes and store trace entries into the peer's
walk region."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = [pytest.mark.gpu, pytest.mark.slow]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _check_pipelined(s, ip, ix, cfg, seeds, rng, slot, sizes):
    import datagen
    import oracle
    ref = oracle.sample(ip, ix, seeds, cfg.fanouts, rng)
    blocks = s.blocks(slot, sizes.numpy())
    for b, r in zip(blocks, ref):
        for key in ("indptr", "indices", "src_ids"):
            if not np.array_equal(getattr(b, key).cpu().numpy(), r[key]):
                raise AssertionError(f"pipelined step rng {rng:#x}: {key}")
    feat = s.feat_buffer(slot)[: blocks[-1].num_src]
    exp = datagen.features_of(ref[-1]["src_ids"], cfg.dim)
    if not np.array_equal(feat.cpu().numpy().view(np.uint32), exp.view(np.uint32)):
        raise AssertionError(f"pipelined step rng {rng:#x}: features")


def _rank(rank, world, port, q, hot=None, scheme="node", channels=1):
    import sys
    here = os.path.dirname(os.path.abspath(__file__))
    sys.path[:0] = [os.path.dirname(here), here]
    import torch.distributed as dist

    import datagen
    import oracle
    import paper_conf_ppopp_caiz0zszck23_b200 as pkg
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    ok, detail = True, ""
    try:
        cfg = datagen.CONFIGS["tiny"]
        ip, ix = datagen.make_graph(cfg)
        bnds = datagen.bounds(cfg.num_nodes, world)
        lo, hi = int(bnds[rank]), int(bnds[rank + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        feats = datagen.features(lo, hi, cfg.dim)
        sizes = (300, 600) if scheme == "layer" else cfg.fanouts
        s = pkg.Sampler(bnds, sip, six, feats, sizes, 32, rank=rank, world_size=world, device=0,
                        exchange=pkg.torch_exchange(), n_slots=2 if channels == 1 else 8,
                        hot_rows=None if hot is None else (hi - lo) * hot // 4, scheme=scheme,
                        max_walks=500, max_walk_length=16, n_workspaces=channels,
                        options={pkg.dsp.DSP_OPT_EXCHANGE_CHANNELS: channels})
        train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
        batches = datagen.rank_seed_batches(train, bnds, rank, 32, 0)
        for step in range(3):
            seeds = batches[step]
            blocks, feat = s.sample_gather(torch.from_numpy(seeds).cuda(), 0x5EED + step, slot=step % 2)
            ref = (oracle.sample_layerwise(ip, ix, seeds, sizes, 0x5EED + step) if scheme == "layer"
                   else oracle.sample(ip, ix, seeds, cfg.fanouts, 0x5EED + step))
            for b, r in zip(blocks, ref):
                for key in ("indptr", "indices", "src_ids"):
                    if not np.array_equal(getattr(b, key).cpu().numpy(), r[key]):
                        ok, detail = False, f"step {step} {key}"
            exp = datagen.features_of(ref[-1]["src_ids"], cfg.dim)
            if not np.array_equal(feat.cpu().numpy().view(np.uint32), exp.view(np.uint32)):
                ok, detail = False, f"step {step} features"
        if channels > 1:
            # several collective calls in flight per rank: step j on stream j % C with
            # workspace j % C (exchange channel j % C), each launch on 1/C of the SMs;
            # pipelined, so step j's features are written by step j + C (or the flush)
            C = channels
            pkg.dsp_set_persistent_blocks(s.ctx, torch.cuda.get_device_properties(0).multi_processor_count // C)
            streams = [torch.cuda.Stream() for _ in range(C)]
            n = 8
            sz = torch.zeros((n, 3 * len(cfg.fanouts)), dtype=torch.int64).pin_memory()
            dev_seeds = [torch.from_numpy(batches[step]).cuda() for step in range(n)]
            for st in streams:   # the seeds' copies were issued on the current stream
                st.wait_stream(torch.cuda.current_stream())
            for step in range(n):
                s.sample_gather(dev_seeds[step], 0xD00 + step, slot=step, sizes_out=sz[step],
                                pipelined=True, ws=step % C, stream=streams[step % C])
            s.flush()
            torch.cuda.synchronize()
            for step in range(n):
                _check_pipelined(s, ip, ix, cfg, batches[step], 0xD00 + step, step, sz[step])
            pkg.dsp_set_persistent_blocks(s.ctx, 0)
        if scheme == "node":
            # pipelined steps: the launch of step t samples batch t while its
            # loader warps gather batch t-1 from both processes' shards; flush() the last
            sz = torch.zeros((4, 3 * len(cfg.fanouts)), dtype=torch.int64).pin_memory()
            for step in range(4):
                s.sample_gather(torch.from_numpy(batches[step]).cuda(), 0xABC + step, slot=step % 2,
                                sizes_out=sz[step], pipelined=True)
                if step >= 1:  # step-1's features were written by this launch
                    torch.cuda.synchronize()
                    _check_pipelined(s, ip, ix, cfg, batches[step - 1], 0xABC + step - 1, (step - 1) % 2,
                                     sz[step - 1])
            s.flush()
            torch.cuda.synchronize()
            _check_pipelined(s, ip, ix, cfg, batches[3], 0xABC + 3, 1, sz[3])
        # random walks over the partitioned graph: walkers cross processes
        starts = np.random.default_rng(rank).integers(0, cfg.num_nodes, size=400 + 50 * rank).astype(np.int32)
        tr = s.random_walk(torch.from_numpy(starts).cuda(), 16, 0xC0DE)
        s.sync()
        if not np.array_equal(tr.cpu().numpy(), oracle.random_walk(ip, ix, starts, 16, 0xC0DE)):
            ok, detail = False, "random walk traces"
        dist.barrier()
        s.close()
    except Exception as e:  # reported to the parent
        ok, detail = False, repr(e)
    finally:
        q.put((rank, ok, detail))
        dist.destroy_process_group()


@pytest.mark.parametrize("hot,scheme,channels", [(None, "node", 1), (1, "node", 1), (None, "layer", 1),
                                                 (None, "node", 2)])
def test_two_processes_one_gpu(hot, scheme, channels):
    """hot = 1: the cold-feature tier with 3/4 of each shard in host memory
    (POSIX shm mapped into the peer process), read over UVA by both GPUs' gathers.
    channels = 2: two collective calls in flight per rank on two streams
    (DSP_OPT_EXCHANGE_CHANNELS), then the synchronous and pipelined steps on a
    single stream keep rotating through the channels."""
    if not torch.cuda.is_available():
        pytest.fail("needs a GPU")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank, args=(r, 2, port, q, hot, scheme, channels)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=600) for _ in procs)
    for p in procs:
        p.join(timeout=120)
    assert all(ok for _, ok, _ in res), res
