"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle,
bit-exact on every block array and on the gathered feature bits.

Sizes: the tiny config on every batch of an epoch (many tiles + ragged
tails), the products-shaped graph at full size in the launch configuration
bench.py times (whole batches: the oracle finishes one in well under a
second), virtual multi-rank worlds (P = 2, 4, 8 ranks sharing the GPU through
dsp_sample_group, same kernels and peer-write protocol as multi-GPU), the
paper's worked examples, and the edge cases (empty / ragged batches, deg <= k,
k = 1 and k = 32, duplicate and out-of-range seeds)."""
import json
import os

import numpy as np
import pytest

import datagen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


@pytest.fixture(scope="module")
def pkg():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device (run under gpurun)")
    import paper_conf_ppopp_caiz0zszck23_b200 as p
    from paper_conf_ppopp_caiz0zszck23_b200 import _build
    _build.build()
    torch.cuda.set_device(0)
    return p


def assert_blocks_equal(got, ref, where=""):
    assert len(got) == len(ref)
    for l, (b, r) in enumerate(zip(got, ref)):
        assert b.num_dst == r["num_dst"] and b.num_src == r["num_src"] and b.num_edges == r["num_edges"], \
            f"{where} layer {l} sizes {(b.num_dst, b.num_src, b.num_edges)} vs " \
            f"{(r['num_dst'], r['num_src'], r['num_edges'])}"
        for key in ("indptr", "indices", "src_ids"):
            got_a = getattr(b, key).cpu().numpy()
            if not np.array_equal(got_a, r[key]):
                bad = np.nonzero(got_a != r[key])[0][:5] if got_a.shape == r[key].shape else "shape"
                raise AssertionError(f"{where} layer {l} {key} differs at {bad}")


def seeds_of(cfg, P, rank, epoch=0, batch=None):
    train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
    return datagen.rank_seed_batches(train, datagen.bounds(cfg.num_nodes, P), rank, batch or cfg.batch, epoch)


@pytest.fixture(scope="module")
def tiny():
    cfg = datagen.CONFIGS["tiny"]
    ip, ix = datagen.make_graph(cfg)
    feats = datagen.features(0, cfg.num_nodes, cfg.dim)
    return cfg, ip, ix, feats


# ------------------------------------------------------------------- P = 1

def test_tiny_every_batch_of_an_epoch(pkg, tiny):
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, cfg.batch)
    batches = seeds_of(cfg, 1, 0)
    assert len(batches) > 100
    for step, seeds in enumerate(batches):
        rng = datagen.BASE_SEED + step
        blocks = s.sample(torch.from_numpy(seeds).cuda(), rng)
        ref = oracle.sample(ip, ix, seeds, cfg.fanouts, rng)
        assert_blocks_equal(blocks, ref, f"tiny step {step}")
        if step % 10 == 0:
            out = s.gather(blocks[-1].src_ids)
            s.sync()
            exp = oracle.gather(feats, ref[-1]["src_ids"])
            assert np.array_equal(out.cpu().numpy().view(np.uint32), exp.view(np.uint32))
    s.close()


@pytest.mark.parametrize("fanouts", [(1,), (32,), (3, 7, 2), (32, 1), (9, 17)])
def test_fanout_range_and_ragged_batches(pkg, tiny, fanouts):
    """k = 1 (random-walk step), k = 32 (full warp), odd k (ragged lane groups),
    and batch sizes that are not a multiple of anything."""
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, fanouts, 100)
    rng = np.random.default_rng(5)
    for B in (1, 2, 33, 97, 100):
        seeds = rng.choice(cfg.num_nodes, size=B, replace=False).astype(np.int32)
        blocks = s.sample(torch.from_numpy(seeds).cuda(), 1000 + B)
        assert_blocks_equal(blocks, oracle.sample(ip, ix, seeds, fanouts, 1000 + B), f"B={B}")
    s.close()


@pytest.mark.parametrize("relabel", ["direct", "direct64", "hash"])
def test_maximum_layers_and_fanout(pkg, tiny, relabel):
    """The ABI's limits: 8 layers of fan-out 32 (the frontier saturates at all
    N nodes, every row of degree <= 32 is taken whole), on each relabel layout
    (DSP_OPT_RELABEL_MAP); fused gather of the last block (every node) and a
    pipelined call."""
    cfg, ip, ix, feats = tiny
    fan = (32,) * 8
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, fan, 64, n_slots=2,
                    options={pkg.dsp.DSP_OPT_RELABEL_MAP: pkg.dsp.RELABEL_MAPS[relabel]})
    seeds = np.random.default_rng(8).choice(cfg.num_nodes, size=64, replace=False).astype(np.int32)
    blocks, feat = s.sample_gather(torch.from_numpy(seeds).cuda(), 77, slot=0)
    ref = oracle.sample(ip, ix, seeds, fan, 77)
    assert_blocks_equal(blocks, ref, f"max {relabel}")
    assert blocks[-1].num_src == len(np.unique(ref[-1]["src_ids"]))
    assert np.array_equal(feat.cpu().numpy().view(np.uint32), oracle.gather(feats, ref[-1]["src_ids"]).view(np.uint32))
    s.close()


def test_empty_batch(pkg, tiny):
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, 8)
    blocks = s.sample(torch.zeros(0, dtype=torch.int32, device="cuda"), 3)
    assert all(b.num_dst == 0 and b.num_edges == 0 and b.num_src == 0 for b in blocks)
    assert blocks[0].indptr.cpu().tolist() == [0]
    s.close()


def test_errors_latched_and_reported(pkg, tiny):
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, 16)
    with pytest.raises(pkg.DSPError) as e:
        s.sample(torch.tensor([5, 9, 5], dtype=torch.int32, device="cuda"), 1)
    assert e.value.status == pkg.dsp.DSP_ERR_DUPLICATE_SEED
    with pytest.raises(pkg.DSPError) as e:
        s.sample(torch.tensor([5, cfg.num_nodes], dtype=torch.int32, device="cuda"), 1)
    assert e.value.status == pkg.dsp.DSP_ERR_OUT_OF_RANGE
    with pytest.raises(pkg.DSPError) as e:
        s.sample(torch.arange(17, dtype=torch.int32, device="cuda"), 1)
    assert e.value.status == pkg.dsp.DSP_ERR_CAPACITY
    # the ctx stays usable after a device-detected error
    seeds = np.array([1, 2, 3], np.int32)
    assert_blocks_equal(s.sample(torch.from_numpy(seeds).cuda(), 4), oracle.sample(ip, ix, seeds, cfg.fanouts, 4))
    with pytest.raises(pkg.DSPError) as e:
        s.gather(torch.tensor([-1], dtype=torch.int32, device="cuda"))
        s.sync()
    assert e.value.status == pkg.dsp.DSP_ERR_OUT_OF_RANGE
    s.close()


def _csr_from_rows(n, rows):
    ip = np.zeros(n + 1, np.int64)
    cols = []
    for v in range(n):
        r = sorted(rows.get(str(v), []))
        cols += r
        ip[v + 1] = ip[v] + len(r)
    return ip, np.array(cols, np.int32)


def test_fig3_worked_example_on_gpu(pkg):
    g = json.load(open(os.path.join(GOLDEN, "fig3_worked_example.json")))
    ip, ix = _csr_from_rows(g["num_nodes"], g["rows"])
    feats = datagen.features(0, g["num_nodes"], 4)
    s = pkg.Sampler([0, g["num_nodes"]], ip, ix, feats, g["fanouts"], 1)
    blocks = s.sample(torch.tensor(g["seeds"], dtype=torch.int32, device="cuda"), 77)
    for b, e in zip(blocks, g["blocks"]):
        for key in ("indptr", "indices", "src_ids"):
            assert getattr(b, key).cpu().tolist() == e[key]
    s.close()


def test_fig5_csp_example_virtual_two_gpus(pkg):
    g = json.load(open(os.path.join(GOLDEN, "fig5_csp_example.json")))
    ip, ix = _csr_from_rows(g["num_nodes"], g["rows"])
    bnds = np.array(g["bounds"], np.int64)
    feats = datagen.features(0, g["num_nodes"], 4)
    shards = []
    for r in range(2):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi]))
    grp = pkg.LocalGroup(bnds, shards, g["fanouts"], 2, devices=[0, 0])
    seeds = [torch.tensor(x, dtype=torch.int32, device="cuda") for x in g["rank_seeds"]]
    res = grp.sample(seeds, 9)
    for r in range(2):
        for b, e in zip(res[r], g["blocks"][r]):
            for key in ("indptr", "indices", "src_ids"):
                assert getattr(b, key).cpu().tolist() == e[key], (r, key)
        # one-sided gather across the two shards
        out = grp.samplers[r].gather(res[r][-1].src_ids)
        grp.samplers[r].sync()
        assert np.array_equal(out.cpu().numpy(), feats[res[r][-1].src_ids.cpu().numpy()])
    grp.close()


# ------------------------------------------------------- virtual P = 2,4,8

@pytest.mark.parametrize("mode", ["direct", "hash"])
@pytest.mark.parametrize("P", [2, 4, 8])
def test_tiny_virtual_ranks(pkg, tiny, P, mode):
    """world > 1: one persistent kernel per rank (virtual ranks each on 1/P of
    the SMs, own stream), with the compact direct or the hashed relabel map."""
    cfg, ip, ix, feats = tiny
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi]))
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, 32, devices=[0] * P,
                         options={pkg.dsp.DSP_OPT_RELABEL_MAP: pkg.dsp.RELABEL_MAPS[mode]})
    per_rank = [seeds_of(cfg, P, r, batch=32) for r in range(P)]
    steps = min(len(x) for x in per_rank)
    for step in range(min(steps, 6)):
        seeds = [per_rank[r][step] for r in range(P)]
        if step == 1:
            seeds[0] = seeds[0][:0]                  # a rank with an empty batch still joins
        if step == 2:
            seeds[P - 1] = np.concatenate([seeds[P - 1][:5], per_rank[0][step][:3]])  # remote seeds
        res = grp.sample([torch.from_numpy(np.ascontiguousarray(s)).cuda() for s in seeds], 0x5EED + step)
        for r in range(P):
            ref = oracle.sample(ip, ix, seeds[r], cfg.fanouts, 0x5EED + step)
            assert_blocks_equal(res[r], ref, f"P={P} rank {r} step {step}")
            out = grp.samplers[r].gather(res[r][-1].src_ids)
            grp.samplers[r].sync()
            exp = oracle.gather(feats, ref[-1]["src_ids"])
            assert np.array_equal(out.cpu().numpy().view(np.uint32), exp.view(np.uint32))
    grp.close()


@pytest.mark.parametrize("P", [2, 4])
def test_virtual_ranks_exchange_channels(pkg, tiny, P):
    """DSP_OPT_EXCHANGE_CHANNELS = 3: consecutive collective calls rotate over
    three exchange regions with their own sequence numbers (a duplicate-seed
    error in between must not desynchronise the rotation); every call equals
    the oracle."""
    cfg, ip, ix, feats = tiny
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi]))
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, 32, devices=[0] * P,
                         options={pkg.dsp.DSP_OPT_EXCHANGE_CHANNELS: 3})
    per_rank = [seeds_of(cfg, P, r, batch=32) for r in range(P)]
    for step in range(8):
        seeds = [per_rank[r][step] for r in range(P)]
        if step == 4:
            bad = [np.ascontiguousarray(x) for x in seeds]
            bad[0] = np.concatenate([bad[0][:3], bad[0][:1]])
            with pytest.raises(pkg.DSPError) as e:
                grp.sample([torch.from_numpy(x).cuda() for x in bad], 9)
            assert e.value.status == pkg.dsp.DSP_ERR_DUPLICATE_SEED
        res = grp.sample([torch.from_numpy(np.ascontiguousarray(x)).cuda() for x in seeds], 0x600 + step)
        for r in range(P):
            assert_blocks_equal(res[r], oracle.sample(ip, ix, seeds[r], cfg.fanouts, 0x600 + step), f"P={P} r{r} {step}")
    grp.close()


@pytest.mark.parametrize("P,K", [(2, 2), (4, 3)])
def test_virtual_ranks_concurrent_group_calls(pkg, tiny, P, K):
    """K asynchronous group calls in flight on K streams (DSP_ASYNC group calls,
    DSP_OPT_EXCHANGE_CHANNELS = K, each rank's launch on 1/(P*K) of the SMs),
    each into its own workspace and output set; every rank's blocks equal the
    oracle (sizes from the oracle, array contents compared)."""
    cfg, ip, ix, feats = tiny
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi]))
    n = 2 * K
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, 32, devices=[0] * P, n_workspaces=K, n_slots=n,
                         options={pkg.dsp.DSP_OPT_EXCHANGE_CHANNELS: K})
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    for s in grp.samplers:
        pkg.dsp_set_persistent_blocks(s.ctx, max(1, sms // (P * K)))
    per_rank = [seeds_of(cfg, P, r, batch=32) for r in range(P)]
    dev = [[torch.from_numpy(np.ascontiguousarray(per_rank[r][i])).cuda() for r in range(P)] for i in range(n)]
    streams = [torch.cuda.Stream() for _ in range(K)]
    torch.cuda.synchronize()
    for i in range(n):   # call i: stream / workspace i % K, output set i (calls i and i + K share a workspace)
        grp.sample(dev[i], 0x900 + i, async_=True, ws=i % K, slot=i, stream=streams[i % K])
    torch.cuda.synchronize()
    for s in grp.samplers:
        s.sync()
    for i in range(n):
        for r in range(P):
            ref = oracle.sample(ip, ix, per_rank[r][i], cfg.fanouts, 0x900 + i)
            sizes = [x for b in ref for x in (b["num_dst"], b["num_src"], b["num_edges"])]
            assert_blocks_equal(grp.samplers[r].blocks(i, sizes), ref, f"P={P} K={K} call {i} rank {r}")
    grp.close()


@pytest.mark.parametrize("mode", ["direct", "hash"])
def test_virtual_ranks_errors(pkg, tiny, mode):
    """Device-detected errors at world > 1 (duplicate seed, out-of-range seed)
    are reported by the group call after the exchange protocol completed, and
    the ranks stay usable; a batch above the reserved size fails before any
    launch on every rank."""
    cfg, ip, ix, feats = tiny
    P = 2
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi]))
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, 16, devices=[0] * P,
                         options={pkg.dsp.DSP_OPT_RELABEL_MAP: pkg.dsp.RELABEL_MAPS[mode]})
    t = lambda x: torch.tensor(x, dtype=torch.int32, device="cuda")
    with pytest.raises(pkg.DSPError) as e:
        grp.sample([t([5, 9, 5]), t([7000])], 1)
    assert e.value.status == pkg.dsp.DSP_ERR_DUPLICATE_SEED
    with pytest.raises(pkg.DSPError) as e:
        grp.sample([t([5]), t([7000, cfg.num_nodes])], 1)
    assert e.value.status == pkg.dsp.DSP_ERR_OUT_OF_RANGE
    with pytest.raises(pkg.DSPError) as e:
        grp.sample([t(list(range(17))), t([7000])], 1)
    assert e.value.status == pkg.dsp.DSP_ERR_CAPACITY
    seeds = [np.array([1, 9000, 3], np.int32), np.array([7000, 2], np.int32)]
    res = grp.sample([torch.from_numpy(x).cuda() for x in seeds], 4)
    for r in range(P):
        assert_blocks_equal(res[r], oracle.sample(ip, ix, seeds[r], cfg.fanouts, 4), f"{mode} rank {r} after errors")
    grp.close()


@pytest.mark.parametrize("mode", ["direct", "hash"])
def test_virtual_ranks_all_empty(pkg, tiny, mode):
    """Every rank with an empty batch: the exchange still runs (empty inboxes),
    every block comes back empty, and the next call is unaffected."""
    cfg, ip, ix, feats = tiny
    P = 2
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi]))
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, 16, devices=[0] * P,
                         options={pkg.dsp.DSP_OPT_RELABEL_MAP: pkg.dsp.RELABEL_MAPS[mode]})
    empty = torch.zeros(0, dtype=torch.int32, device="cuda")
    res = grp.sample([empty, empty], 3)
    for r in range(P):
        assert all(b.num_dst == 0 and b.num_src == 0 and b.num_edges == 0 for b in res[r])
        assert res[r][0].indptr.cpu().tolist() == [0]
    seeds = [np.array([3, 9000], np.int32), np.array([7, 5001], np.int32)]
    res = grp.sample([torch.from_numpy(x).cuda() for x in seeds], 4)
    for r in range(P):
        assert_blocks_equal(res[r], oracle.sample(ip, ix, seeds[r], cfg.fanouts, 4), f"{mode} rank {r}")
    grp.close()


# ----------------------------------------------------- products, full size

@pytest.fixture(scope="module")
def products():
    cfg = datagen.CONFIGS["products"]
    ip, ix = datagen.make_graph(cfg)
    return cfg, ip, ix


@pytest.mark.slow
def test_products_full_size_p1(pkg, products):
    """BASELINE.json configs[1] in bench.py's launch configuration: whole
    1024-seed batches compared bit-exactly; the gather checked on every row
    against the closed-form feature recipe."""
    cfg, ip, ix = products
    feats = datagen.features(0, cfg.num_nodes, cfg.dim)
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, cfg.batch)
    batches = seeds_of(cfg, 1, 0)
    for step in (0, 1, len(batches) - 1):
        seeds = batches[step]
        rng = datagen.BASE_SEED + step
        blocks = s.sample(torch.from_numpy(seeds).cuda(), rng)
        ref = oracle.sample(ip, ix, seeds, cfg.fanouts, rng)
        assert_blocks_equal(blocks, ref, f"products step {step}")
        out = s.gather(blocks[-1].src_ids)
        s.sync()
        exp = datagen.features_of(ref[-1]["src_ids"], cfg.dim)
        assert np.array_equal(out.cpu().numpy().view(np.uint32), exp.view(np.uint32))
    s.close()


@pytest.mark.slow
def test_products_virtual_p4(pkg, products):
    cfg, ip, ix = products
    P = 4
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, datagen.features(lo, hi, cfg.dim)))
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, cfg.batch, devices=[0] * P)
    seeds = [seeds_of(cfg, P, r)[0] for r in range(P)]
    res = grp.sample([torch.from_numpy(s).cuda() for s in seeds], 0x5EED)
    for r in range(P):
        assert_blocks_equal(res[r], oracle.sample(ip, ix, seeds[r], cfg.fanouts, 0x5EED), f"rank {r}")
    out = grp.samplers[1].gather(res[1][-1].src_ids)
    grp.samplers[1].sync()
    exp = datagen.features_of(res[1][-1].src_ids.cpu().numpy(), cfg.dim)
    assert np.array_equal(out.cpu().numpy().view(np.uint32), exp.view(np.uint32))
    grp.close()


# ------------------------------------------------------ fused step (one call)

def test_sample_gather_sync_and_async(pkg, tiny):
    """dsp_sample_gather: the whole step in one call (one persistent kernel at
    world 1); synchronous and DSP_ASYNC with two alternating output sets."""
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2)
    batches = seeds_of(cfg, 1, 0)
    for step in range(4):
        blocks, feat = s.sample_gather(torch.from_numpy(batches[step]).cuda(), 50 + step, slot=step % 2)
        ref = oracle.sample(ip, ix, batches[step], cfg.fanouts, 50 + step)
        assert_blocks_equal(blocks, ref, f"sync step {step}")
        assert np.array_equal(feat.cpu().numpy().view(np.uint32),
                              oracle.gather(feats, ref[-1]["src_ids"]).view(np.uint32))
    L = len(cfg.fanouts)
    sizes = torch.zeros((6, 3 * L), dtype=torch.int64).pin_memory()
    dev = [torch.from_numpy(batches[10 + j]).cuda() for j in range(6)]
    for j in range(6):
        s.sample_gather(dev[j], 900 + j, slot=j % 2, sizes_out=sizes[j], async_=True)
    s.sync()
    for j in range(6):
        ref = oracle.sample(ip, ix, batches[10 + j], cfg.fanouts, 900 + j)
        exp = [v for r in ref for v in (r["num_dst"], r["num_src"], r["num_edges"])]
        assert sizes[j].tolist() == exp
        if j >= 4:   # the last two steps are still in the two output sets
            blocks = s.blocks(j % 2, sizes=sizes[j].tolist())
            assert_blocks_equal(blocks, ref, f"async step {j}")
            feat = s.feat_buffer(j % 2)[: blocks[-1].num_src]
            assert np.array_equal(feat.cpu().numpy().view(np.uint32),
                                  oracle.gather(feats, ref[-1]["src_ids"]).view(np.uint32))
    s.close()


@pytest.mark.slow
def test_products_fused_step(pkg, products):
    cfg, ip, ix = products
    feats = datagen.features(0, cfg.num_nodes, cfg.dim)
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2)
    batches = seeds_of(cfg, 1, 0)
    for step in (5, 6):
        blocks, feat = s.sample_gather(torch.from_numpy(batches[step]).cuda(), 7 + step, slot=step % 2)
        ref = oracle.sample(ip, ix, batches[step], cfg.fanouts, 7 + step)
        assert_blocks_equal(blocks, ref, f"products fused step {step}")
        exp = datagen.features_of(ref[-1]["src_ids"], cfg.dim)
        assert np.array_equal(feat.cpu().numpy().view(np.uint32), exp.view(np.uint32))
    s.close()


def _check_step(s, slot, sizes, seeds, rng, ip, ix, feats_of, weights=None):
    ref = oracle.sample(ip, ix, seeds, s.fanouts, rng, weights=weights)
    exp = [v for r in ref for v in (r["num_dst"], r["num_src"], r["num_edges"])]
    assert [int(x) for x in sizes] == exp
    blocks = s.blocks(slot, sizes=[int(x) for x in sizes])
    assert_blocks_equal(blocks, ref, f"pipelined rng {rng}")
    feat = s.feat_buffer(slot)[: blocks[-1].num_src]
    assert np.array_equal(feat.cpu().numpy().view(np.uint32), feats_of(ref[-1]["src_ids"]).view(np.uint32))


def test_pipelined_steps_biased(pkg, tiny, tiny_weights):
    """DSP_PIPELINED with DSP_BIASED (its own launch shape: fewer loader warps)."""
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2,
                    edge_weights=tiny_weights)
    batches = seeds_of(cfg, 1, 0)
    L = len(cfg.fanouts)
    sizes = torch.zeros((6, 3 * L), dtype=torch.int64).pin_memory()
    for j in range(6):
        s.sample_gather(torch.from_numpy(batches[j]).cuda(), 500 + j, slot=j % 2, sizes_out=sizes[j],
                        pipelined=True, biased=True)
        if j >= 1:
            s.sync()
            ref = oracle.sample(ip, ix, batches[j - 1], cfg.fanouts, 500 + j - 1, weights=tiny_weights)
            assert [int(x) for x in sizes[j - 1]] == [v for r in ref for v in (r["num_dst"], r["num_src"], r["num_edges"])]
            blocks = s.blocks((j - 1) % 2, sizes=[int(x) for x in sizes[j - 1]])
            assert_blocks_equal(blocks, ref, f"biased pipelined step {j - 1}")
            feat = s.feat_buffer((j - 1) % 2)[: blocks[-1].num_src]
            assert np.array_equal(feat.cpu().numpy(), oracle.gather(feats, ref[-1]["src_ids"]))
    s.flush()
    s.sync()
    s.close()


def test_pipelined_steps(pkg, tiny):
    """DSP_PIPELINED: step j samples batch j while its loader warps gather the
    features of batch j-1; flush gathers the last one."""
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2)
    batches = seeds_of(cfg, 1, 0)
    L = len(cfg.fanouts)
    sizes = torch.zeros((8, 3 * L), dtype=torch.int64).pin_memory()
    feats_of = lambda ids: oracle.gather(feats, ids)
    for j in range(8):
        s.sample_gather(torch.from_numpy(batches[j]).cuda(), 300 + j, slot=j % 2, sizes_out=sizes[j], pipelined=True)
        if j >= 1:
            s.sync()
            _check_step(s, (j - 1) % 2, sizes[j - 1], batches[j - 1], 300 + j - 1, ip, ix, feats_of)
    s.flush()
    s.sync()
    _check_step(s, 7 % 2, sizes[7], batches[7], 307, ip, ix, feats_of)
    # a non-pipelined call after pipelined ones settles nothing twice and still matches
    blocks, feat = s.sample_gather(torch.from_numpy(batches[9]).cuda(), 99, slot=0)
    assert_blocks_equal(blocks, oracle.sample(ip, ix, batches[9], cfg.fanouts, 99))
    s.close()


@pytest.mark.slow
def test_products_pipelined(pkg, products):
    cfg, ip, ix = products
    feats = datagen.features(0, cfg.num_nodes, cfg.dim)
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2)
    batches = seeds_of(cfg, 1, 0)
    L = len(cfg.fanouts)
    sizes = torch.zeros((3, 3 * L), dtype=torch.int64).pin_memory()
    feats_of = lambda ids: datagen.features_of(ids, cfg.dim)
    for j in range(3):
        s.sample_gather(torch.from_numpy(batches[20 + j]).cuda(), 40 + j, slot=j % 2, sizes_out=sizes[j],
                        pipelined=True)
    s.sync()
    _check_step(s, 1, sizes[1], batches[21], 41, ip, ix, feats_of)
    s.flush()
    s.sync()
    _check_step(s, 0, sizes[2], batches[22], 42, ip, ix, feats_of)
    s.close()


@pytest.mark.slow
@pytest.mark.parametrize("biased", [False, True])
def test_products_bench_launch_configuration(pkg, products, biased):
    """configs[1] at full size in exactly the launch configuration bench.py
    times: K concurrent step streams (2 for uniform steps, 4 for biased ones),
    each pipelined persistent launch on 148 / K SMs with its own workspace,
    2K output sets, sizes returned asynchronously;
    every step whose output set survives is checked against the oracle
    (blocks bit-exact, every gathered row against the closed-form features)."""
    cfg, ip, ix = products
    feats = datagen.features(0, cfg.num_nodes, cfg.dim)
    ew = datagen.edge_weights(ix, datagen.node_weights(cfg.num_nodes)) if biased else None
    K = 4 if biased else 2
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2 * K,
                    n_workspaces=K, edge_weights=ew)
    pkg.dsp_set_persistent_blocks(s.ctx, torch.cuda.get_device_properties(0).multi_processor_count // K)
    batches = seeds_of(cfg, 1, 0)
    L = len(cfg.fanouts)
    n = 12
    sizes = torch.zeros((n, 3 * L), dtype=torch.int64).pin_memory()
    dev = [torch.from_numpy(batches[i]).cuda() for i in range(n)]   # resident, as in bench.py
    main = torch.cuda.current_stream()
    streams = [torch.cuda.Stream() for _ in range(K)]
    for st in streams:
        st.wait_stream(main)
    for i in range(n):
        s.sample_gather(dev[i], 0x5EED + i, slot=i % (2 * K), sizes_out=sizes[i],
                        async_=True, pipelined=True, biased=biased, ws=i % K, stream=streams[i % K])
    for st in streams:
        with torch.cuda.stream(st):
            s.flush()
    for st in streams:
        main.wait_stream(st)
    s.sync()
    torch.cuda.synchronize()
    feats_of = lambda ids: datagen.features_of(ids, cfg.dim)
    for i in range(n - 2 * K, n):
        _check_step(s, i % (2 * K), sizes[i], batches[i], 0x5EED + i, ip, ix, feats_of, weights=ew)
    s.close()


# ------------------------------------------------------------ biased

@pytest.fixture(scope="module")
def tiny_weights(tiny):
    cfg, ip, ix, feats = tiny
    return datagen.edge_weights(ix, datagen.node_weights(cfg.num_nodes))


@pytest.mark.parametrize("fanouts", [(5, 5), (1, 32), (15, 10, 5)])
def test_biased_tiny(pkg, tiny, tiny_weights, fanouts):
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, fanouts, 64, edge_weights=tiny_weights)
    batches = seeds_of(cfg, 1, 0)
    for step in range(6):
        blocks = s.sample(torch.from_numpy(batches[step]).cuda(), 70 + step, biased=True)
        ref = oracle.sample(ip, ix, batches[step], fanouts, 70 + step, weights=tiny_weights)
        assert_blocks_equal(blocks, ref, f"biased step {step}")
    blocks, feat = s.sample_gather(torch.from_numpy(batches[7]).cuda(), 5, biased=True)
    ref = oracle.sample(ip, ix, batches[7], fanouts, 5, weights=tiny_weights)
    assert_blocks_equal(blocks, ref, "biased fused")
    assert np.array_equal(feat.cpu().numpy(), oracle.gather(feats, ref[-1]["src_ids"]))
    s.close()


@pytest.mark.parametrize("P", [2, 4])
def test_biased_virtual_ranks(pkg, tiny, tiny_weights, P):
    cfg, ip, ix, feats = tiny
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi], tiny_weights[ip[lo]:ip[hi]]))
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, 32, devices=[0] * P)
    seeds = [seeds_of(cfg, P, r, batch=32)[0] for r in range(P)]
    res = grp.sample([torch.from_numpy(x).cuda() for x in seeds], 0xB1A5, biased=True)
    for r in range(P):
        assert_blocks_equal(res[r], oracle.sample(ip, ix, seeds[r], cfg.fanouts, 0xB1A5, weights=tiny_weights),
                            f"biased P={P} rank {r}")
    grp.close()


def _long_row_graph(heavy=False):
    """30k nodes, rows of degree <= 40 plus hubs of degree 300 / 1000 / 5000
    (chunk-sum path, 256 < d <= 8192), 9000 / 20000 (very long rows), and a hub
    whose 5000 weights are all zero but 3 (every positive one taken, no draw).
    Weights below 714 keep every running weight of a row of <= 256 positions
    under 2^32 (the 32-bit rounds of the register path); heavy weights (up to
    65535) push rows of more than 32 positions past it (the 64-bit rounds)."""
    rng = np.random.default_rng(31)
    N = 30000
    degs = rng.integers(0, 41, size=N)
    hubs = {0: 300, 1: 1000, 2: 5000, 3: 9000, 4: 20000, 5: 5000}
    for h, d in hubs.items():
        degs[h] = d
    rows = []
    for v in range(N):
        nb = rng.choice(N - 1, size=int(degs[v]), replace=False)
        nb[nb >= v] += 1   # no self loop
        rows.append(np.sort(nb))
    ip = np.zeros(N + 1, np.int64)
    ip[1:] = np.cumsum([len(r) for r in rows])
    ix = np.concatenate(rows).astype(np.int32)
    w = (rng.integers(0, 5000, size=len(ix)) / 7.0).astype(np.float32)
    if heavy:
        w = (w * 91.75).astype(np.float32)
    w[rng.random(len(ix)) < 0.1] = 0.0
    w[ip[5]:ip[6]] = 0.0
    w[ip[5] + np.array([7, 2000, 4999])] = 3.5
    return N, ip, ix, w


@pytest.mark.parametrize("heavy", [False, True])
def test_biased_long_rows(pkg, heavy):
    """Biased sampling on every row-length path of the warp sampler (one
    position per lane, registers with 32- or 64-bit running weights, chunk
    sums, very long rows, <= k positive weights) at P = 1 and at virtual P = 2
    (the owner-side sampler of the multi-rank kernel)."""
    N, ip, ix, w = _long_row_graph(heavy)
    if heavy:
        wf = np.floor(w.astype(np.float64) * 65536)
        big = [v for v in range(6, N) if 32 < ip[v + 1] - ip[v] and wf[ip[v]:ip[v + 1]].sum() >= 2 ** 32]
        assert len(big) > 1000
    feats = datagen.features(0, N, 4)
    fan = (15, 10)
    seeds = np.array([0, 1, 2, 3, 4, 5, 11, 29999, 15000], np.int32)
    s = pkg.Sampler(datagen.bounds(N, 1), ip, ix, feats, fan, 16, edge_weights=w)
    for rng in (1, 2, 3):
        blocks = s.sample(torch.from_numpy(seeds).cuda(), rng, biased=True)
        assert_blocks_equal(blocks, oracle.sample(ip, ix, seeds, fan, rng, weights=w), f"long rows rng {rng}")
    s.close()
    bnds = datagen.bounds(N, 2)
    shards = []
    for r in range(2):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi], w[ip[lo]:ip[hi]]))
    grp = pkg.LocalGroup(bnds, shards, fan, 16, devices=[0, 0])
    rs = [seeds[:6], seeds[6:]]
    res = grp.sample([torch.from_numpy(np.ascontiguousarray(x)).cuda() for x in rs], 9, biased=True)
    for r in range(2):
        assert_blocks_equal(res[r], oracle.sample(ip, ix, rs[r], fan, 9, weights=w), f"long rows P=2 rank {r}")
    grp.close()


def _group_boundary_graph():
    """Rows on both sides of every boundary of the biased sampler (lane groups
    of 8 / 16 / 32 lanes x 8 positions: degrees 64 / 128 / 256; aligned
    chunk sums up to 4 x 32 lines, then re-reads), at every alignment of the
    row start inside a 128-byte line, with weights in (0, 256] (the lane-group
    limit is 2^24 = 256.0 in 16.16), some heavier than 256 (the warp-wide
    sampler takes those rows), zero weights, a row of 256 weights of exactly
    256.0 (its total is 2^32: the 32-bit running weights would wrap, so the
    warp-wide sampler takes it) and rows whose positive weights are <= k."""
    rng = np.random.default_rng(77)
    special = [0, 1, 2, 5, 7, 8, 9, 16, 17, 31, 32, 33, 63, 64, 65, 100, 127, 128, 129, 200, 255, 256, 257,
               300, 1000, 4000, 4033, 4064, 4065, 4100, 6000]
    N = 20000
    degs = rng.integers(0, 60, size=N)
    hubs = []
    for r, d in enumerate(special * 3):
        hubs.append(r)
        degs[r] = d
    rows = []
    for v in range(N):
        nb = rng.choice(N - 1, size=int(degs[v]), replace=False)
        nb[nb >= v] += 1
        rows.append(np.sort(nb))
    ip = np.zeros(N + 1, np.int64)
    ip[1:] = np.cumsum([len(r) for r in rows])
    ix = np.concatenate(rows).astype(np.int32)
    w = (rng.integers(1, 4097, size=len(ix)) / 16.0).astype(np.float32)   # (0, 256], exact in 16.16
    w[rng.random(len(ix)) < 0.05] = 0.0
    n = len(special)
    heavy_rows = list(range(n, 2 * n))          # second copy: a few weights above 256
    for v in heavy_rows:
        a, b = ip[v], ip[v + 1]
        if b > a:
            w[a + rng.integers(0, b - a, size=max(1, (b - a) // 16))] = 300.5
    full = special.index(256) + 2 * n            # third copy of degree 256: every weight 256.0
    w[ip[full]:ip[full + 1]] = 256.0
    few = special.index(100) + 2 * n             # third copy of degree 100: 3 positive weights
    w[ip[few]:ip[few + 1]] = 0.0
    w[ip[few] + np.array([3, 50, 99])] = 1.5
    return N, ip, ix, w, hubs


@pytest.mark.parametrize("fan", [(5, 3), (8, 1), (9, 16), (17, 2), (32, 5)])
def test_biased_group_boundaries(pkg, fan):
    N, ip, ix, w, hubs = _group_boundary_graph()
    feats = datagen.features(0, N, 4)
    seeds = np.array(hubs, np.int32)
    s = pkg.Sampler(datagen.bounds(N, 1), ip, ix, feats, fan, len(seeds), edge_weights=w)
    for rng_seed in (3, 4):
        blocks = s.sample(torch.from_numpy(seeds).cuda(), rng_seed, biased=True)
        assert_blocks_equal(blocks, oracle.sample(ip, ix, seeds, fan, rng_seed, weights=w), f"fan {fan} rng {rng_seed}")
    s.close()
    # the owner-side sampler of the multi-rank kernel (virtual P = 2)
    bnds = datagen.bounds(N, 2)
    shards = []
    for r in range(2):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi], w[ip[lo]:ip[hi]]))
    grp = pkg.LocalGroup(bnds, shards, fan, len(seeds), devices=[0, 0])
    rs = [seeds[seeds < bnds[1]], seeds[seeds >= bnds[1]]]
    res = grp.sample([torch.from_numpy(np.ascontiguousarray(x)).cuda() for x in rs], 11, biased=True)
    for r in range(2):
        assert_blocks_equal(res[r], oracle.sample(ip, ix, rs[r], fan, 11, weights=w), f"fan {fan} P=2 rank {r}")
    grp.close()


def test_biased_errors(pkg, tiny):
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, 8)
    with pytest.raises(pkg.DSPError) as e:   # no weights loaded
        s.sample(torch.arange(4, dtype=torch.int32, device="cuda"), 1, biased=True)
    assert e.value.status == pkg.dsp.DSP_ERR_STATE
    s.close()
    # negative, >= 2^16, NaN, and positive weights below 2^-16 (they would quantize
    # to 0 in 16.16 fixed point and never be sampled, R24) are rejected
    for x in (-1.0, 65536.0, float("nan"), 2.0 ** -17, 1e-30):
        bad = np.ones(len(ix), np.float32)
        bad[7] = x
        with pytest.raises(pkg.DSPError) as e:
            pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, 8, edge_weights=bad)
        assert e.value.status == pkg.dsp.DSP_ERR_INVALID_ARG, x
    ok = np.ones(len(ix), np.float32)
    ok[7], ok[8] = 0.0, 2.0 ** -16          # zero and the smallest positive fixed-point weight are accepted
    pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, 8, edge_weights=ok).close()


# ------------------------------------------------------ random walks

def test_random_walks_tiny(pkg, tiny):
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, 8)
    isolated = np.nonzero(np.diff(ip) == 0)[0][:3]
    starts = np.concatenate([np.arange(0, 10_000, 7), isolated, [5, 5]]).astype(np.int32)
    for L in (1, 5, 80):
        tr = s.random_walk(torch.from_numpy(starts).cuda(), L, 0xA11 + L)
        s.sync()
        assert np.array_equal(tr.cpu().numpy(), oracle.random_walk(ip, ix, starts, L, 0xA11 + L)), L
    with pytest.raises(pkg.DSPError):
        s.random_walk(torch.tensor([cfg.num_nodes], dtype=torch.int32, device="cuda"), 3, 1)
        s.sync()
    s.close()


@pytest.mark.parametrize("P", [2, 4, 8])
def test_random_walks_virtual_ranks(pkg, tiny, P):
    """Walks over a partitioned graph (CSP push, reshuffle removed):
    every rank's traces equal the single-device oracle's, whatever P; walks
    start on any owner, meet, terminate at isolated nodes; a rank with no
    walks still takes part; repeated calls reuse the exchange region."""
    cfg, ip, ix, feats = tiny
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi]))
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, 8, devices=[0] * P, max_walks=3000, max_walk_length=64)
    isolated = np.nonzero(np.diff(ip) == 0)[0][:2].astype(np.int32)
    rng = np.random.default_rng(P)
    for call, L in enumerate((1, 7, 64)):
        starts = [rng.integers(0, cfg.num_nodes, size=int(rng.integers(1, 3000)), dtype=np.int64).astype(np.int32)
                  for _ in range(P)]
        starts[0] = np.concatenate([starts[0], isolated, starts[0][:3]])   # dead ends + shared walkers
        if call == 1:
            starts[P - 1] = starts[P - 1][:0]                              # a rank without walks
        tr = grp.random_walk([torch.from_numpy(x).cuda() for x in starts], L, 0xBEEF + L)
        for r in range(P):
            grp.samplers[r].sync()
            exp = oracle.random_walk(ip, ix, starts[r], L, 0xBEEF + L)
            assert np.array_equal(tr[r].cpu().numpy(), exp), (P, r, L)
    with pytest.raises(pkg.DSPError) as e:   # beyond the reserved length
        grp.random_walk([torch.zeros(1, dtype=torch.int32, device="cuda") for _ in range(P)], 65, 1)
    assert e.value.status == pkg.dsp.DSP_ERR_CAPACITY
    grp.close()


@pytest.mark.parametrize("P", [1, 2, 4])
def test_random_walks_independent(pkg, tiny, P):
    """DSP_WALK_INDEPENDENT (R35): walk i draws with its own index, so the
    repeated starts of one call give different walks; traces equal the
    oracle's independent mode at P = 1 (thread per walk) and across virtual
    ranks (CSP push: the walk index travels with the walker)."""
    cfg, ip, ix, feats = tiny
    rng = np.random.default_rng(40 + P)
    hub = int(np.argmax(np.diff(ip)))
    starts = [np.concatenate([np.full(200, hub, np.int32),
                              rng.integers(0, cfg.num_nodes, size=300).astype(np.int32)]) for _ in range(P)]
    L = 20
    if P == 1:
        s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, 8)
        trs = [s.random_walk(torch.from_numpy(starts[0]).cuda(), L, 0xFEED, independent=True)]
        s.sync()
        s.close()
    else:
        bnds = datagen.bounds(cfg.num_nodes, P)
        shards = [datagen.shard(ip, ix, int(bnds[r]), int(bnds[r + 1])) + (feats[int(bnds[r]):int(bnds[r + 1])],)
                  for r in range(P)]
        grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, 8, devices=[0] * P, max_walks=1000, max_walk_length=32)
        trs = grp.random_walk([torch.from_numpy(x).cuda() for x in starts], L, 0xFEED, independent=True)
        for smp in grp.samplers:
            smp.sync()
        grp.close()
    for r in range(P):
        got = trs[r].cpu().numpy()
        assert np.array_equal(got, oracle.random_walk(ip, ix, starts[r], L, 0xFEED, independent=True)), (P, r)
        assert len({tuple(row) for row in got[:200]}) > 150      # the 200 walks from the hub differ


def test_random_walks_need_reservation(pkg, tiny):
    cfg, ip, ix, feats = tiny
    bnds = datagen.bounds(cfg.num_nodes, 2)
    shards = [datagen.shard(ip, ix, int(bnds[r]), int(bnds[r + 1])) + (feats[int(bnds[r]):int(bnds[r + 1])],)
              for r in range(2)]
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, 8, devices=[0, 0])
    with pytest.raises(pkg.DSPError) as e:
        grp.random_walk([torch.zeros(1, dtype=torch.int32, device="cuda") for _ in range(2)], 3, 1)
    assert e.value.status == pkg.dsp.DSP_ERR_STATE
    grp.close()


@pytest.mark.slow
def test_random_walks_products(pkg, products):
    cfg, ip, ix = products
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, None, cfg.fanouts, 8)
    starts = np.arange(0, cfg.num_nodes, 13, dtype=np.int32)
    tr = s.random_walk(torch.from_numpy(starts).cuda(), 40, 77)
    s.sync()
    sel = np.arange(0, len(starts), 101)
    assert np.array_equal(tr.cpu().numpy()[sel], oracle.random_walk(ip, ix, starts[sel], 40, 77))
    s.close()


def test_set_option_validation(pkg, tiny):
    """dsp_set_option: unknown options and out-of-range values are
    DSP_ERR_INVALID_ARG; layout options after the layout exists are
    DSP_ERR_STATE (the relabel map and the exchange channels after
    dsp_reserve, the row layout after dsp_load_partition)."""
    cfg, ip, ix, feats = tiny
    d = pkg.dsp
    c = pkg.dsp_create(0, 1, 0)
    try:
        for opt, val in ((99, 1), (d.DSP_OPT_RELABEL_MAP, 4), (d.DSP_OPT_LANE_ROUNDS, 0), (d.DSP_OPT_LOADER_ROWS, 33),
                         (d.DSP_OPT_GATHER_REGLOADS, 2), (d.DSP_OPT_EXCHANGE_CHANNELS, 9), (d.DSP_OPT_SPLIT_ROWS, 2)):
            with pytest.raises(pkg.DSPError) as e:
                pkg.dsp_set_option(c, opt, val)
            assert e.value.status == d.DSP_ERR_INVALID_ARG, (opt, val)
        pkg.dsp_set_option(c, d.DSP_OPT_SPLIT_ROWS, 1)
        pkg.dsp_load_partition(c, datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.dim)
        with pytest.raises(pkg.DSPError) as e:
            pkg.dsp_set_option(c, d.DSP_OPT_SPLIT_ROWS, 0)
        assert e.value.status == d.DSP_ERR_STATE
        pkg.dsp_set_option(c, d.DSP_OPT_RELABEL_MAP, 2)
        pkg.dsp_reserve(c, 16, cfg.fanouts)
        for opt in (d.DSP_OPT_RELABEL_MAP, d.DSP_OPT_EXCHANGE_CHANNELS):
            with pytest.raises(pkg.DSPError) as e:
                pkg.dsp_set_option(c, opt, 1)
            assert e.value.status == d.DSP_ERR_STATE
        pkg.dsp_set_option(c, d.DSP_OPT_LANE_ROUNDS, 4)      # tuning knobs stay settable
        pkg.dsp_set_option(c, d.DSP_OPT_LOADER_ROWS, 16)
    finally:
        pkg.dsp_destroy(c)
