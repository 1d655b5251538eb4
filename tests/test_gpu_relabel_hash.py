"""GPU parity under each layout of the relabel map, forced with
dsp_set_option(DSP_OPT_RELABEL_MAP) on
graphs the oracle checks quickly: the batch-sized hash table (the default for
graphs of more than 3M nodes -- papers / Friendster -- where a direct map over
all N ids cannot stay in L2), the compact 4-byte direct map (the default
below that) and the 8-byte epoch-word direct map.  The layout only changes
where the relabel words live, so every block must stay bit-identical to the
oracle: P = 1 (persistent kernel, plain / fused / pipelined), virtual ranks
(one persistent kernel per rank), biased sampling, duplicate-seed
detection, and enough calls on one workspace to cross the 255-epoch windows
that zero the hash table and the compact map."""
import numpy as np
import pytest

import datagen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pkg():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device (run under gpurun)")
    import paper_conf_ppopp_caiz0zszck23_b200 as p
    from paper_conf_ppopp_caiz0zszck23_b200 import _build
    _build.build()
    torch.cuda.set_device(0)
    return p


@pytest.fixture(params=["hash", "direct", "direct64"])
def hashed(request, pkg):
    """Sampler / LocalGroup options selecting the relabel-map layout."""
    return {pkg.dsp.DSP_OPT_RELABEL_MAP: pkg.dsp.RELABEL_MAPS[request.param]}


@pytest.fixture(scope="module")
def tiny():
    cfg = datagen.CONFIGS["tiny"]
    ip, ix = datagen.make_graph(cfg)
    return cfg, ip, ix, datagen.features(0, cfg.num_nodes, cfg.dim)


def blocks_equal(got, ref, where):
    for l, (b, r) in enumerate(zip(got, ref)):
        assert (b.num_dst, b.num_src, b.num_edges) == (r["num_dst"], r["num_src"], r["num_edges"]), (where, l)
        for key in ("indptr", "indices", "src_ids"):
            assert np.array_equal(getattr(b, key).cpu().numpy(), r[key]), (where, l, key)


def batches_of(cfg, P, r, batch=None):
    train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
    return datagen.rank_seed_batches(train, datagen.bounds(cfg.num_nodes, P), r, batch or cfg.batch, 0)


def test_hash_tiny_every_batch_and_tag_wrap(pkg, tiny, hashed):
    """> 85 three-layer calls on one workspace: the epoch passes 255 at least
    once, so the table is zeroed mid-run and tags are reused afterwards."""
    cfg, ip, ix, feats = tiny
    fan = (15, 10, 5)
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, fan, cfg.batch, options=hashed)
    batches = batches_of(cfg, 1, 0)
    assert 3 * len(batches) > 255
    for step, seeds in enumerate(batches):
        blocks = s.sample(torch.from_numpy(seeds).cuda(), 900 + step)
        blocks_equal(blocks, oracle.sample(ip, ix, seeds, fan, 900 + step), f"hash step {step}")
    s.close()


def test_hash_fused_and_pipelined(pkg, tiny, hashed):
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2, options=hashed)
    batches = batches_of(cfg, 1, 0)
    blocks, feat = s.sample_gather(torch.from_numpy(batches[0]).cuda(), 5, slot=0)
    ref = oracle.sample(ip, ix, batches[0], cfg.fanouts, 5)
    blocks_equal(blocks, ref, "fused")
    assert np.array_equal(feat.cpu().numpy().view(np.uint32), oracle.gather(feats, ref[-1]["src_ids"]).view(np.uint32))
    L = len(cfg.fanouts)
    sizes = torch.zeros((6, 3 * L), dtype=torch.int64).pin_memory()
    for j in range(6):
        s.sample_gather(torch.from_numpy(batches[j]).cuda(), 40 + j, slot=j % 2, sizes_out=sizes[j], pipelined=True)
    s.flush()
    s.sync()
    for j in (4, 5):
        blocks = s.blocks(j % 2, sizes=[int(x) for x in sizes[j]])
        ref = oracle.sample(ip, ix, batches[j], cfg.fanouts, 40 + j)
        blocks_equal(blocks, ref, f"pipelined {j}")
        feat = s.feat_buffer(j % 2)[: blocks[-1].num_src]
        assert np.array_equal(feat.cpu().numpy().view(np.uint32),
                              oracle.gather(feats, ref[-1]["src_ids"]).view(np.uint32))
    s.close()


def test_hash_duplicate_seed(pkg, tiny, hashed):
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, 64, options=hashed)
    for dup in ([5, 9, 5], list(range(40)) + [17]):
        with pytest.raises(pkg.DSPError) as e:
            s.sample(torch.tensor(dup, dtype=torch.int32, device="cuda"), 1)
        assert e.value.status == pkg.dsp.DSP_ERR_DUPLICATE_SEED
    seeds = np.arange(0, 640, 10, dtype=np.int32)
    blocks_equal(s.sample(torch.from_numpy(seeds).cuda(), 3), oracle.sample(ip, ix, seeds, cfg.fanouts, 3), "after")
    s.close()


@pytest.mark.parametrize("P", [2, 4])
def test_hash_virtual_ranks(pkg, tiny, hashed, P):
    cfg, ip, ix, feats = tiny
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi]))
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, 32, devices=[0] * P, options=hashed)
    train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
    per_rank = [np.concatenate([datagen.rank_seed_batches(train, bnds, r, 32, e) for e in (0, 1)])
                for r in range(P)]
    assert min(len(x) for x in per_rank) >= 90
    for step in range(90):   # crosses the tag wrap
        seeds = [per_rank[r][step] for r in range(P)]
        res = grp.sample([torch.from_numpy(np.ascontiguousarray(x)).cuda() for x in seeds], 0x77 + step)
        if step % 15 == 0 or step > 80:
            for r in range(P):
                blocks_equal(res[r], oracle.sample(ip, ix, seeds[r], cfg.fanouts, 0x77 + step), (P, r, step))
    grp.close()


def test_hash_biased(pkg, tiny, hashed):
    cfg, ip, ix, feats = tiny
    w = datagen.edge_weights(ix, datagen.node_weights(cfg.num_nodes))
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, cfg.batch, edge_weights=w, options=hashed)
    batches = batches_of(cfg, 1, 0)
    for step in range(4):
        blocks = s.sample(torch.from_numpy(batches[step]).cuda(), 60 + step, biased=True)
        blocks_equal(blocks, oracle.sample(ip, ix, batches[step], cfg.fanouts, 60 + step, weights=w), "biased")
    s.close()


@pytest.mark.slow
def test_hash_products(pkg, hashed):
    cfg = datagen.CONFIGS["products"]
    ip, ix = datagen.make_graph(cfg)
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, None, cfg.fanouts, cfg.batch, options=hashed)
    batches = batches_of(cfg, 1, 0)
    for step in (0, 1):
        blocks = s.sample(torch.from_numpy(batches[step]).cuda(), 5 + step)
        blocks_equal(blocks, oracle.sample(ip, ix, batches[step], cfg.fanouts, 5 + step), f"products {step}")
    s.close()
