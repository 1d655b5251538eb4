"""GPU parity for layer-wise CSP (DSP_LAYERWISE; Eq. 2, Table 7;
DESIGN.md R28-R30) against oracle.sample_layerwise, bit-exact on every block
array: P = 1 and virtual P = 2 / 4 worlds (the degree lookups then read peer
indptr shards and the tasks go to the owners), layer sizes from 1 to the
8192 maximum, tasks with 32 < c_u < deg (the block-per-task Floyd kernel),
empty and ragged batches, the fused and pipelined steps, and Table 7's
configuration on the products-shaped graph."""
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


@pytest.fixture(scope="module")
def tiny():
    cfg = datagen.CONFIGS["tiny"]
    ip, ix = datagen.make_graph(cfg)
    feats = datagen.features(0, cfg.num_nodes, cfg.dim)
    return cfg, ip, ix, feats


def assert_blocks_equal(got, ref, where=""):
    assert len(got) == len(ref)
    for l, (b, r) in enumerate(zip(got, ref)):
        assert (b.num_dst, b.num_src, b.num_edges) == (r["num_dst"], r["num_src"], r["num_edges"]), \
            f"{where} layer {l}: {(b.num_dst, b.num_src, b.num_edges)} vs {(r['num_dst'], r['num_src'], r['num_edges'])}"
        for key in ("indptr", "indices", "src_ids"):
            g = getattr(b, key).cpu().numpy()
            if not np.array_equal(g, r[key]):
                bad = np.nonzero(g != r[key])[0][:5] if g.shape == r[key].shape else "shape"
                raise AssertionError(f"{where} layer {l} {key} differs at {bad}")


def _big_tasks(ip, seeds, n):
    """Frontier nodes of layer 0 whose expected draw count is in (32, deg)."""
    d = np.diff(ip)[seeds].astype(float)
    c = n * d / d.sum()
    return int(((c > 40) & (c < d * 0.9)).sum())


@pytest.mark.parametrize("sizes", [(200, 300), (1000, 1000), (1,), (8192,), (50, 50, 50), (3, 4000)])
def test_layerwise_tiny_p1(pkg, tiny, sizes):
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, sizes, 64, scheme="layer")
    rng = np.random.default_rng(len(sizes) * 7 + sizes[0])
    for step, B in enumerate((64, 64, 1, 17, 0, 63)):
        seeds = rng.choice(cfg.num_nodes, size=B, replace=False).astype(np.int32)
        blocks = s.sample(torch.from_numpy(seeds).cuda(), 500 + step)
        assert_blocks_equal(blocks, oracle.sample_layerwise(ip, ix, seeds, sizes, 500 + step), f"{sizes} B={B}")
    s.close()


def test_layerwise_big_tasks_exercised(pkg, tiny):
    """n = 1000 over 64 seeds: hub seeds get 32 < c < deg draws."""
    cfg, ip, ix, feats = tiny
    deg = np.diff(ip)
    hubs = np.argsort(-deg)[:8].astype(np.int32)
    seeds = np.concatenate([hubs, np.setdiff1d(np.arange(0, cfg.num_nodes, 181, dtype=np.int32), hubs)[:56]])
    assert _big_tasks(ip, seeds, 1000) > 0
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, (1000, 1000), 64, scheme="layer")
    for rng in range(5):
        blocks = s.sample(torch.from_numpy(seeds).cuda(), rng)
        assert_blocks_equal(blocks, oracle.sample_layerwise(ip, ix, seeds, (1000, 1000), rng), f"rng {rng}")
    s.close()


@pytest.mark.parametrize("P", [2, 4])
def test_layerwise_virtual_ranks(pkg, tiny, P):
    cfg, ip, ix, feats = tiny
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi]))
    sizes = (700, 1500)
    grp = pkg.LocalGroup(bnds, shards, sizes, 64, devices=[0] * P, scheme="layer")
    train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
    per_rank = [datagen.rank_seed_batches(train, bnds, r, 48, 0) for r in range(P)]
    for step in range(4):
        seeds = [per_rank[r][step] for r in range(P)]
        if step == 1:
            seeds[0] = seeds[0][:0]
        if step == 2:
            seeds[P - 1] = np.concatenate([seeds[P - 1][:5], per_rank[0][step][:3]])
        res = grp.sample([torch.from_numpy(np.ascontiguousarray(x)).cuda() for x in seeds], 0x1A + step)
        for r in range(P):
            assert_blocks_equal(res[r], oracle.sample_layerwise(ip, ix, seeds[r], sizes, 0x1A + step),
                                f"P={P} rank {r} step {step}")
            out = grp.samplers[r].gather(res[r][-1].src_ids)
            grp.samplers[r].sync()
            exp = oracle.gather(feats, res[r][-1].src_ids.cpu().numpy())
            assert np.array_equal(out.cpu().numpy().view(np.uint32), exp.view(np.uint32))
    grp.close()


def test_layerwise_fused_and_pipelined(pkg, tiny):
    cfg, ip, ix, feats = tiny
    sizes = (400, 800)
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, sizes, 64, n_slots=2, scheme="layer")
    train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
    batches = datagen.rank_seed_batches(train, datagen.bounds(cfg.num_nodes, 1), 0, 64, 0)
    blocks, feat = s.sample_gather(torch.from_numpy(batches[0]).cuda(), 3, slot=0)
    ref = oracle.sample_layerwise(ip, ix, batches[0], sizes, 3)
    assert_blocks_equal(blocks, ref)
    assert np.array_equal(feat.cpu().numpy().view(np.uint32), oracle.gather(feats, ref[-1]["src_ids"]).view(np.uint32))
    L = len(sizes)
    hs = torch.zeros((4, 3 * L), dtype=torch.int64).pin_memory()
    for j in range(4):
        s.sample_gather(torch.from_numpy(batches[1 + j]).cuda(), 10 + j, slot=j % 2, sizes_out=hs[j], pipelined=True)
    s.flush()
    s.sync()
    for j in (2, 3):
        ref = oracle.sample_layerwise(ip, ix, batches[1 + j], sizes, 10 + j)
        exp = [v for r in ref for v in (r["num_dst"], r["num_src"], r["num_edges"])]
        assert hs[j].tolist() == exp
        blocks = s.blocks(j % 2, sizes=hs[j].tolist())
        assert_blocks_equal(blocks, ref)
        got = s.feat_buffer(j % 2)[: blocks[-1].num_src].cpu().numpy()
        assert np.array_equal(got.view(np.uint32), oracle.gather(feats, ref[-1]["src_ids"]).view(np.uint32))
    s.close()


def test_layerwise_concurrent_streams(pkg, tiny):
    """world 1: pipelined layer-wise calls on 3 workspaces / streams at once
    (each persistent call keeps its exchange slots in its own workspace)."""
    cfg, ip, ix, feats = tiny
    sizes = (300, 500)
    K = 3
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, sizes, 64, scheme="layer", n_slots=2 * K,
                    n_workspaces=K)
    pkg.dsp_set_persistent_blocks(s.ctx, 16)
    rng = np.random.default_rng(3)
    n = 9
    seeds = [rng.choice(cfg.num_nodes, size=64, replace=False).astype(np.int32) for _ in range(n)]
    dev = [torch.from_numpy(x).cuda() for x in seeds]
    L = len(sizes)
    hs = torch.zeros((n, 3 * L), dtype=torch.int64).pin_memory()
    main = torch.cuda.current_stream()
    streams = [torch.cuda.Stream() for _ in range(K)]
    for st in streams:
        st.wait_stream(main)
    for i in range(n):
        s.sample_gather(dev[i], 40 + i, slot=i % (2 * K), sizes_out=hs[i], async_=True, pipelined=True, ws=i % K,
                        stream=streams[i % K])
    for st in streams:
        with torch.cuda.stream(st):
            s.flush()
    for st in streams:
        main.wait_stream(st)
    torch.cuda.synchronize()
    for i in range(n - 2 * K, n):
        ref = oracle.sample_layerwise(ip, ix, seeds[i], sizes, 40 + i)
        blocks = s.blocks(i % (2 * K), sizes=[int(x) for x in hs[i]])
        assert_blocks_equal(blocks, ref, f"concurrent {i}")
        feat = s.feat_buffer(i % (2 * K))[: blocks[-1].num_src]
        assert np.array_equal(feat.cpu().numpy().view(np.uint32), oracle.gather(feats, ref[-1]["src_ids"]).view(np.uint32))
    s.close()


def test_layerwise_errors(pkg, tiny):
    cfg, ip, ix, feats = tiny
    bn = datagen.bounds(cfg.num_nodes, 1)
    with pytest.raises(pkg.DSPError) as e:
        pkg.Sampler(bn, ip, ix, feats, (8193,), 8, scheme="layer")
    assert e.value.status == pkg.dsp.DSP_ERR_INVALID_ARG
    s = pkg.Sampler(bn, ip, ix, feats, (100, 100), 16, scheme="layer")
    with pytest.raises(pkg.DSPError) as e:
        s.sample(torch.tensor([5, 9, 5], dtype=torch.int32, device="cuda"), 1)
    assert e.value.status == pkg.dsp.DSP_ERR_DUPLICATE_SEED
    with pytest.raises(pkg.DSPError) as e:
        s.sample(torch.tensor([5, cfg.num_nodes], dtype=torch.int32, device="cuda"), 1)
    assert e.value.status == pkg.dsp.DSP_ERR_OUT_OF_RANGE
    with pytest.raises(pkg.DSPError) as e:
        s.sample(torch.tensor([5, 6], dtype=torch.int32, device="cuda"), 1, biased=True)
    assert e.value.status in (pkg.dsp.DSP_ERR_INVALID_ARG, pkg.dsp.DSP_ERR_STATE)
    seeds = np.array([1, 2, 3], np.int32)
    assert_blocks_equal(s.sample(torch.from_numpy(seeds).cuda(), 4), oracle.sample_layerwise(ip, ix, seeds, (100, 100), 4))
    # a workspace shared with node-wise calls keeps both correct (one relabel map, one epoch)
    n = pkg.Sampler(bn, ip, ix, feats, (5, 5), 16)
    s.close()
    n.close()


@pytest.mark.slow
def test_layerwise_products_table7(pkg):
    """Table 7: batch 1024, layer size 1000 for both layers."""
    cfg = datagen.CONFIGS["products"]
    ip, ix = datagen.make_graph(cfg)
    feats = datagen.features(0, cfg.num_nodes, cfg.dim)
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, (1000, 1000), cfg.batch, scheme="layer")
    train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
    batches = datagen.rank_seed_batches(train, datagen.bounds(cfg.num_nodes, 1), 0, cfg.batch, 0)
    for step in (0, 1, 7):
        blocks = s.sample(torch.from_numpy(batches[step]).cuda(), 90 + step)
        assert_blocks_equal(blocks, oracle.sample_layerwise(ip, ix, batches[step], (1000, 1000), 90 + step))
    s.close()
