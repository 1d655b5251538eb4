"""GPU parity for the cold-feature tier ("we cache as many hot
nodes as possible in GPU memory and store the other nodes (called cold nodes)
in CPU memory and access them using the UVA technique"; P:L224 feature
position list).  Whatever the hot/cold split, the gathered rows must be
bit-identical to the oracle gather of the whole feature matrix: all rows hot,
none hot, a degree-ranked fraction hot; through the standalone gather, the
fused sample+gather step, the pipelined step (loader warps) and virtual
multi-rank worlds where cold rows of a peer live in that peer's host memory."""
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


def _bits(x):
    return np.ascontiguousarray(x).view(np.uint32)


def _seeds(cfg, P, r, batch):
    train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
    return datagen.rank_seed_batches(train, datagen.bounds(cfg.num_nodes, P), r, batch, 0)


@pytest.mark.parametrize("hot,regloads", [(0, 0), (1, 0), (3000, 0), (10_000, 0), (-1, 0), (0, 1), (3000, 1)])
def test_tiered_gather_p1(pkg, tiny, hot, regloads):
    """regloads = 0: the gathers bulk-copy (TMA) cold rows straight from host
    memory; 1: register loads (DSP_OPT_GATHER_REGLOADS = 1)."""
    cfg, ip, ix, feats = tiny
    s = pkg.Sampler(datagen.bounds(cfg.num_nodes, 1), ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2,
                    hot_rows=hot, options={pkg.dsp.DSP_OPT_GATHER_REGLOADS: regloads})
    # standalone gather over ids covering every row, in a scrambled order with repeats
    rng = np.random.default_rng(hot & 0xFFFF)
    ids = np.concatenate([rng.permutation(cfg.num_nodes), rng.integers(0, cfg.num_nodes, 777)]).astype(np.int32)
    out = s.gather(torch.from_numpy(ids).cuda())
    s.sync()
    assert np.array_equal(_bits(out.cpu().numpy()), _bits(oracle.gather(feats, ids)))
    # fused step and pipelined steps (the loader warps read cold rows too)
    batches = _seeds(cfg, 1, 0, cfg.batch)
    blocks, feat = s.sample_gather(torch.from_numpy(batches[0]).cuda(), 11, slot=0)
    ref = oracle.sample(ip, ix, batches[0], cfg.fanouts, 11)
    assert np.array_equal(blocks[-1].src_ids.cpu().numpy(), ref[-1]["src_ids"])
    assert np.array_equal(_bits(feat.cpu().numpy()), _bits(oracle.gather(feats, ref[-1]["src_ids"])))
    L = len(cfg.fanouts)
    sizes = torch.zeros((4, 3 * L), dtype=torch.int64).pin_memory()
    for j in range(4):
        s.sample_gather(torch.from_numpy(batches[1 + j]).cuda(), 60 + j, slot=j % 2, sizes_out=sizes[j],
                        pipelined=True)
    s.flush()
    s.sync()
    for j in (2, 3):
        ref = oracle.sample(ip, ix, batches[1 + j], cfg.fanouts, 60 + j)
        n = int(sizes[j][3 * L - 2])
        assert n == ref[-1]["num_src"]
        got = s.feat_buffer(j % 2)[:n].cpu().numpy()
        assert np.array_equal(_bits(got), _bits(oracle.gather(feats, ref[-1]["src_ids"])))
    s.close()


@pytest.mark.parametrize("P", [2, 4])
def test_tiered_virtual_ranks(pkg, tiny, P):
    """Cold rows of rank o live in rank o's pinned host memory; a requester
    gathers them over UVA like its peers' hot rows over peer memory."""
    cfg, ip, ix, feats = tiny
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi]))
    hot = [(hi - lo) * f // 4 for f, (lo, hi) in zip([0, 1, 2, 3, 4, 1, 2, 3],
                                                      zip(bnds[:-1].tolist(), bnds[1:].tolist()))][:P]
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, 32, devices=[0] * P, hot_rows=hot)
    per_rank = [_seeds(cfg, P, r, 32) for r in range(P)]
    for step in range(3):
        seeds = [per_rank[r][step] for r in range(P)]
        res = grp.sample([torch.from_numpy(np.ascontiguousarray(x)).cuda() for x in seeds], 0x77 + step)
        for r in range(P):
            ref = oracle.sample(ip, ix, seeds[r], cfg.fanouts, 0x77 + step)
            assert np.array_equal(res[r][-1].src_ids.cpu().numpy(), ref[-1]["src_ids"])
            out = grp.samplers[r].gather(res[r][-1].src_ids)
            grp.samplers[r].sync()
            assert np.array_equal(_bits(out.cpu().numpy()), _bits(oracle.gather(feats, ref[-1]["src_ids"])))
    grp.close()


def test_tiered_errors(pkg, tiny):
    cfg, ip, ix, feats = tiny
    bn = datagen.bounds(cfg.num_nodes, 1)
    s = pkg.Sampler(bn, ip, ix, feats, cfg.fanouts, 16)
    with pytest.raises(pkg.DSPError) as e:            # features already resident
        pkg.dsp_load_features_tiered(s.ctx, feats, cfg.dim, 10)
    assert e.value.status == pkg.dsp.DSP_ERR_STATE
    s.close()


@pytest.mark.parametrize("dim", [100, 36, 128, 8])
@pytest.mark.parametrize("P,hot", [(1, None), (1, 3), (2, None), (2, 2)])
def test_split_rows_layout(pkg, tiny, dim, P, hot):
    """DSP_OPT_SPLIT_ROWS = 1: rows stored as a 128-byte-line head plus a tail
    (dim 100: 384 + 16 B, 36: 128 + 16, 128: head only, 8: tail only), in the
    HBM shard, in the cold region and across virtual ranks; every gather path
    (standalone, fused, pipelined loader warps) returns the rows bit-exactly."""
    cfg, ip, ix, _ = tiny
    feats = datagen.features(0, cfg.num_nodes, dim)
    bnds = datagen.bounds(cfg.num_nodes, P)
    opts = {pkg.dsp.DSP_OPT_SPLIT_ROWS: 1}
    ids = np.random.default_rng(dim + P).permutation(cfg.num_nodes).astype(np.int32)
    if P == 1:
        s = pkg.Sampler(bnds, ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2, options=opts,
                        hot_rows=None if hot is None else cfg.num_nodes * hot // 4)
        out = s.gather(torch.from_numpy(ids).cuda())
        s.sync()
        assert np.array_equal(_bits(out.cpu().numpy()), _bits(oracle.gather(feats, ids)))
        batches = _seeds(cfg, 1, 0, cfg.batch)
        blocks, feat = s.sample_gather(torch.from_numpy(batches[0]).cuda(), 21, slot=0)
        ref = oracle.sample(ip, ix, batches[0], cfg.fanouts, 21)
        assert np.array_equal(_bits(feat.cpu().numpy()), _bits(oracle.gather(feats, ref[-1]["src_ids"])))
        L = len(cfg.fanouts)
        sizes = torch.zeros((3, 3 * L), dtype=torch.int64).pin_memory()
        for j in range(3):
            s.sample_gather(torch.from_numpy(batches[1 + j]).cuda(), 30 + j, slot=j % 2, sizes_out=sizes[j],
                            pipelined=True)
            if j >= 1:
                torch.cuda.synchronize()
                ref = oracle.sample(ip, ix, batches[j], cfg.fanouts, 30 + j - 1)
                got = s.feat_buffer((j - 1) % 2)[: int(sizes[j - 1][3 * (L - 1) + 1])]
                assert np.array_equal(_bits(got.cpu().numpy()), _bits(oracle.gather(feats, ref[-1]["src_ids"])))
        s.flush()
        s.sync()
        s.close()
        return
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, feats[lo:hi]))
    hr = None if hot is None else [(int(bnds[r + 1]) - int(bnds[r])) * hot // 4 for r in range(P)]
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, 32, devices=[0] * P, hot_rows=hr, options=opts)
    for r in range(P):
        out = grp.samplers[r].gather(torch.from_numpy(ids).cuda())
        grp.samplers[r].sync()
        assert np.array_equal(_bits(out.cpu().numpy()), _bits(oracle.gather(feats, ids)))
    grp.close()
