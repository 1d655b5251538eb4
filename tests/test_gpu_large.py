"""Parity at BASELINE.json's two largest configurations (papers- and
Friendster-shaped, configs[3] and [4]) on one B200: the whole graph at P = 1,
and the 8-GPU partitioning as 8 virtual ranks sharing the device
(dsp_sample_group: the same kernels, exchange flags and peer writes as 8 GPUs).
Whole 1024-seed batches are compared bit-exactly with the oracle on the full
CSR; gathered rows against the closed-form feature recipe.

Host graph generation takes a few minutes at this size (about 220 s for both
configs on the GPU box, inside the -m gpu suite's budget); the cases run in
every `pytest -m gpu`.  They cover int64 row offsets (papers and Friendster at
P = 1 have nnz > 2^31), the hashed relabel map at N = 111M and 66M, and the
8-rank exchange of the BASELINE configs[3] / configs[4] partitioning."""
import numpy as np
import pytest

import datagen
import oracle

torch = pytest.importorskip("torch")
pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.fixture(scope="module")
def pkg():
    import paper_conf_ppopp_caiz0zszck23_b200 as p
    torch.cuda.set_device(0)
    return p


def assert_blocks_equal(got, ref, where):
    for l, (b, r) in enumerate(zip(got, ref)):
        assert (b.num_dst, b.num_src, b.num_edges) == (r["num_dst"], r["num_src"], r["num_edges"]), (where, l)
        for key in ("indptr", "indices", "src_ids"):
            assert np.array_equal(getattr(b, key).cpu().numpy(), r[key]), (where, l, key)


def check_rows(out, ids, dim, n_check=20000):
    sel = np.linspace(0, len(ids) - 1, min(n_check, len(ids))).astype(np.int64)
    exp = datagen.features_of(ids[sel], dim)
    assert np.array_equal(out[sel].view(np.uint32), exp.view(np.uint32))


@pytest.mark.parametrize("name", ["papers", "friendster"])
def test_large_config(pkg, name):
    cfg = datagen.CONFIGS[name]
    ip, ix = datagen.make_graph(cfg)
    assert int(ip[-1]) > 2**31      # int64 row offsets are exercised at P = 1
    train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
    # ---- P = 1: the whole graph on one GPU
    bnds = datagen.bounds(cfg.num_nodes, 1)
    feats = datagen.features(0, cfg.num_nodes, cfg.dim)
    s = pkg.Sampler(bnds, ip, ix, feats, cfg.fanouts, cfg.batch, n_slots=2)
    del feats
    batches = datagen.rank_seed_batches(train, bnds, 0, cfg.batch, 0)
    for step in (0, 1):
        blocks, feat = s.sample_gather(torch.from_numpy(batches[step]).cuda(), 11 + step, slot=step)
        ref = oracle.sample(ip, ix, batches[step], cfg.fanouts, 11 + step)
        assert_blocks_equal(blocks, ref, f"{name} P=1 step {step}")
        check_rows(feat.cpu().numpy(), ref[-1]["src_ids"], cfg.dim)
    s.close()
    torch.cuda.empty_cache()
    # ---- P = 8 virtual ranks (the BASELINE 8-GPU partitioning)
    P = 8
    bnds = datagen.bounds(cfg.num_nodes, P)
    shards = []
    for r in range(P):
        lo, hi = int(bnds[r]), int(bnds[r + 1])
        sip, six = datagen.shard(ip, ix, lo, hi)
        shards.append((sip, six, datagen.features(lo, hi, cfg.dim)))
    grp = pkg.LocalGroup(bnds, shards, cfg.fanouts, cfg.batch, devices=[0] * P)
    del shards
    seeds = [datagen.rank_seed_batches(train, bnds, r, cfg.batch, 0)[0] for r in range(P)]
    res = grp.sample([torch.from_numpy(x).cuda() for x in seeds], 0x5EED)
    for r in (0, 3, 7):
        ref = oracle.sample(ip, ix, seeds[r], cfg.fanouts, 0x5EED)
        assert_blocks_equal(res[r], ref, f"{name} P=8 rank {r}")
        out = grp.samplers[r].gather(res[r][-1].src_ids)
        grp.samplers[r].sync()
        check_rows(out.cpu().numpy(), ref[-1]["src_ids"], cfg.dim)
    grp.close()
