"""Pins for the oracle's layer-wise sampling (Sec. 4.2, Eq. 2;
Table 7 "layer-wise sampling without replacement"; R28-R30).

Eq. 2 allocation: n draws with replacement over the frontier, node u with
probability W_u / sum W (W_u = deg u), c_u = times u was drawn.  Pinned by the
exact multinomial law (scipy), the draw -> interval map read off the top bits
of the Philox word when T is a power of two, the paper's equivalence with
drawing n edges from the concatenated adjacency lists, and special cases.
Per-node sampling with c_u > 32 (Floyd beyond a warp): exact subset
uniformity.  Whole layer-wise samples: structural invariants and CSP-replay
invariance across rank counts."""
import itertools
import json
import os
from collections import Counter

import numpy as np
import pytest
from scipy.stats import chisquare, multinomial

import datagen
import oracle
from csp_replay import replay_layerwise_inprocess

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
TAG_L = 0x4453504C   # "DSPL"


def test_alloc_special_cases():
    assert oracle.layer_alloc(1, 0, 0, [0, 0, 0], 10).tolist() == [0, 0, 0]      # T = 0: nothing to sample
    assert oracle.layer_alloc(1, 0, 0, [], 10).tolist() == []
    for s in range(20):
        assert oracle.layer_alloc(s, 3, 1, [0, 0, 7, 0], 13).tolist() == [0, 0, 13, 0]
        c = oracle.layer_alloc(s, 3, 1, [4, 0, 9, 1, 0, 2], 50)
        assert c.sum() == 50 and c[1] == 0 and c[4] == 0


def test_alloc_draw_interval_from_top_bits():
    """T = 4 with unit weights: r = floor(word * 4 / 2^64) is the word's top 2
    bits, so draw j lands on frontier index word_j >> 62."""
    for s in range(200):
        word = oracle.draw_word_tag(s, 0, 77, 2, TAG_L)
        c = oracle.layer_alloc(s, 77, 2, [1, 1, 1, 1], 1)
        assert c.tolist() == [int(i == word >> 62) for i in range(4)]
    # W = [2, 0, 1, 1] (T = 4): index 0 takes top bits 0b00 and 0b01, index 2 0b10, index 3 0b11
    for s in range(200):
        words = [oracle.draw_word_tag(s, j, 5, 0, TAG_L) >> 62 for j in range(3)]
        exp = [sum(w in (0, 1) for w in words), 0, sum(w == 2 for w in words), sum(w == 3 for w in words)]
        assert oracle.layer_alloc(s, 5, 0, [2, 0, 1, 1], 3).tolist() == exp


@pytest.mark.parametrize("W,n", [([1, 2], 2), ([3, 1, 2], 3), ([5, 0, 2, 1], 4)])
def test_alloc_is_exact_multinomial(W, n):
    T = sum(W)
    p = [w / T for w in W]
    trials = 30_000
    got = Counter(tuple(oracle.layer_alloc(s, 11, 0, W, n).tolist()) for s in range(trials))
    outcomes = [c for c in itertools.product(range(n + 1), repeat=len(W)) if sum(c) == n
                and all(ci == 0 for ci, w in zip(c, W) if w == 0)]
    assert set(got) <= set(outcomes)
    obs = np.array([got[c] for c in outcomes], float)
    exp = np.array([multinomial.pmf(c, n, p) * trials for c in outcomes])
    assert abs(exp.sum() - trials) < 1e-6 * trials
    assert chisquare(obs, exp).pvalue > 1e-4


def test_alloc_equals_sampling_from_concatenated_lists():
    """'equivalent to fetching the adjacency lists of the frontier
    nodes and then conducting sampling': drawing n edges uniformly with
    replacement from the concatenated lists gives c ~ Multinomial(n, d/T);
    compare mean and variance of every c_i against numpy draws of that."""
    d = np.array([1, 7, 3, 12, 5, 2], np.uint64)
    n, trials = 40, 20_000
    ours = np.array([oracle.layer_alloc(s, 2, 1, d, n) for s in range(trials)], float)
    owner = np.repeat(np.arange(len(d)), d.astype(np.int64))
    rng = np.random.default_rng(0)
    ref = np.stack([np.bincount(owner[rng.integers(0, len(owner), n)], minlength=len(d)) for _ in range(trials)])
    p = d / d.sum()
    assert np.allclose(ours.mean(0), n * p, atol=0.06 * np.sqrt(n))
    assert np.allclose(ours.mean(0), ref.mean(0), atol=0.08 * np.sqrt(n))
    assert np.allclose(ours.var(0), n * p * (1 - p), rtol=0.06, atol=0.05)


def test_large_fanout_floyd_uniform():
    """c_u > 32 (beyond one warp): d = 36, k = 34 leaves out a uniformly random
    pair; d = 100, k = 40 includes every position with probability 0.4."""
    pairs = Counter()
    n = 25_000
    for v in range(n):
        pos = oracle.node_positions(9, v, 1, 36, 34)
        assert len(pos) == 34 and np.all(np.diff(pos) > 0)
        pairs[tuple(sorted(set(range(36)) - set(pos.tolist())))] += 1
    assert len(pairs) == 630
    assert chisquare(np.array(list(pairs.values()), float), np.full(630, n / 630)).pvalue > 1e-4
    incl = np.zeros(100)
    for v in range(4000):
        incl[oracle.node_positions(3, v, 0, 100, 40)] += 1
    assert chisquare(incl, np.full(100, 4000 * 0.4)).pvalue > 1e-4


def _rows(ip, ix, v):
    return ix[ip[v]:ip[v + 1]]


def test_layerwise_blocks_invariants(tiny_graph):
    ip, ix = tiny_graph
    deg = np.diff(ip)
    seeds = np.arange(0, 10_000, 97, dtype=np.int32)
    sizes = [200, 300, 50]
    blocks = oracle.sample_layerwise(ip, ix, seeds, sizes, 5)
    frontier = seeds
    for b, n in zip(blocks, sizes):
        assert b["num_dst"] == len(frontier) and np.array_equal(b["src_ids"][:b["num_dst"]], frontier)
        assert b["num_edges"] <= n
        src = b["src_ids"]
        for i, v in enumerate(frontier):
            got = src[b["indices"][b["indptr"][i]:b["indptr"][i + 1]]]
            row = _rows(ip, ix, v)
            pos = np.searchsorted(row, got)
            assert np.all(row[np.minimum(pos, len(row) - 1)] == got) and np.all(np.diff(pos) > 0)
            assert len(got) <= deg[v]
        # new nodes in first-occurrence order, each once
        assert len(set(src.tolist())) == len(src)
        frontier = src
    again = oracle.sample_layerwise(ip, ix, seeds, sizes, 5)
    assert all(np.array_equal(x["indices"], y["indices"]) for x, y in zip(blocks, again))


def test_layerwise_dense_rows_take_exactly_n():
    """Every frontier node with degree >= n: the layer has exactly n edges."""
    N = 64
    rows = [[u for u in range(N) if u != v] for v in range(N)]
    ip = np.concatenate([[0], np.cumsum([len(r) for r in rows])]).astype(np.int64)
    ix = np.concatenate(rows).astype(np.int32)
    for s in range(10):
        b = oracle.sample_layerwise(ip, ix, np.array([3, 9, 40], np.int32), [60], s)[0]
        assert b["num_edges"] == 60


def _fig3_csr():
    """The Fig. 3 graph of tests/golden/fig3_worked_example.json (P:L81,
    P:L146): node v's in-neighbour row is rows[str(v)], empty when absent."""
    g = json.load(open(os.path.join(GOLDEN, "fig3_worked_example.json")))
    n = g["num_nodes"]
    ip = np.zeros(n + 1, np.int64)
    cols = []
    for v in range(n):
        r = sorted(g["rows"].get(str(v), []))
        cols.extend(r)
        ip[v + 1] = ip[v] + len(r)
    return g, ip, np.array(cols, np.int32)


def test_fig3_layerwise_fanout_two():
    """P:L102 (layer-wise: 'the total number of sampled nodes' per layer is
    the fan-out) on the Fig. 3 graph A:[C,E], C:[B,K], E:[G,H] (P:L81,
    P:L146) with layer sizes [2, 2] (R28).

    Layer 0: the frontier is {A} alone, so both Eq. 2 draws pick A (c_A = 2 =
    deg A) and A's whole row is taken: block 0 equals the node-wise Fig. 3
    block (indptr [0,2], src_ids [A,C,E]) for every rng_seed.
    Layer 1: frontier [A,C,E] with W = deg = [2,2,2]; (c_A,c_C,c_E) ~
    Multinomial(2, 1/3 each) and u takes min(c_u, 2) of its 2 neighbours
    without replacement, so there are exactly 2 edges, each drawn from the row
    of its dst, and the edge set has the closed-form law: {both neighbours of
    u} with probability 1/9 for each u, {one neighbour of u, one of w} with
    probability (2/9)(1/2)(1/2) = 1/18 for each pair u < w and each of the 4
    neighbour choices (3 * 1/9 + 12 * 1/18 = 1)."""
    g, ip, ix = _fig3_csr()
    assert ip.tolist() == [0, 2, 2, 4, 6, 6, 6, 6] and ix.tolist() == [2, 3, 1, 6, 4, 5]
    A, B, C, E, G, H, K = range(7)
    row = {A: (C, E), C: (B, K), E: (G, H)}
    law = {}
    for u in (A, C, E):
        law[frozenset({(u, row[u][0]), (u, row[u][1])})] = 1 / 9
    for u, w in ((A, C), (A, E), (C, E)):
        for x in row[u]:
            for y in row[w]:
                law[frozenset({(u, x), (w, y)})] = 1 / 18
    assert abs(sum(law.values()) - 1) < 1e-12 and len(law) == 15
    trials = 6000
    seen = Counter()
    for s in range(trials):
        b0, b1 = oracle.sample_layerwise(ip, ix, g["seeds"], [2, 2], s)
        exp0 = g["blocks"][0]
        for key in ("indptr", "indices", "src_ids"):
            assert b0[key].tolist() == exp0[key], (s, key)
        assert (b1["num_dst"], b1["num_edges"]) == (3, 2), s
        assert b1["src_ids"][:3].tolist() == [A, C, E]
        assert b1["indptr"][0] == 0 and b1["indptr"][3] == 2 and np.all(np.diff(b1["indptr"]) >= 0)
        pairs = set()
        for i, u in enumerate((A, C, E)):
            for e in range(b1["indptr"][i], b1["indptr"][i + 1]):
                w = int(b1["src_ids"][b1["indices"][e]])
                assert w in row[u], (s, u, w)
                pairs.add((u, w))
        assert len(pairs) == 2
        seen[frozenset(pairs)] += 1
    assert set(seen) <= set(law)
    keys = sorted(law, key=lambda k: sorted(k))
    obs = np.array([seen[k] for k in keys], float)
    exp = np.array([law[k] * trials for k in keys])
    assert chisquare(obs, exp).pvalue > 1e-4


@pytest.mark.parametrize("P", [2, 3, 4])
def test_layerwise_csp_replay_equals_single_device(tiny_graph, P):
    ip, ix = tiny_graph
    bnds = datagen.bounds(10_000, P)
    seeds = [np.arange(int(bnds[r]) + 5, int(bnds[r + 1]), 173, dtype=np.int32) for r in range(P)]
    seeds[-1] = np.concatenate([seeds[-1], seeds[0][:4]])        # remote seeds too
    sizes = [120, 400]
    rep = replay_layerwise_inprocess(ip, ix, bnds, seeds, sizes, 31)
    for r in range(P):
        ref = oracle.sample_layerwise(ip, ix, seeds[r], sizes, 31)
        for b, e in zip(rep[r], ref):
            for key in ("indptr", "indices", "src_ids"):
                assert np.array_equal(b[key], e[key])
