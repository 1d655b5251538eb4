"""Pins for the oracle's biased node-wise sampling (Sec. 4.2; DESIGN.md
R24-R26): the fixed-point weight conversion, the exact successive-sampling
distribution (computed in closed form here with fractions), the paper's
first-pick probability w_u / sum w, zero weights, and CSP-replay invariance."""
import itertools
import math
from collections import Counter
from fractions import Fraction

import numpy as np
import pytest
from scipy.stats import chisquare

import datagen
import oracle
from csp_replay import replay_inprocess


def test_weight_fixed_point_is_exact_floor():
    rng = np.random.default_rng(1)
    ws = np.concatenate([rng.uniform(0, 65535.99, 2000).astype(np.float32),
                         np.float32([0.0, 1.0, 0.5, 1 / 65536, 65535.0, 3.14159, 1e-8])])
    for w in ws:
        exp = math.floor(Fraction(float(w)) * 65536)        # exact rational floor (library routine)
        assert oracle.weight_fixed(float(w)) == exp
    for bad in (-1.0, 65536.0, float("nan"), float("inf")):
        assert oracle.weight_fixed(bad) == 0xFFFFFFFF


def exact_subset_probs(a, k):
    """Successive sampling without replacement, probabilities by enumeration of orders."""
    idx = [p for p in range(len(a)) if a[p] > 0]
    probs = Counter()
    for order in itertools.permutations(idx, k):
        pr = Fraction(1)
        remaining = sum(a[p] for p in idx)
        for p in order:
            pr *= Fraction(a[p], remaining)
            remaining -= a[p]
        probs[tuple(sorted(order))] += pr
    return probs


@pytest.mark.parametrize("a,k", [([1, 2, 3, 0, 4], 2), ([5, 1, 1, 1, 7, 2], 3), ([65536, 1, 300000, 12], 2)])
def test_successive_sampling_distribution(a, k):
    exact = exact_subset_probs(a, k)
    assert sum(exact.values()) == 1
    n = 40_000
    c = Counter(tuple(oracle.node_positions_biased(s, 9, 1, a, k).tolist()) for s in range(n))
    assert set(c) <= set(exact)
    keys = sorted(exact)
    obs = np.array([c[key] for key in keys], float)
    exp = np.array([float(exact[key]) * n for key in keys])
    assert chisquare(obs, exp).pvalue > 1e-4


def test_first_pick_is_the_papers_probability():
    """neighbour u is sampled with probability w_u / sum w (the first draw)."""
    a = [3, 0, 1, 6, 2, 8]
    n = 40_000
    c = Counter(int(oracle.biased_picks(s, 4, 0, a, 3)[0]) for s in range(n))
    assert c[1] == 0
    idx = [p for p in range(len(a)) if a[p]]
    obs = np.array([c[p] for p in idx], float)
    exp = np.array([a[p] / sum(a) * n for p in idx])
    assert chisquare(obs, exp).pvalue > 1e-4


def test_zero_weights_and_few_candidates():
    assert oracle.node_positions_biased(1, 2, 0, [0, 0, 0], 2).tolist() == []
    for s in range(50):   # <= k positive weights: all of them, no draw
        assert oracle.node_positions_biased(s, 2, 0, [0, 5, 0, 1, 0], 2).tolist() == [1, 3]
        assert oracle.node_positions_biased(s, 2, 0, [0, 5, 0, 1, 0], 7).tolist() == [1, 3]
    for s in range(200):
        pos = oracle.node_positions_biased(s, 3, 1, [4, 0, 4, 4, 0, 4], 3)
        assert 1 not in pos and 4 not in pos and len(pos) == 3


def test_equal_weights_give_uniform_subsets():
    n = 30_000
    c = Counter(tuple(oracle.node_positions_biased(s, 77, 1, [7] * 6, 3).tolist()) for s in range(n))
    assert len(c) == 20
    assert chisquare(np.array(list(c.values()), float), np.full(20, n / 20)).pvalue > 1e-4


def test_biased_key_layout():
    """Counter {t, v, l, 'DSPB'}: a distinct stream from the uniform sampler."""
    x = oracle.philox4x32_10([2, 7, 1, 0x44535042], [99, 0])
    w = (int(x[1]) << 32) | int(x[0])
    assert w != oracle.draw_word(99, 2, 7, 1)
    # single positive weight among many: always that one, whatever the word
    for s in range(20):
        assert oracle.biased_picks(s, 7, 1, [0] * 10 + [3] + [0] * 5, 1).tolist() == [10]


def _weights_for(indices):
    w = datagen.node_weights(10_000)
    return datagen.edge_weights(indices, w)


def test_biased_blocks_invariants(tiny_graph):
    ip, ix = tiny_graph
    ew = _weights_for(ix)
    seeds = np.arange(0, 10_000, 157, dtype=np.int32)
    blocks = oracle.sample(ip, ix, seeds, [5, 5], 21, weights=ew)
    frontier = seeds
    for b in blocks:
        src = b["src_ids"]
        for i, v in enumerate(frontier):
            row = ix[ip[v]:ip[v + 1]]
            rw = ew[ip[v]:ip[v + 1]]
            got = src[b["indices"][b["indptr"][i]:b["indptr"][i + 1]]]
            assert len(got) == min(int((rw > 0).sum()), 5)
            pos = np.searchsorted(row, got)
            assert np.all(rw[pos] > 0) and np.all(np.diff(pos) > 0)
        frontier = src
    # deterministic, and different from the uniform stream
    again = oracle.sample(ip, ix, seeds, [5, 5], 21, weights=ew)
    assert all(np.array_equal(x["indices"], y["indices"]) for x, y in zip(blocks, again))
    unif = oracle.sample(ip, ix, seeds, [5, 5], 21)
    assert not np.array_equal(blocks[1]["src_ids"], unif[1]["src_ids"])


@pytest.mark.parametrize("P", [2, 4])
def test_biased_csp_replay_equals_single_device(tiny_graph, P):
    """Weights travel with the owner's shard, tasks are pushed to them."""
    ip, ix = tiny_graph
    ew = _weights_for(ix)
    bnds = datagen.bounds(10_000, P)
    seeds = [np.arange(int(bnds[r]), int(bnds[r + 1]), 211, dtype=np.int32) for r in range(P)]
    blocks = replay_inprocess(ip, ix, bnds, seeds, [5, 3], 8, weights=ew)
    for r in range(P):
        ref = oracle.sample(ip, ix, seeds[r], [5, 3], 8, weights=ew)
        for b, e in zip(blocks[r], ref):
            for key in ("indptr", "indices", "src_ids"):
                assert np.array_equal(b[key], e[key])
