"""Pins for the oracle's random walks (R27): a functional
graph gives the iterated function, dead ends terminate, each step is the
fan-out-1 node-wise sample (read off oracle.sample's blocks through local ids),
and the walk's distribution on a small regular graph converges to uniform."""
from collections import Counter

import numpy as np
import pytest
from scipy.stats import chisquare

import oracle


def csr(n, rows):
    ip = np.zeros(n + 1, np.int64)
    cols = []
    for v in range(n):
        r = sorted(rows.get(v, []))
        cols += r
        ip[v + 1] = ip[v] + len(r)
    return ip, np.array(cols, np.int32)


def test_functional_graph_is_iterated_function():
    n = 11
    f = {v: (3 * v + 2) % n for v in range(n)}
    ip, ix = csr(n, {v: [f[v]] for v in range(n)})
    tr = oracle.random_walk(ip, ix, [0, 5, 7], 20, 1234)
    for row in tr:
        for a, b in zip(row[:-1], row[1:]):
            assert b == f[a]


def test_dead_end_terminates():
    ip, ix = csr(4, {0: [1], 1: [2], 2: [], 3: [0]})
    tr = oracle.random_walk(ip, ix, [3, 2], 5, 9)
    assert tr[0].tolist() == [3, 0, 1, 2, -1, -1]
    assert tr[1].tolist() == [2, -1, -1, -1, -1, -1]


def test_steps_are_fanout_one_node_wise_samples(tiny_graph):
    ip, ix = tiny_graph
    starts = np.arange(0, 10_000, 97, dtype=np.int32)
    L = 6
    tr = oracle.random_walk(ip, ix, starts, L, 0x5EED)
    blocks = oracle.sample(ip, ix, starts, [1] * L, 0x5EED)
    loc = np.arange(len(starts))
    alive = np.ones(len(starts), bool)
    for l, b in enumerate(blocks):
        cnt = b["indptr"][loc + 1] - b["indptr"][loc]
        alive &= cnt > 0
        nxt = np.where(alive, b["indices"][np.minimum(b["indptr"][loc], max(len(b["indices"]) - 1, 0))], -1)
        glob = np.where(alive, b["src_ids"][np.maximum(nxt, 0)], -1)
        assert np.array_equal(tr[:, l + 1], glob)
        loc = np.where(alive, nxt, 0)


def test_walk_mixes_to_uniform_on_regular_graph():
    """4-regular non-bipartite circulant graph: the position after 40 steps is
    uniform over the 9 nodes (stationary distribution deg/2m = 1/9)."""
    n = 9
    ip, ix = csr(n, {v: [(v + 1) % n, (v - 1) % n, (v + 2) % n, (v - 2) % n] for v in range(n)})
    ends = Counter(int(oracle.random_walk(ip, ix, [0], 40, s)[0, -1]) for s in range(18_000))
    obs = np.array([ends[v] for v in range(n)], float)
    assert chisquare(obs, np.full(n, obs.sum() / n)).pvalue > 1e-4


def test_errors():
    ip, ix = csr(3, {0: [1], 1: [0], 2: []})
    with pytest.raises(oracle.OracleError):
        oracle.random_walk(ip, ix, [3], 2, 1)
    with pytest.raises(oracle.OracleError):
        oracle.random_walk(ip, ix, [0], 0, 1)


# ------------------------------------------- independent walks (R35)

def test_independent_structure_and_dead_ends(tiny_graph):
    """Every step goes to a neighbour of the previous node, a dead end
    terminates, a degree-1 node is followed without a draw (functional graph
    = the iterated function, as in the node-keyed mode)."""
    ip, ix = tiny_graph
    starts = np.arange(0, 10_000, 37, dtype=np.int32)
    tr = oracle.random_walk(ip, ix, starts, 12, 0xABC, independent=True)
    for row in tr:
        for a, b in zip(row[:-1], row[1:]):
            if a < 0:
                assert b == -1
            elif ip[a + 1] == ip[a]:
                assert b == -1
            else:
                assert b in ix[ip[a]:ip[a + 1]]
    n = 11
    f = {v: (3 * v + 2) % n for v in range(n)}
    fip, fix = csr(n, {v: [f[v]] for v in range(n)})
    for row in oracle.random_walk(fip, fix, [0, 5, 7, 0], 15, 3, independent=True):
        assert all(b == f[a] for a, b in zip(row[:-1], row[1:]))
    dip, dix = csr(4, {0: [1], 1: [2], 2: [], 3: [0]})
    assert oracle.random_walk(dip, dix, [3], 5, 9, independent=True)[0].tolist() == [3, 0, 1, 2, -1, -1]


def test_independent_walks_from_one_start_are_independent_and_uniform():
    """Star: node 0 with neighbours 1..6.  In one call, 24,000 walks from node
    0: the first steps are uniform over the 6 neighbours and consecutive walks
    are independent (chi-square over the 36 ordered pairs).  In the
    node-keyed mode (R27) the same walks are all identical."""
    m = 6
    ip, ix = csr(m + 1, {0: list(range(1, m + 1)), **{v: [0] for v in range(1, m + 1)}})
    starts = np.zeros(24_000, np.int32)
    tr = oracle.random_walk(ip, ix, starts, 1, 0x1D, independent=True)
    first = tr[:, 1]
    c = Counter(first.tolist())
    assert set(c) == set(range(1, m + 1))
    assert chisquare(np.array([c[v] for v in range(1, m + 1)], float), np.full(m, len(first) / m)).pvalue > 1e-4
    pairs = Counter(zip(first[0::2].tolist(), first[1::2].tolist()))
    obs = np.array([pairs[(a, b)] for a in range(1, m + 1) for b in range(1, m + 1)], float)
    assert chisquare(obs, np.full(m * m, obs.sum() / (m * m))).pvalue > 1e-4
    keyed = oracle.random_walk(ip, ix, starts[:100], 1, 0x1D)
    assert len(set(keyed[:, 1].tolist())) == 1


def test_independent_walks_mix_within_one_call():
    """The 4-regular circulant graph of test_walk_mixes_to_uniform_on_regular_graph:
    18,000 walks from node 0 in ONE call end uniformly over the 9 nodes."""
    n = 9
    ip, ix = csr(n, {v: [(v + 1) % n, (v - 1) % n, (v + 2) % n, (v - 2) % n] for v in range(n)})
    ends = oracle.random_walk(ip, ix, np.zeros(18_000, np.int32), 40, 5, independent=True)[:, -1]
    c = Counter(ends.tolist())
    obs = np.array([c[v] for v in range(n)], float)
    assert chisquare(obs, np.full(n, obs.sum() / n)).pvalue > 1e-4
