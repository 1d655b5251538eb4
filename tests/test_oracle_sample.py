"""Pins for the oracle's multi-layer sampling, block construction and gather:
the paper's worked examples (Fig. 3, Fig. 5), invariants, the full-row special
case against scipy.sparse, CSP-replay invariance and error behaviour."""
import json
import os

import numpy as np
import pytest
import scipy.sparse as sp

import datagen
import oracle
from csp_replay import owner_of, replay_inprocess

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def csr_from_rows(n, rows):
    indptr = np.zeros(n + 1, np.int64)
    cols = []
    for v in range(n):
        r = sorted(rows.get(str(v), []))
        cols.extend(r)
        indptr[v + 1] = indptr[v] + len(r)
    return indptr, np.array(cols, np.int32)


def assert_block_eq(got, exp):
    for key in ("num_dst", "num_src", "num_edges"):
        assert int(got[key]) == int(exp[key]), key
    for key in ("indptr", "indices", "src_ids"):
        assert np.asarray(got[key]).tolist() == list(exp[key]), key


# ---------------------------------------------------------------- worked examples

def test_fig3_worked_example():
    g = json.load(open(os.path.join(GOLDEN, "fig3_worked_example.json")))
    ip, ix = csr_from_rows(g["num_nodes"], g["rows"])
    for rng_seed in (0, 1, 0x5EED):          # no draw is consumed: any seed
        blocks = oracle.sample(ip, ix, g["seeds"], g["fanouts"], rng_seed)
        for b, e in zip(blocks, g["blocks"]):
            assert_block_eq(b, e)
    # the graph sample needs exactly the features of A, B, C, E, G, H, K
    names = g["names"]
    assert sorted(names[i] for i in blocks[-1]["src_ids"]) == sorted(g["loader_node_set"])
    # layer 1 outputs C and E; layer 2: C -> B, K and E -> G, H
    b0, b1 = blocks
    assert [names[b0["src_ids"][j]] for j in b0["indices"]] == ["C", "E"]
    pairs = {names[b1["src_ids"][i]]: [names[b1["src_ids"][j]] for j in
                                        b1["indices"][b1["indptr"][i]:b1["indptr"][i + 1]]]
             for i in range(b1["num_dst"])}
    assert pairs["C"] == ["B", "K"] and pairs["E"] == ["G", "H"]


def test_fig5_csp_example():
    g = json.load(open(os.path.join(GOLDEN, "fig5_csp_example.json")))
    ip, ix = csr_from_rows(g["num_nodes"], g["rows"])
    log = []
    blocks = replay_inprocess(ip, ix, np.array(g["bounds"]), g["rank_seeds"], g["fanouts"], 7, log)
    # message pattern of P:L148: E goes GPU1 -> GPU2, B goes GPU2 -> GPU1, A and F stay
    assert log[0]["shuffle"] == g["messages"]["shuffle"]
    rr = {k: {str(kk): vv for kk, vv in v.items()} for k, v in log[0]["reshuffle_rows"].items()}
    assert rr == g["messages"]["reshuffle_rows"]
    for r in range(2):
        for b, e in zip(blocks[r], g["blocks"][r]):
            assert_block_eq(b, e)
        # invariance: the single-device oracle on the same seeds gives the same blocks
        for b, e in zip(oracle.sample(ip, ix, g["rank_seeds"][r], g["fanouts"], 7), g["blocks"][r]):
            assert_block_eq(b, e)


# ------------------------------------------------------------------- invariants

def check_block_invariants(b, frontier, indptr, indices, k):
    F = len(frontier)
    src = b["src_ids"]
    assert b["num_dst"] == F and len(src) == b["num_src"]
    assert src[:F].tolist() == list(frontier)
    assert len(np.unique(src)) == len(src)
    ip = b["indptr"]
    assert ip[0] == 0 and ip[-1] == b["num_edges"] and np.all(np.diff(ip) >= 0)
    for i in range(F):
        v = frontier[i]
        row = indices[indptr[v]:indptr[v + 1]]
        got = src[b["indices"][ip[i]:ip[i + 1]]]
        assert len(got) == min(len(row), k)                 # cnt = min(deg, k)
        assert np.all(np.isin(got, row))                     # membership
        assert len(np.unique(got)) == len(got)               # no duplicates
        pos = np.searchsorted(row, got)
        assert np.all(np.diff(pos) > 0)                      # ascending row position
    # new nodes in first-occurrence order over the edge list (np.unique, library routine)
    edge_src = src[b["indices"]]
    new_mask = ~np.isin(edge_src, frontier)
    cand = edge_src[new_mask]
    _, first = np.unique(cand, return_index=True)
    assert src[F:].tolist() == cand[np.sort(first)].tolist()


def test_tiny_invariants(tiny_graph):
    ip, ix = tiny_graph
    cfg = datagen.CONFIGS["tiny"]
    train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
    seeds = datagen.rank_seed_batches(train, datagen.bounds(cfg.num_nodes, 1), 0, cfg.batch, 0)[0]
    blocks = oracle.sample(ip, ix, seeds, cfg.fanouts, 0x5EED)
    frontier = seeds
    for l, b in enumerate(blocks):
        check_block_invariants(b, frontier, ip, ix, cfg.fanouts[l])
        frontier = b["src_ids"]


def test_sampled_rows_match_node_positions(tiny_graph):
    """The layer pieces agree with the per-node positions they are built from."""
    ip, ix = tiny_graph
    ids = np.arange(0, 10_000, 37, dtype=np.int32)
    cnt, rows = oracle.sample_rows(ip, ix, ids, 7, 1, 99)
    for i, v in enumerate(ids):
        pos = oracle.node_positions(99, int(v), 1, int(ip[v + 1] - ip[v]), 7)
        assert cnt[i] == len(pos)
        assert rows[i, :cnt[i]].tolist() == ix[ip[v] + pos].tolist()
        assert np.all(rows[i, cnt[i]:] == -1)


def random_capped_graph(n, max_deg, seed):
    rng = np.random.default_rng(seed)
    rows = {}
    for v in range(n):
        d = int(rng.integers(0, max_deg + 1))
        nb = rng.choice(n, size=d, replace=False)
        rows[str(v)] = sorted(int(x) for x in nb if x != v)
    return csr_from_rows(n, rows)


def test_full_row_special_case_is_khop_bfs():
    """k >= max degree: sampling is deterministic and each block is CSR row
    slicing of the frontier (scipy.sparse), with new nodes in first-occurrence
    order (np.unique)."""
    n = 300
    ip, ix = random_capped_graph(n, 12, 3)
    A = sp.csr_matrix((np.ones(len(ix)), ix, ip), shape=(n, n))
    A.sort_indices()
    seeds = np.array([5, 17, 250, 3], np.int32)
    fan = [12, 16, 32]
    blocks = oracle.sample(ip, ix, seeds, fan, 1234)
    blocks2 = oracle.sample(ip, ix, seeds, fan, 4321)
    frontier = seeds
    for b, b2 in zip(blocks, blocks2):
        for key in ("indptr", "indices", "src_ids"):
            assert np.array_equal(b[key], b2[key])
        sub = A[frontier]
        assert b["indptr"].tolist() == sub.indptr.tolist()
        assert b["src_ids"][b["indices"]].tolist() == sub.indices.tolist()
        cand = sub.indices[~np.isin(sub.indices, frontier)]
        _, first = np.unique(cand, return_index=True)
        assert b["src_ids"].tolist() == list(frontier) + cand[np.sort(first)].tolist()
        # the node set is the BFS ball: frontier plus its out-neighbours (symmetric not needed)
        ball = set(frontier.tolist()) | set(sub.indices.tolist())
        assert set(b["src_ids"].tolist()) == ball
        frontier = b["src_ids"]


def test_degree_zero_and_edge_cases():
    rows = {"0": [], "1": [0], "2": [0, 1], "3": [0, 1, 2], "4": [0, 1, 2, 3]}
    ip, ix = csr_from_rows(5, rows)
    b = oracle.sample(ip, ix, [0, 4, 2], [3], 5)[0]
    assert b["indptr"].tolist() == [0, 0, 3, 5]                # deg 0, deg k+1, deg < k
    assert b["src_ids"][:3].tolist() == [0, 4, 2]
    # empty batch is allowed and yields empty blocks
    e = oracle.sample(ip, ix, np.zeros(0, np.int32), [3, 2], 5)
    assert all(x["num_dst"] == 0 and x["num_edges"] == 0 for x in e)
    # deg == k takes the whole row in order
    b = oracle.sample(ip, ix, [3], [3], 5)[0]
    assert b["src_ids"][b["indices"]].tolist() == [0, 1, 2]


def test_errors():
    ip, ix = csr_from_rows(3, {"0": [1], "1": [0, 2], "2": [1]})
    with pytest.raises(oracle.OracleError) as e:
        oracle.sample(ip, ix, [0, 0], [2], 1)
    assert e.value.code == oracle.ERR_DUPLICATE_SEED
    with pytest.raises(oracle.OracleError) as e:
        oracle.sample(ip, ix, [3], [2], 1)
    assert e.value.code == oracle.ERR_OUT_OF_RANGE
    with pytest.raises(oracle.OracleError) as e:
        oracle.sample(ip, ix, [-1], [2], 1)
    assert e.value.code == oracle.ERR_OUT_OF_RANGE
    for bad in ([0], [33], [2] * 9, []):
        with pytest.raises(oracle.OracleError) as e:
            oracle.sample(ip, ix, [0], bad, 1)
        assert e.value.code == oracle.ERR_INVALID_ARG


# --------------------------------------------------------- partition invariance

@pytest.mark.parametrize("P", [2, 3, 4, 8])
def test_csp_replay_equals_single_device(tiny_graph, P):
    """Each rank's blocks under the shuffle/sample/reshuffle replay equal the
    single-device oracle on that rank's seeds (CSP is exact)."""
    ip, ix = tiny_graph
    cfg = datagen.CONFIGS["tiny"]
    bnds = datagen.bounds(cfg.num_nodes, P)
    train = datagen.train_ids(cfg.num_nodes, cfg.train_count)
    seeds = [datagen.rank_seed_batches(train, bnds, r, 32, 1)[0] for r in range(P)]
    blocks = replay_inprocess(ip, ix, bnds, seeds, cfg.fanouts, 0x5EED + 3)
    for r in range(P):
        assert np.all(owner_of(seeds[r], bnds) == r)          # co-partitioned seeds
        ref = oracle.sample(ip, ix, seeds[r], cfg.fanouts, 0x5EED + 3)
        for b, e in zip(blocks[r], ref):
            for key in ("indptr", "indices", "src_ids"):
                assert np.array_equal(b[key], e[key])


def test_same_node_same_samples_across_requesters(tiny_graph):
    """DESIGN.md R16: the draw key is (seed, layer, node, slot), not the requester."""
    ip, ix = tiny_graph
    a = oracle.sample(ip, ix, [10, 20, 30], [5, 5], 77)
    b = oracle.sample(ip, ix, [30, 40], [5, 5], 77)
    def row(bl, v):
        i = bl["src_ids"].tolist().index(v)
        return bl["src_ids"][bl["indices"][bl["indptr"][i]:bl["indptr"][i + 1]]].tolist()
    assert row(a[0], 30) == row(b[0], 30)


# ----------------------------------------------------------------------- gather

def test_gather_is_row_copy():
    f = datagen.features(0, 500, 16)
    ids = np.array([3, 499, 0, 3, 250], np.int32)
    out = oracle.gather(f, ids)
    assert out.view(np.uint32).tolist() == f[ids].view(np.uint32).tolist()
    # closed form of the feature recipe (datagen.c): SURVEY.md 8(c) values
    assert hex(out[2, 0].view(np.uint32)) == "0x3fcbac1a"
    with pytest.raises(oracle.OracleError):
        oracle.gather(f, np.array([500], np.int32))
