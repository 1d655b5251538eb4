"""Pins for the oracle's randomness: Philox4x32-10, the key layout, the
multiply-shift range map and Floyd's algorithm (R5-R7)."""
import itertools
import math
import os
from collections import Counter

import numpy as np
import pytest

import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _kat():
    rows = []
    with open(os.path.join(GOLDEN, "philox4x32_10_kat.txt")) as f:
        for line in f:
            if line.strip() and not line.startswith("#"):
                w = [int(x, 16) for x in line.split()]
                rows.append((w[0:4], w[4:6], w[6:10]))
    return rows


@pytest.mark.parametrize("ctr,key,expect", _kat())
def test_philox_random123_kat(ctr, key, expect):
    """Published Random123 known-answer vectors (tests/golden/philox4x32_10_kat.txt)."""
    assert oracle.philox4x32_10(ctr, key).tolist() == expect


def test_draw_word_key_layout():
    """ctr = {slot, v, l, 'DSP1'}, key = {lo32(seed), hi32(seed)}, word = x1:x0
    (R5).  Cross-check against an independent derivation: the
    SURVEY.md 8(c) golden draws, produced by a separate Python Philox."""
    assert oracle.draw_word(0x5EED, 0, 12345, 0) == 0xB692378201EFCEA3
    assert oracle.draw_word(0x5EED, 1, 12345, 0) == 0x59AE8CE8C523349C
    assert oracle.draw_word(0x5EED, 11, 12345, 0) == 0x0D2EA10D17C3D5DE
    assert oracle.draw_word(0x5EED, 12, 12345, 0) == 0x433BF8BDE755FF88
    assert oracle.draw_word(0x5EED, 14, 12345, 0) == 0xC77F55D63E317688
    assert oracle.draw_word(0x5EEE, 0, 7, 2) == 0xD7B719EB4A325F91
    assert oracle.draw_word(0x5EEE, 4, 7, 2) == 0xAB6B7B3E3189279E
    assert oracle.draw_word(0xFFFFFFFFFFFFFFFF, 0, 2147483646, 1) == 0x2943F932D340C8EB
    assert oracle.draw_word(0xFFFFFFFFFFFFFFFF, 9, 2147483646, 1) == 0x52CCAEB3A7FFB752
    # the counter words are distinct inputs: permuting them changes the word
    w = oracle.draw_word(99, 3, 5, 1)
    assert w != oracle.draw_word(99, 5, 3, 1) and w != oracle.draw_word(99, 3, 1, 5)
    # the fourth counter word is the constant "DSP1"
    x = oracle.philox4x32_10([3, 5, 1, 0x44535031], [99, 0])
    assert w == (int(x[1]) << 32) | int(x[0])


def test_node_positions_golden():
    """End-to-end positions for the SURVEY.md 8(c) rows (one has two Floyd
    collisions at slots 11 and 12)."""
    assert oracle.node_positions(0x5EED, 12345, 0, 50, 15).tolist() == \
        [0, 2, 8, 12, 15, 16, 18, 20, 25, 27, 31, 38, 41, 46, 47]
    assert oracle.node_positions(0x5EEE, 7, 2, 6, 5).tolist() == [0, 1, 2, 3, 4]
    assert oracle.node_positions(0xFFFFFFFFFFFFFFFF, 2147483646, 1, 10**6, 10).tolist() == \
        [161191, 205751, 323435, 369474, 435986, 468464, 510994, 654202, 786444, 875354]
    # slot 11 draws 2 (already chosen) -> j = 46; slot 12 draws 12 -> j = 47
    assert oracle.draw(0x5EED, 11, 12345, 0, 47) == 2
    assert oracle.draw(0x5EED, 12, 12345, 0, 48) == 12


@pytest.mark.parametrize("m", [1, 2, 3, 5, 7, 10, 36, 1000, 999_991, 2**31 - 1, 2**32 - 1])
def test_mulhi_range_closed_form(m):
    """floor(x m / 2^64): value j has preimage [ceil(j 2^64/m), ceil((j+1) 2^64/m)),
    so each of the m values has floor or ceil of 2^64/m preimages.  Check the
    boundaries exactly with Python integers."""
    two64 = 1 << 64
    js = sorted(j for j in {0, 1, m // 2, m - 2, m - 1} if 0 <= j < m)
    for j in js:
        lo = -(-(j * two64) // m)              # ceil(j 2^64 / m)
        hi = -(-((j + 1) * two64) // m)        # ceil((j+1) 2^64 / m)
        assert oracle.mulhi_range(lo, m) == j
        assert oracle.mulhi_range(hi - 1, m) == j
        if hi < two64:
            assert oracle.mulhi_range(hi, m) == j + 1
        assert (hi - lo) in (two64 // m, -(-two64 // m))
    assert oracle.mulhi_range(two64 - 1, m) == m - 1
    assert oracle.mulhi_range(0, m) == 0


@pytest.mark.parametrize("d,k", [(5, 2), (6, 3), (7, 4), (8, 8), (9, 1), (6, 6), (7, 2), (5, 4)])
def test_floyd_exhaustive(d, k):
    """Every draw vector r_t in [0, d-k+t] yields k distinct positions in
    [0, d) and each of the C(d, k) subsets occurs exactly k! times
    (d!/(d-k)! vectors in total)."""
    seen = Counter()
    ranges = [range(d - k + t + 1) for t in range(k)]
    total = 0
    for r in itertools.product(*ranges):
        pos = oracle.floyd(d, k, r)
        assert len(set(pos.tolist())) == k
        assert pos.min() >= 0 and pos.max() < d
        seen[tuple(sorted(pos.tolist()))] += 1
        total += 1
    assert total == math.factorial(d) // math.factorial(d - k)
    assert len(seen) == math.comb(d, k)
    assert set(seen.values()) == {math.factorial(k)}


def test_floyd_slot_convention():
    """Slot t chooses among j + 1 = d - k + t + 1 positions; a repeated draw
    takes j itself (Floyd 1987 / Bentley 'Programming Pearls')."""
    assert oracle.floyd(5, 3, [0, 0, 0]).tolist() == [0, 3, 4]
    assert oracle.floyd(5, 3, [2, 3, 4]).tolist() == [2, 3, 4]
    assert oracle.floyd(5, 3, [1, 1, 1]).tolist() == [1, 3, 4]
    assert oracle.floyd(5, 3, [0, 1, 1]).tolist() == [0, 1, 4]
    assert oracle.floyd(5, 3, [2, 0, 2]).tolist() == [2, 0, 4]


def test_node_positions_whole_row_consumes_no_draws():
    for d in range(0, 6):
        assert oracle.node_positions(123, 4, 0, d, 5).tolist() == list(range(d))
        assert oracle.node_positions(456, 4, 0, d, 5).tolist() == list(range(d))


def _chi2_pvalue(counts, expected):
    from scipy.stats import chisquare
    return chisquare(counts, expected).pvalue


def test_uniformity_over_seeds():
    """k-subsets of a (d=6, k=3) row across 60k rng_seeds: chi-square with 19 df."""
    n = 60_000
    c = Counter(tuple(oracle.node_positions(s, 77, 1, 6, 3).tolist()) for s in range(n))
    assert len(c) == 20
    counts = np.array(list(c.values()), float)
    assert _chi2_pvalue(counts, np.full(20, n / 20)) > 1e-4


def test_uniformity_over_nodes():
    """Same-degree rows of distinct nodes at one rng_seed: chi-square with 9 df."""
    n = 40_000
    c = Counter(tuple(oracle.node_positions(0x5EED, v, 0, 5, 2).tolist()) for v in range(n))
    assert len(c) == 10
    counts = np.array(list(c.values()), float)
    assert _chi2_pvalue(counts, np.full(10, n / 10)) > 1e-4


def test_hub_inclusion_frequency():
    """Each neighbour of a d = 10^4 hub is included with probability k/d."""
    d, k, n = 10_000, 5, 20_000
    hits = np.zeros(d)
    for s in range(n):
        hits[oracle.node_positions(s, 3, 2, d, k)] += 1
    # total inclusions exactly n k; per-decile frequency within 3 sigma of k/d
    assert hits.sum() == n * k
    dec = hits.reshape(10, -1).sum(1)
    exp = n * k / 10
    assert np.all(np.abs(dec - exp) < 4 * np.sqrt(exp))


def test_fanout_one_is_uniform_walk_step():
    """k = 1 is a random-walk step: uniform over the d neighbours."""
    d, n = 7, 35_000
    c = Counter(int(oracle.node_positions(s, 11, 0, d, 1)[0]) for s in range(n))
    counts = np.array([c[i] for i in range(d)], float)
    assert _chi2_pvalue(counts, np.full(d, n / d)) > 1e-4
