"""Pins for the oracle's randomness (reading R1) -- no GPU.

Philox4x32-10 is pinned by the Random123 known-answer vectors (Salmon et al.,
SC'11, kat_vectors); the root draw (Alg. 2 l.6) by its closed form for
n = 2^a and by a chi-square uniformity test.
"""
import json
import os

import numpy as np
import pytest

import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "philox_kat.json")


def test_philox_known_answers():
    with open(GOLDEN) as f:
        kats = json.load(f)["vectors"]
    assert len(kats) >= 3
    for kat in kats:
        ctr = [int(x, 16) for x in kat["ctr"]]
        key = [int(x, 16) for x in kat["key"]]
        want = [int(x, 16) for x in kat["out"]]
        got = [int(x) for x in oracle.philox4x32_10(ctr, key)]
        assert got == want, kat


def test_counter_layout_and_tags():
    # counter = (lo q, hi q, lo s, (hi s & 0x3fffffff) | tag << 30), key = (lo seed, hi seed)
    seed, s, q = 0x0123456789ABCDEF, (5 << 32) | 77, (3 << 32) | 9
    for tag in (0, 1, 2):
        out = oracle.philox4x32_10(
            [q & 0xFFFFFFFF, q >> 32, s & 0xFFFFFFFF, ((s >> 32) & 0x3FFFFFFF) | (tag << 30)],
            [seed & 0xFFFFFFFF, seed >> 32])
        for w in range(4):
            assert oracle.draw(seed, s, tag, q, w) == int(out[w])
    # edge e uses quad e>>2, word e&3 of tag 0; LT vertex u uses quad u>>2, word u&3 of tag 2
    for e in (0, 1, 2, 3, 4, 7, 12345, (1 << 33) + 6):
        assert oracle.edge_draw(seed, s, e) == oracle.draw(seed, s, 0, e >> 2, e & 3)
    for u in (0, 3, 4, 1000001):
        assert oracle.lt_draw(seed, s, u) == oracle.draw(seed, s, 2, u >> 2, u & 3)
    # the three streams differ
    assert oracle.draw(seed, s, 0, 0, 0) != oracle.draw(seed, s, 1, 0, 0)
    assert oracle.draw(seed, s, 1, 0, 0) != oracle.draw(seed, s, 2, 0, 0)


@pytest.mark.parametrize("a", [1, 5, 10, 20, 31])
def test_root_power_of_two_closed_form(a):
    n = 1 << a
    for s in range(200):
        r64 = oracle.draw(7, s, 1, 0, 0) | (oracle.draw(7, s, 1, 0, 1) << 32)
        assert oracle.root(7, s, n) == r64 >> (64 - a)


def test_root_general_n_is_floor_of_product():
    for n in (3, 1000, 4847571, 65608366, 2**32 - 2):
        for s in range(50):
            r64 = oracle.draw(3, s, 1, 0, 0) | (oracle.draw(3, s, 1, 0, 1) << 32)
            assert oracle.root(3, s, n) == (r64 * n) >> 64
            assert 0 <= oracle.root(3, s, n) < n


def test_root_uniformity_chi_square():
    from scipy.stats import chisquare
    n = 64
    counts = np.zeros(n)
    for s in range(64 * 400):
        counts[oracle.root(11, s, n)] += 1
    p = chisquare(counts).pvalue
    assert p > 1e-4, p


def test_edge_draw_uniform_bits():
    # mean of u32 draws over 40k edges within 6 sigma of 2^31
    vals = np.array([oracle.edge_draw(1, 2, e) for e in range(40000)], dtype=np.float64)
    sigma = (2.0**32) / np.sqrt(12.0) / np.sqrt(vals.size)
    assert abs(vals.mean() - 2.0**31) < 6 * sigma
