"""Pins for the per-edge / per-vertex decisions of the diffusion models.

IC (Alg. 2 l.17 "r <= p_vu", P:59 p = 1/d): reading R2, r = draw/2^32,
live <=> r < 1/d.  Pinned by exact rational arithmetic (fractions) on every
boundary draw, and by the closed form T = floor((2^32-1)/d) it must equal.

LT: reading R3-R5, prefix-scan choice over weights 1/d.
Pinned by the closed form floor(tau * d / 2^32) -- a different algorithm
from the oracle's scan -- and by exact Fractions at every boundary.
"""
from fractions import Fraction

import pytest

import oracle

TWO32 = 1 << 32


def _degrees():
    ds = list(range(1, 300)) + [2**k for k in range(1, 32)] + [3 * 2**k for k in range(0, 30)]
    ds += [51141, 88370, 1_000_003, 2**31 - 1, 2**32 - 1]
    return sorted(set(ds))


def test_ic_live_degree_one_always_live():
    for draw in (0, 1, 2**31, TWO32 - 1):
        assert oracle.ic_live(draw, 1)


def test_ic_live_degree_two_exactly_half():
    assert oracle.ic_live(2**31 - 1, 2)
    assert not oracle.ic_live(2**31, 2)


@pytest.mark.parametrize("d", _degrees())
def test_ic_live_matches_exact_rational_at_boundaries(d):
    T = (TWO32 - 1) // d  # survey closed form; equals ceil(2^32/d) - 1
    assert T == -(-TWO32 // d) - 1
    for draw in {0, max(T - 1, 0), T, min(T + 1, TWO32 - 1), TWO32 - 1}:
        exact = Fraction(draw, TWO32) < Fraction(1, d)
        assert oracle.ic_live(draw, d) == exact, (d, draw)
        assert exact == (draw <= T)


def _scan_choice(tau, d):
    """Independent restatement of P:136: first j whose inclusive weight sum exceeds tau."""
    t = Fraction(tau, TWO32)
    acc = Fraction(0)
    for j in range(d):
        acc += Fraction(1, d)
        if acc > t:
            return j
    return None


@pytest.mark.parametrize("d", [1, 2, 3, 5, 7, 8, 13, 64, 100, 255, 1000, 4096])
def test_lt_choice_scan_and_closed_form_on_all_boundaries(d):
    for j in range(d):
        Bj = -(-(j * TWO32) // d)  # ceil(j 2^32 / d): smallest tau choosing >= j
        for tau in {Bj - 1, Bj, Bj + 1}:
            if not (0 <= tau < TWO32):
                continue
            got = oracle.lt_choice(tau, d)
            assert got == (tau * d) >> 32, (d, tau)
            if d <= 256:
                assert got == _scan_choice(tau, d), (d, tau)


def test_lt_choice_large_degrees_closed_form():
    import random
    rng = random.Random(5)
    for d in (51141, 88370, 2**20 + 7):
        for _ in range(200):
            tau = rng.randrange(TWO32)
            assert oracle.lt_choice(tau, d) == (tau * d) >> 32
        assert oracle.lt_choice(0, d) == 0
        assert oracle.lt_choice(TWO32 - 1, d) == d - 1
