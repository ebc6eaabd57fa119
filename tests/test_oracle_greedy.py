"""Pins for the oracle's greedy NodeSelection (Alg. 3).

Brute force on tiny instances: every gain_j equals the maximal marginal
coverage given the earlier picks, the pick is the lowest id among the
maximisers (reading R10), cov is the size of the union of covered sets, the
(1 - (1-1/k)^k) >= (1-1/e) approximation bound against brute-force OPT, and
gains are non-increasing (submodularity of coverage).
"""
import itertools

import numpy as np
import pytest

import oracle


def _random_arena(rng, n, num_sets, max_len):
    sets = []
    for _ in range(num_sets):
        L = int(rng.integers(1, max_len + 1))
        sets.append(sorted(rng.choice(n, size=min(L, n), replace=False).tolist()))
    offsets = np.zeros(num_sets + 1, dtype=np.uint64)
    offsets[1:] = np.cumsum([len(s) for s in sets])
    members = np.array([x for s in sets for x in s], dtype=np.uint32)
    return sets, offsets, members


def _coverage(sets, S):
    S = set(S)
    return sum(1 for s in sets if S.intersection(s))


@pytest.mark.parametrize("trial", range(40))
def test_greedy_against_brute_force(trial):
    rng = np.random.default_rng(1000 + trial)
    n = int(rng.integers(3, 12))
    num_sets = int(rng.integers(1, 30))
    k = int(rng.integers(1, min(4, n) + 1))
    sets, offsets, members = _random_arena(rng, n, num_sets, 4)
    seeds, gains, cov = oracle.greedy(n, offsets, members, k)
    chosen = []
    for j in range(k):
        best_gain = max(_coverage(sets, chosen + [u]) - _coverage(sets, chosen)
                        for u in range(n) if u not in chosen)
        argmins = [u for u in range(n) if u not in chosen
                   and _coverage(sets, chosen + [u]) - _coverage(sets, chosen) == best_gain]
        assert int(gains[j]) == best_gain
        assert int(seeds[j]) == min(argmins)
        chosen.append(int(seeds[j]))
    assert cov == _coverage(sets, chosen) == int(gains.sum())
    assert all(gains[j] >= gains[j + 1] for j in range(k - 1))
    opt = max(_coverage(sets, S) for S in itertools.combinations(range(n), k))
    assert cov >= (1 - (1 - 1 / k) ** k) * opt - 1e-12
    assert cov >= (1 - 1 / np.e) * opt - 1e-12


def test_all_zero_case_picks_lowest_unselected_ids():
    # one set {5}; after picking 5 every count is 0 -> lowest unselected ids 0, 1, 2
    offsets = np.array([0, 1], dtype=np.uint64)
    members = np.array([5], dtype=np.uint32)
    seeds, gains, cov = oracle.greedy(8, offsets, members, 4)
    assert list(seeds) == [5, 0, 1, 2]
    assert list(gains) == [1, 0, 0, 0] and cov == 1
    seeds, gains, cov = oracle.greedy(4, np.zeros(1, dtype=np.uint64), np.zeros(0, dtype=np.uint32), 4)
    assert list(seeds) == [0, 1, 2, 3] and cov == 0


def test_ties_resolve_to_lowest_id():
    # {1,2} {1,2} {3}: 1 and 2 tie at 2 -> pick 1; then 3 (gain 1) vs 2 (gain 0)
    offsets = np.array([0, 2, 4, 5], dtype=np.uint64)
    members = np.array([1, 2, 1, 2, 3], dtype=np.uint32)
    seeds, gains, cov = oracle.greedy(6, offsets, members, 3)
    assert list(seeds) == [1, 3, 0] and list(gains) == [2, 1, 0] and cov == 3


def test_monotone_submodular_coverage_on_random_subsets():
    rng = np.random.default_rng(3)
    sets, offsets, members = _random_arena(rng, 20, 60, 6)
    for _ in range(200):
        T = set(rng.choice(20, size=8, replace=False).tolist())
        S = set(list(T)[:4])
        x = int(rng.integers(0, 20))
        assert _coverage(sets, S) <= _coverage(sets, T)
        if x not in T:
            assert (_coverage(sets, S | {x}) - _coverage(sets, S)
                    >= _coverage(sets, T | {x}) - _coverage(sets, T))
