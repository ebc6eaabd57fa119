"""Pins for the oracle's general edge probabilities (NEXT-3; P:57, P:61,
P:136-138; reading R25: p_e = (x_e + 1) / 2^32).

1. Weights derived from the weighted cascade reproduce the pinned WC path
   exactly (IC: x = floor((2^32-1)/d); LT: x_j = ceil((j+1) 2^32/d) -
   ceil(j 2^32/d) - 1), sets and IMM.
2. Decision boundaries restated with exact rationals (the first
   in-neighbour whose inclusive running sum exceeds tau).
3. Exact enumeration of all live-edge worlds under non-uniform weights,
   including the LT "no in-neighbour" outcome (sum p < 1): chi-square of the
   set distribution and the RIS identity n Pr[S meets RR] = E[I(S)].
"""
import itertools
from fractions import Fraction

import numpy as np
import pytest

import inputs
import oracle
from test_oracle_sets import TINY_EDGES, TINY_N, _reach

TWO32 = 2**32


def _wc_weights(off, model):
    d = np.diff(off).astype(np.int64)
    x = []
    for v in range(off.size - 1):
        dv = int(d[v])
        for j in range(dv):
            if model == "IC":
                x.append((TWO32 - 1) // dv)
            else:
                b0 = -(-j * TWO32 // dv)
                b1 = -(-(j + 1) * TWO32 // dv)
                x.append(b1 - b0 - 1)
    return np.array(x, dtype=np.uint32)


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_wc_derived_weights_reproduce_wc(model):
    for off, nbr in (inputs.config_graph("C1"), inputs.rmat(300, 3000, seed=5), inputs.star_out(40)):
        x = _wc_weights(off, model)
        a = oracle.sample(off, nbr, model, 3, 17, 3000, nthreads=4)
        b = oracle.sample(off, nbr, model, 3, 17, 3000, nthreads=4, x=x)
        assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1]) and a[2] == b[2]
    off, nbr = inputs.config_graph("C1")
    x = _wc_weights(off, model)
    r1 = oracle.imm(off, nbr, 5, 0.5, 1.0, model, 2)
    r2 = oracle.imm(off, nbr, 5, 0.5, 1.0, model, 2, x=x)
    for key in ("seeds", "theta", "spread", "theta_i", "cov_i", "edges_examined", "arena_elems"):
        assert np.array_equal(r1[key], r2[key]), key


def test_ic_boundaries():
    rng = np.random.default_rng(1)
    for x in [0, 1, 2**31 - 1, 2**31, TWO32 - 2, TWO32 - 1, *rng.integers(0, TWO32, 50).tolist()]:
        p = Fraction(x + 1, TWO32)
        for draw in {max(x - 1, 0), x, min(x + 1, TWO32 - 1)}:
            assert oracle.ic_live_w(draw, x) == (Fraction(draw, TWO32) < p)
    assert all(oracle.ic_live_w(d, TWO32 - 1) for d in (0, 2**31, TWO32 - 1))


def test_lt_boundaries_and_no_neighbour():
    rng = np.random.default_rng(2)
    for trial in range(200):
        d = int(rng.integers(1, 9))
        w = rng.integers(1, TWO32 // d, size=d)
        if trial % 3 == 0:
            w[-1] = TWO32 - int(w[:-1].sum())     # sum p = 1 exactly
        x = (w - 1).astype(np.uint32)
        cum = np.cumsum(w)
        taus = {0, TWO32 - 1}
        for c in cum:
            taus |= {int(c) - 1, int(c), min(int(c) + 1, TWO32 - 1)}
        for tau in taus:
            if tau >= TWO32:
                continue
            # P:136 in exact rationals: first j whose inclusive sum of p exceeds tau/2^32
            want, s = None, Fraction(0)
            for j in range(d):
                s += Fraction(int(w[j]), TWO32)
                if s > Fraction(tau, TWO32):
                    want = j
                    break
            assert oracle.lt_choice_w(tau, x) == want, (w, tau)
    assert oracle.lt_choice_w(5, np.zeros(0, dtype=np.uint32)) is None


def test_lt_weight_sum_validated():
    off, nbr = inputs.from_edges(3, [(0, 2), (1, 2)])
    assert oracle.lt_weights_ok(off, np.array([2**31 - 1, 2**31 - 1], dtype=np.uint32))       # sum = 1
    assert not oracle.lt_weights_ok(off, np.array([2**31, 2**31 - 1], dtype=np.uint32))       # sum > 1
    with pytest.raises(RuntimeError):
        oracle.imm(off, nbr, 1, 0.5, 1.0, "LT", 1, x=np.array([2**31, 2**31 - 1], dtype=np.uint32))
    oracle.imm(off, nbr, 1, 0.5, 1.0, "IC", 1, x=np.array([2**31, 2**31 - 1], dtype=np.uint32))


# dyadic probabilities so the enumeration is exact and small
P_CHOICES = [Fraction(1, 4), Fraction(1, 2), Fraction(3, 4), Fraction(1, 8), Fraction(5, 8), Fraction(1, 1)]


def _tiny_weights(model, seed):
    off, nbr = inputs.from_edges(TINY_N, TINY_EDGES)
    rng = np.random.default_rng(seed)
    p = []
    for v in range(TINY_N):
        dv = int(off[v + 1] - off[v])
        if model == "IC":
            p += [P_CHOICES[i] for i in rng.integers(0, len(P_CHOICES), dv)]
        else:  # random split of a total mass < 1 (room for "no neighbour") or = 1
            total = Fraction(int(rng.integers(4, 9)), 8)
            cuts = sorted(Fraction(int(c), 16) * total for c in rng.integers(1, 16, dv - 1))
            parts = [b - a for a, b in zip([Fraction(0)] + cuts, cuts + [total])]
            parts = [q if q > 0 else Fraction(1, 64) for q in parts]
            scale = min(Fraction(1), total / sum(parts))
            p += [q * scale for q in parts]
    x = np.array([int(q * TWO32) - 1 for q in p], dtype=np.uint32)
    return off, nbr, p, x


def _worlds_w(model, off, nbr, p):
    n = off.size - 1
    edges = [(int(nbr[e]), v, p[e]) for v in range(n) for e in range(int(off[v]), int(off[v + 1]))]
    if model == "IC":
        for mask in range(1 << len(edges)):
            pr = Fraction(1)
            live = []
            for i, (u, v, pe) in enumerate(edges):
                if mask >> i & 1:
                    pr *= pe
                    live.append((u, v))
                else:
                    pr *= 1 - pe
            if pr:
                yield pr, live
    else:
        choices = []
        for v in range(n):
            row = [(int(nbr[e]), v, p[e]) for e in range(int(off[v]), int(off[v + 1]))]
            rest = 1 - sum(q for (_, _, q) in row)
            choices.append(row + ([(None, v, rest)] if rest > 0 else []))
        for combo in itertools.product(*choices):
            pr = Fraction(1)
            for (_, _, q) in combo:
                pr *= q
            yield pr, [(u, v) for (u, v, _) in combo if u is not None]


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_exact_enumeration_general_weights(model):
    from scipy.stats import chisquare
    off, nbr, p, x = _tiny_weights(model, 11)
    n = TINY_N
    dist, spread = {}, {}
    seeds_sets = [frozenset([a]) for a in range(n)] + [frozenset(c) for c in itertools.combinations(range(n), 2)]
    for pr, live in _worlds_w(model, off, nbr, p):
        for r in range(n):
            X = _reach(n, live, [r], forward=False)
            dist[X] = dist.get(X, 0) + pr / n
        for S in seeds_sets:
            spread[S] = spread.get(S, 0) + pr * len(_reach(n, live, S, forward=True))
    assert sum(dist.values()) == 1
    for S in seeds_sets:
        assert spread[S] == n * sum(q for X, q in dist.items() if X & S)
    N = 200_000
    offs, mem, _ = oracle.sample(off, nbr, model, 91, 0, N, nthreads=8, x=x)
    sets = [frozenset(mem[offs[i]:offs[i + 1]].tolist()) for i in range(N)]
    emp = {}
    for X in sets:
        emp[X] = emp.get(X, 0) + 1
    assert set(emp) <= set(dist)
    keys = sorted(dist, key=lambda X: (len(X), sorted(X)))
    f_exp = np.array([float(dist[X]) * N for X in keys])
    f_obs = np.array([emp.get(X, 0) for X in keys], dtype=float)
    big = f_exp >= 5
    f_obs = np.append(f_obs[big], f_obs[~big].sum())
    f_exp = np.append(f_exp[big], f_exp[~big].sum())
    if f_exp[-1] == 0:
        f_obs, f_exp = f_obs[:-1], f_exp[:-1]
    assert chisquare(f_obs, f_exp).pvalue > 1e-6
    for S in seeds_sets:
        hits = sum(1 for X in sets if X & S)
        pS = float(spread[S]) / n
        sigma = n * np.sqrt(max(pS * (1 - pS), 1e-12) / N)
        assert abs(n * hits / N - float(spread[S])) < 5 * sigma + 1e-12
