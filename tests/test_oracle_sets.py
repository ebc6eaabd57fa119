"""Pins for the oracle's RRR sets (Alg. 2; LT P:134-140).

1. The lazy BFS / walk equals reverse reachability of the root in the fully
   materialised live-edge world W_s, computed with scipy's BFS (a different
   algorithm and code base) -- every sample of the tested ranges.
2. Closed forms on special graphs (empty, path, star, cycle).
3. Exact enumeration of all live-edge worlds on tiny graphs: the empirical
   distribution of RRR sets matches the exact one (chi-square), and the RIS
   estimate n * F_R(S) matches the exact expected spread E[I(S)]
   (IC P:57/59, LT P:61) within 5 sigma.
"""
import itertools
from fractions import Fraction

import numpy as np
import pytest
from scipy.sparse import csr_matrix
from scipy.sparse.csgraph import breadth_first_order

import inputs
import oracle

SEED = 0x5EED


def _live_world_ic(off, nbr, seed, s):
    n = off.size - 1
    rows, cols = [], []
    for u in range(n):
        d = int(off[u + 1] - off[u])
        for e in range(int(off[u]), int(off[u + 1])):
            if oracle.ic_live(oracle.edge_draw(seed, s, e), d):
                rows.append(u)            # reverse edge u -> v (target to source)
                cols.append(int(nbr[e]))
    return rows, cols


def _live_world_lt(off, nbr, seed, s):
    n = off.size - 1
    rows, cols = [], []
    for u in range(n):
        d = int(off[u + 1] - off[u])
        if d == 0:
            continue
        j = oracle.lt_choice(oracle.lt_draw(seed, s, u), d)
        rows.append(u)
        cols.append(int(nbr[int(off[u]) + j]))
    return rows, cols


def _reverse_reach(n, rows, cols, root):
    A = csr_matrix((np.ones(len(rows)), (rows, cols)), shape=(n, n))
    order = breadth_first_order(A, root, directed=True, return_predecessors=False)
    return np.sort(order.astype(np.uint32))


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_lazy_traversal_equals_materialised_world(model):
    off, nbr = inputs.rmat(256, 2048, seed=3)
    n = 256
    world = _live_world_ic if model == "IC" else _live_world_lt
    for s in range(60):
        rows, cols = world(off, nbr, SEED, s)
        want = _reverse_reach(n, rows, cols, oracle.root(SEED, s, n))
        got = oracle.rrr_set(off, nbr, model, SEED, s)
        assert np.array_equal(got, want), (model, s)


def test_lazy_traversal_equals_world_on_C1_graph():
    off, nbr = inputs.config_graph("C1")
    n = off.size - 1
    for s in range(0, 400, 37):
        rows, cols = _live_world_ic(off, nbr, 1, s)
        want = _reverse_reach(n, rows, cols, oracle.root(1, s, n))
        assert np.array_equal(oracle.rrr_set(off, nbr, "IC", 1, s), want), s


def test_sample_range_matches_single_sets_and_is_thread_independent():
    off, nbr = inputs.config_graph("C1")
    o1, m1, ex1 = oracle.sample(off, nbr, "IC", 9, 100, 300, nthreads=1)
    o4, m4, ex4 = oracle.sample(off, nbr, "IC", 9, 100, 300, nthreads=4)
    assert np.array_equal(o1, o4) and np.array_equal(m1, m4) and ex1 == ex4
    for i in range(0, 300, 29):
        assert np.array_equal(m1[o1[i]:o1[i + 1]], oracle.rrr_set(off, nbr, "IC", 9, 100 + i))
    # composability: [a,b) ++ [b,c) == [a,c)
    oa, ma, _ = oracle.sample(off, nbr, "IC", 9, 100, 120)
    ob, mb, _ = oracle.sample(off, nbr, "IC", 9, 220, 180)
    assert np.array_equal(np.concatenate([ma, mb]), m1)
    assert np.array_equal(np.concatenate([oa[:-1], ob + oa[-1]]), o1)


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_empty_graph_sets_are_roots(model):
    off, nbr = inputs.empty_graph(50)
    for s in range(100):
        assert list(oracle.rrr_set(off, nbr, model, 4, s)) == [oracle.root(4, s, 50)]


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_path_graph_sets_are_prefixes(model):
    off, nbr = inputs.path_graph(40)  # in-degree 1 => p = 1 (IC) / forced choice (LT)
    for s in range(100):
        r = oracle.root(4, s, 40)
        assert list(oracle.rrr_set(off, nbr, model, 4, s)) == list(range(r + 1))


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_star_and_cycle(model):
    off, nbr = inputs.star_out(30)
    for s in range(60):
        r = oracle.root(2, s, 30)
        want = [0] if r == 0 else [0, r]
        assert list(oracle.rrr_set(off, nbr, model, 2, s)) == want
    off, nbr = inputs.cycle_graph(25)
    for s in range(30):
        assert list(oracle.rrr_set(off, nbr, model, 2, s)) == list(range(25))


# ---------------------------------------------------------------- enumeration
# In-degrees are powers of two so the discrete live probability is exactly 1/d.
TINY_EDGES = [(1, 0), (2, 0), (3, 0), (4, 0), (0, 1), (2, 1), (3, 2), (0, 3), (4, 3),
              (1, 4), (5, 4), (6, 5), (7, 6), (5, 7)]
TINY_N = 8


def _tiny():
    return inputs.from_edges(TINY_N, TINY_EDGES)


def _worlds(model, off, nbr):
    """Yield (probability, list of live edges (src, dst)) for every live-edge world."""
    n = off.size - 1
    if model == "IC":
        edges = []
        for v in range(n):
            d = int(off[v + 1] - off[v])
            for e in range(int(off[v]), int(off[v + 1])):
                edges.append((int(nbr[e]), v, Fraction(1, d)))
        sure = [(u, v) for (u, v, pe) in edges if pe == 1]
        edges = [x for x in edges if x[2] != 1]
        for mask in range(1 << len(edges)):
            p = Fraction(1)
            live = list(sure)
            for i, (u, v, pe) in enumerate(edges):
                if mask >> i & 1:
                    p *= pe
                    live.append((u, v))
                else:
                    p *= 1 - pe
            yield p, live
    else:
        choices = []
        for v in range(n):
            d = int(off[v + 1] - off[v])
            choices.append([(int(nbr[e]), v) for e in range(int(off[v]), int(off[v + 1]))] or [None])
        for combo in itertools.product(*choices):
            p = Fraction(1)
            for v in range(n):
                d = int(off[v + 1] - off[v])
                if d:
                    p *= Fraction(1, d)
            yield p, [c for c in combo if c is not None]


def _reach(n, live, start, forward):
    adj = [[] for _ in range(n)]
    for (u, v) in live:
        if forward:
            adj[u].append(v)
        else:
            adj[v].append(u)
    seen = set(start)
    stack = list(start)
    while stack:
        x = stack.pop()
        for y in adj[x]:
            if y not in seen:
                seen.add(y)
                stack.append(y)
    return frozenset(seen)


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_exact_enumeration_distribution_and_ris_spread(model):
    from scipy.stats import chisquare
    off, nbr = _tiny()
    n = TINY_N
    dist = {}
    spread = {}
    seeds_sets = [frozenset([a]) for a in range(n)] + [frozenset(c) for c in itertools.combinations(range(n), 2)]
    for p, live in _worlds(model, off, nbr):
        for r in range(n):
            X = _reach(n, live, [r], forward=False)
            dist[X] = dist.get(X, 0) + p / n
        for S in seeds_sets:
            spread[S] = spread.get(S, 0) + p * len(_reach(n, live, S, forward=True))
    assert sum(dist.values()) == 1
    # RIS identity on the exact quantities: E[I(S)] = n Pr[S meets RR]
    for S in seeds_sets:
        assert spread[S] == n * sum(q for X, q in dist.items() if X & S)
    N = 200_000
    offs, mem, _ = oracle.sample(off, nbr, model, 77, 0, N, nthreads=8)
    sets = [frozenset(mem[offs[i]:offs[i + 1]].tolist()) for i in range(N)]
    emp = {}
    for X in sets:
        emp[X] = emp.get(X, 0) + 1
    assert set(emp) <= set(dist), "oracle produced a set with zero exact probability"
    keys = sorted(dist, key=lambda X: (len(X), sorted(X)))
    exp_counts = np.array([float(dist[X]) * N for X in keys])
    obs = np.array([emp.get(X, 0) for X in keys], dtype=float)
    big = exp_counts >= 5
    f_obs = np.append(obs[big], obs[~big].sum())
    f_exp = np.append(exp_counts[big], exp_counts[~big].sum())
    if f_exp[-1] == 0:
        f_obs, f_exp = f_obs[:-1], f_exp[:-1]
    assert chisquare(f_obs, f_exp).pvalue > 1e-6
    for S in seeds_sets:
        hits = sum(1 for X in sets if X & S)
        est = n * hits / N
        pS = float(spread[S]) / n
        sigma = n * np.sqrt(max(pS * (1 - pS), 1e-12) / N)
        assert abs(est - float(spread[S])) < 5 * sigma + 1e-12, (S, est, float(spread[S]))
