"""Pins for the oracle's NEXT rows.

NEXT-1, source-vertex elimination (reading R22): a set is the
plain RRR set without its source (root) vertex; IMM keeps the first non-empty
sets in sample-id order, |R| counts kept sets only.  Pinned by
  - the set relation plain(s) = elim(s) + {root(s)}, root from the pinned
    orc_root (every id of the tested ranges, IC and LT);
  - closed forms on the path and star graphs (IMM picks the vertex every kept
    set contains; ids_sampled is fixed by the root draws alone);
  - exact enumeration of all live-edge worlds: the law of the kept sets is
    Pr[RR \\ {root} = X] / Pr[RR \\ {root} != {}] (chi-square);
  - the kept collection equals the non-empty sets of ids [0, ids_sampled),
    the last id kept; the theta schedule recomputed from (theta_i, cov_i).
NEXT-4, fresh final phase (R23): the estimation phase is the plain run's;
the final NodeSelection runs on theta = ceil(lambda*/LB) sets of ids
FRESH_BASE.. (pinned against the pinned sampler and greedy).
"""
import itertools
import math
from fractions import Fraction

import numpy as np
import pytest

import inputs
import oracle

from test_oracle_sets import _reach, _tiny, _worlds, TINY_N  # noqa: E402

ELIM, FRESH = oracle.SOURCE_ELIM, oracle.FRESH_FINAL


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_elim_set_is_plain_set_minus_root(model):
    for off, nbr, seed in ((*inputs.rmat(300, 3000, seed=5), 3), (*inputs.config_graph("C1"), 1)):
        n = off.size - 1
        po, pm, pe = oracle.sample(off, nbr, model, seed, 40, 700, per_set_edges=True)
        eo, em, ee = oracle.sample(off, nbr, model, seed, 40, 700, nthreads=3, flags=ELIM, per_set_edges=True)
        assert np.array_equal(pe, ee)  # the traversal is unchanged: same work per set
        for i in range(700):
            plain = pm[po[i]:po[i + 1]].tolist()
            el = em[eo[i]:eo[i + 1]].tolist()
            r = oracle.root(seed, 40 + i, n)
            assert r in plain and r not in el
            assert sorted(el + [r]) == plain
            assert el == sorted(el)


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_elim_imm_path_graph_closed_form(model):
    n = 40
    off, nbr = inputs.path_graph(n)  # p = 1 on every edge: RR(j) = {0..j}; kept set = {0..j-1}
    r = oracle.imm(off, nbr, 3, 0.5, 1.0, model, 11, flags=ELIM)
    assert r["seeds"][0] == 0 and r["cov"] == r["theta"] and r["spread"] == float(n)
    # ids_sampled: the theta-th id whose root is not vertex 0, plus one
    kept, s = 0, 0
    while kept < r["theta"]:
        kept += oracle.root(11, s, n) != 0
        s += 1
    assert r["ids_sampled"] == s
    # arena: a kept set of root j has j members
    roots = [oracle.root(11, t, n) for t in range(s)]
    assert r["arena_elems"] == sum(j for j in roots if j)


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_elim_star_graph_closed_form(model):
    n = 30
    off, nbr = inputs.star_out(n)  # hub 0 -> leaves: kept set of a leaf root = {0}; hub root -> empty
    o, m, _ = oracle.sample(off, nbr, model, 4, 0, 500, flags=ELIM)
    for i in range(500):
        want = [] if oracle.root(4, i, n) == 0 else [0]
        assert m[o[i]:o[i + 1]].tolist() == want
    r = oracle.imm(off, nbr, 2, 0.5, 1.0, model, 4, flags=ELIM)
    assert r["seeds"][0] == 0 and r["cov"] == r["theta"] and r["arena_elems"] == r["theta"]


def test_elim_rejects_graphs_without_proper_edges():
    for off, nbr in (inputs.empty_graph(16), inputs.from_edges(4, [(0, 0), (2, 2)])):
        with pytest.raises(RuntimeError):
            oracle.imm(off, nbr, 1, 0.5, 1.0, "IC", 1, flags=ELIM)
    # a single proper edge is enough
    r = oracle.imm(*inputs.from_edges(4, [(0, 0), (1, 2)]), 1, 0.5, 1.0, "IC", 1, flags=ELIM)
    assert r["seeds"][0] == 1 and r["cov"] == r["theta"]


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_elim_exact_enumeration_of_kept_set_law(model):
    from scipy.stats import chisquare
    off, nbr = _tiny()
    n = TINY_N
    dist = {}
    for p, live in _worlds(model, off, nbr):
        for r in range(n):
            X = _reach(n, live, [r], forward=False) - {r}
            dist[X] = dist.get(X, 0) + p / n
    assert sum(dist.values()) == 1
    q_empty = dist.pop(frozenset(), Fraction(0))
    kept = {X: q / (1 - q_empty) for X, q in dist.items()}
    N = 200_000
    offs, mem, _ = oracle.sample(off, nbr, model, 78, 0, N, nthreads=8, flags=ELIM)
    lens = np.diff(offs)
    emp = {}
    for i in np.nonzero(lens)[0]:
        X = frozenset(mem[offs[i]:offs[i + 1]].tolist())
        emp[X] = emp.get(X, 0) + 1
    nk = int((lens > 0).sum())
    # the fraction of empty (discarded) sets is the exact Pr[RR = {root}]
    sd = math.sqrt(float(q_empty * (1 - q_empty)) / N)
    assert abs((N - nk) / N - float(q_empty)) <= 5 * sd   # LT here: every root has a proper in-edge, q = 0
    assert set(emp) <= set(kept)
    keys = sorted(kept, key=lambda X: (len(X), sorted(X)))
    f_exp = np.array([float(kept[X]) * nk for X in keys])
    f_obs = np.array([emp.get(X, 0) for X in keys], dtype=float)
    big = f_exp >= 5
    f_obs = np.append(f_obs[big], f_obs[~big].sum())
    f_exp = np.append(f_exp[big], f_exp[~big].sum())
    if f_exp[-1] == 0:
        f_obs, f_exp = f_obs[:-1], f_exp[:-1]
    assert chisquare(f_obs, f_exp).pvalue > 1e-6


@pytest.mark.parametrize("model", ["IC", "LT"])
@pytest.mark.parametrize("seed", [1, 2])
def test_elim_imm_keeps_first_nonempty_sets_in_id_order(model, seed):
    off, nbr = inputs.config_graph("C1")
    n, k, eps = 1024, 5, 0.5
    r = oracle.imm(off, nbr, k, eps, 1.0, model, seed, flags=ELIM)
    S = r["ids_sampled"]
    o, m, ex = oracle.sample(off, nbr, model, seed, 0, S, nthreads=4, flags=ELIM, per_set_edges=True)
    lens = np.diff(o)
    assert int((lens > 0).sum()) == r["theta"] and lens[-1] > 0   # minimal prefix of ids
    assert r["arena_elems"] == int(m.size)
    assert r["edges_examined"] == int(ex.sum())
    # final greedy on the kept sets (pinned greedy)
    keep = np.nonzero(lens)[0]
    ko = np.zeros(keep.size + 1, dtype=np.uint64)
    ko[1:] = np.cumsum(lens[keep])
    km = np.concatenate([m[o[i]:o[i + 1]] for i in keep])
    seeds, gains, cov = oracle.greedy(n, ko, km, k)
    assert np.array_equal(seeds, r["seeds"]) and cov == r["cov"]
    assert r["spread"] == n * cov / r["theta"]
    # theta schedule on kept counts
    p = oracle.imm_params(n, k, eps, 1.0)
    lb = 1.0
    for i, (th, c) in enumerate(zip(r["theta_i"], r["cov_i"]), start=1):
        assert th == math.ceil(math.ldexp(p.lambda_p, i) / n)
        if c * 2.0**i >= (1.0 + p.eps_p) * th:
            lb = (n * c) / ((1.0 + p.eps_p) * th)
    assert r["lb"] == lb and r["theta"] == max(r["theta_i"][-1], math.ceil(p.lambda_s / lb))


@pytest.mark.parametrize("model", ["IC", "LT"])
@pytest.mark.parametrize("flags", [FRESH, FRESH | ELIM])
def test_fresh_final_phase(model, flags):
    off, nbr = inputs.config_graph("C1")
    n, k, eps = 1024, 5, 0.5
    base = oracle.imm(off, nbr, k, eps, 1.0, model, 2, flags=flags & ELIM)
    r = oracle.imm(off, nbr, k, eps, 1.0, model, 2, flags=flags)
    for key in ("rounds", "theta_i", "cov_i", "lb", "lambda_p", "lambda_s"):
        assert r[key] == base[key], key
    p = oracle.imm_params(n, k, eps, 1.0)
    theta = math.ceil(p.lambda_s / r["lb"])
    assert r["theta"] == theta            # exactly ceil(lambda*/LB), even below the estimation |R|
    # ids of the estimation phase: the shortest id prefix with theta_i[-1] kept sets
    eo, _, eex = oracle.sample(off, nbr, model, 2, 0, base["ids_sampled"], nthreads=4, flags=flags & ELIM,
                               per_set_edges=True)
    est_ids = int(np.searchsorted(np.cumsum(np.diff(eo) > 0 if flags & ELIM else np.ones(eo.size - 1)),
                                  r["theta_i"][-1])) + 1
    o, m, ex = oracle.sample(off, nbr, model, 2, oracle.FRESH_BASE, theta * 3, nthreads=4, flags=flags & ELIM,
                             per_set_edges=True)
    lens = np.diff(o)
    keep = np.nonzero(lens)[0][:theta] if flags & ELIM else np.arange(theta)
    assert keep.size == theta
    ko = np.zeros(theta + 1, dtype=np.uint64)
    ko[1:] = np.cumsum(lens[keep])
    km = np.concatenate([m[o[i]:o[i + 1]] for i in keep])
    seeds, gains, cov = oracle.greedy(n, ko, km, k)
    assert np.array_equal(seeds, r["seeds"]) and cov == r["cov"]
    assert r["arena_elems"] == int(km.size)
    assert r["spread"] == n * cov / theta
    fresh_ids = int(keep[-1]) + 1
    assert r["ids_sampled"] == est_ids + fresh_ids
    assert r["edges_examined"] == int(eex[:est_ids].sum()) + int(ex[:fresh_ids].sum())
