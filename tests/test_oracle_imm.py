"""Pins for the oracle's IMM driver (Alg. 1; [22] Alg. 2, Eq. 6, 9).

- lambda', lambda*, ln C(n,k) against mpmath at 40 digits (1e-9 relative);
- the theta_i schedule ceil(lambda' 2^i / n) (mpmath) for the five configs;
- the stop test, LB and final theta recomputed from the reported (cov_i, |R|);
- the spread on the empty graph equals n * #{s : root_s in S} / theta exactly;
- the path graph (p = 1): greedy takes vertex 0 first with gain theta.
"""
import math

import mpmath
import numpy as np
import pytest

import inputs
import oracle

mpmath.mp.dps = 40


def _mp_params(n, k, eps, ell):
    n_, k_, eps_, ell_ = mpmath.mpf(n), k, mpmath.mpf(eps), mpmath.mpf(ell)
    ln_n = mpmath.log(n_)
    ell_p = ell_ * (1 + mpmath.log(2) / ln_n)
    eps_p = mpmath.sqrt(2) * eps_
    lnC = mpmath.log(mpmath.binomial(n_, k_))
    lam_p = (2 + mpmath.mpf(2) / 3 * eps_p) * (lnC + ell_p * ln_n + mpmath.log(mpmath.log(n_, 2))) * n_ / eps_p**2
    e1 = 1 - 1 / mpmath.e
    alpha = mpmath.sqrt(ell_p * ln_n + mpmath.log(2))
    beta = mpmath.sqrt(e1 * (lnC + ell_p * ln_n + mpmath.log(2)))
    lam_s = 2 * n_ * (e1 * alpha + beta) ** 2 / eps_**2
    return dict(ell_p=ell_p, eps_p=eps_p, lnC=lnC, lambda_p=lam_p, lambda_s=lam_s)


CASES = [(c["n"], c["k"], c["eps"], c["ell"]) for c in inputs.CONFIGS.values()] + [
    (2, 1, 0.1, 1.0), (100, 100, 0.9, 2.0), (12345, 7, 0.05, 1.0), (2**31, 1000, 0.2, 1.5)]


@pytest.mark.parametrize("n,k,eps,ell", CASES)
def test_params_against_mpmath(n, k, eps, ell):
    p = oracle.imm_params(n, k, eps, ell)
    ref = _mp_params(n, k, eps, ell)
    for f in ("ell_p", "eps_p", "lnC", "lambda_p", "lambda_s"):
        got, want = getattr(p, f), float(ref[f])
        assert abs(got - want) <= 1e-9 * abs(want), (f, got, want)


# Survey §8(c) table: theta_1..theta_7 = ceil(lambda' 2^i / n), ell = 1.
THETA_TABLE = {
    "C1": [394, 787, 1574, 3147, 6294, 12587, 25173],
    "C2": [6331, 12662, 25324, 50647, 101294, 202587, 405174],
    "C3": [29139, 58277, 116553, 233106, 466211, 932422, 1864844],
    "C4": [7417, 14834, 29667, 59333, 118665, 237330, 474659],
    "C5": [577720, 1155440, 2310880, 4621760, 9243519, 18487037, 36974073],
}


@pytest.mark.parametrize("cfg", sorted(THETA_TABLE))
def test_theta_schedule(cfg):
    c = inputs.CONFIGS[cfg]
    p = oracle.imm_params(c["n"], c["k"], c["eps"], c["ell"])
    ref = _mp_params(c["n"], c["k"], c["eps"], c["ell"])
    for i, want in enumerate(THETA_TABLE[cfg], start=1):
        exact = ref["lambda_p"] * 2**i / c["n"]
        assert int(mpmath.ceil(exact)) == want
        # not a knife edge for ceil(), so the double evaluation must agree
        assert math.ceil(math.ldexp(p.lambda_p, i) / c["n"]) == want


def _check_schedule(r, n, k, eps, ell):
    p = oracle.imm_params(n, k, eps, ell)
    R_prev = 0
    lb = 1.0
    for i, (th, cov) in enumerate(zip(r["theta_i"], r["cov_i"]), start=1):
        assert th == max(R_prev, math.ceil(math.ldexp(p.lambda_p, i) / n))
        R_prev = th
        stop = cov * 2.0**i >= (1.0 + p.eps_p) * th
        last = i == len(r["theta_i"])
        if not last:
            assert not stop
        if stop:
            lb = (n * cov) / ((1.0 + p.eps_p) * th)
    if lb == 1.0:  # no break: the loop ran for every i < log2 n
        assert len(r["theta_i"]) == math.ceil(math.log2(n)) - 1
    assert r["lb"] == lb
    assert r["theta"] == max(R_prev, math.ceil(p.lambda_s / lb))
    assert r["spread"] == n * r["cov"] / r["theta"]


@pytest.mark.parametrize("model", ["IC", "LT"])
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_imm_schedule_recomputed_C1(model, seed):
    off, nbr = inputs.config_graph("C1")
    r = oracle.imm(off, nbr, 5, 0.5, 1.0, model, seed)
    _check_schedule(r, 1024, 5, 0.5, 1.0)
    assert len(set(r["seeds"].tolist())) == 5


def test_imm_empty_graph_closed_form():
    n, k = 64, 3
    off, nbr = inputs.empty_graph(n)
    r = oracle.imm(off, nbr, k, 0.5, 1.0, "IC", 5)
    _check_schedule(r, n, k, 0.5, 1.0)
    roots = np.array([oracle.root(5, s, n) for s in range(r["theta"])])
    counts = np.bincount(roots, minlength=n)
    # greedy on singleton sets = most frequent roots, ties to lowest id
    order = sorted(range(n), key=lambda v: (-counts[v], v))[:k]
    assert list(r["seeds"]) == order
    hits = int(np.isin(roots, order).sum())
    assert r["cov"] == hits
    assert r["spread"] == n * hits / r["theta"]


def test_imm_path_graph_first_pick_covers_everything():
    off, nbr = inputs.path_graph(32)   # every RRR set contains vertex 0
    r = oracle.imm(off, nbr, 2, 0.5, 1.0, "IC", 1)
    assert r["seeds"][0] == 0 and r["cov"] == r["theta"] and r["spread"] == 32.0


def test_invalid_parameters():
    for args in [(1, 1, 0.5, 1.0), (10, 0, 0.5, 1.0), (10, 11, 0.5, 1.0), (10, 2, 0.0, 1.0),
                 (10, 2, 1.0, 1.0), (10, 2, 0.5, 0.0)]:
        with pytest.raises(ValueError):
            oracle.imm_params(*args)


# ---------------------------------------------------------------- closed forms
# The stop test, LB and theta of the martingale loop ([22] Alg. 2; prose at
# P:65 and P:76) pinned on graphs where one vertex lies in EVERY RRR set
# (path 0 -> 1 -> ..., hub -> leaves, directed cycle; in-degree <= 1 means
# p = 1 under WC, so IC and LT sets are the same deterministic sets): the
# first greedy pick covers all of R, so cov_i = |R| = theta_i in every round
# and the stop test cov_i 2^i >= (1+eps') |R| reduces to 2^i >= 1+eps'.  The
# loop therefore breaks at the first i >= 1 with 2^i >= 1+eps' (i = 1 when
# eps <= 1/sqrt 2, else i = 2), provided i < log2 n; then LB = n / (1+eps')
# and theta = max(theta_i, ceil(lambda* (1+eps') / n)).  If the loop runs out
# (i < log2 n fails first) LB = 1 and theta = max(theta_last, ceil(lambda*)).
# Everything below is evaluated in mpmath at 40 digits, independently of the
# oracle's double arithmetic; a wrong comparison (> vs >=, <= log2 n), a wrong
# LB or theta_i instead of |R| changes one of the integers.
def _mp_ceil_safe(x):
    c = mpmath.ceil(x)
    assert c - x > mpmath.mpf("1e-9") or x == c, f"knife edge for ceil: {x}"
    return int(c)


def closed_form_all_covered(n, k, eps, ell):
    mp = _mp_params(n, k, eps, ell)
    log2n = mpmath.log(n, 2)
    thetas, lb, i = [], None, 1
    while i < log2n:
        thetas.append(_mp_ceil_safe(mp["lambda_p"] * 2**i / n))
        if 2**i >= 1 + mp["eps_p"]:
            lb = n / (1 + mp["eps_p"])
            break
        i += 1
    theta = max(thetas[-1] if thetas else 0, _mp_ceil_safe(mp["lambda_s"] / (lb if lb is not None else 1)))
    return dict(theta_i=thetas, lb=lb, theta=theta)


ALL_COVERED_GRAPHS = {"path": inputs.path_graph, "star": inputs.star_out, "cycle": inputs.cycle_graph}
ALL_COVERED_CASES = [  # (n, k, eps, ell): i* = 1 / i* = 2 / loop bound hit / no round at all
    (33, 1, 0.5, 1.0), (33, 3, 0.9, 1.0), (1000, 2, 0.1, 2.0), (5, 2, 0.9, 1.0), (4, 1, 0.9, 1.0),
    (4, 2, 0.5, 1.0), (2, 1, 0.3, 1.0), (300, 5, 0.69, 0.5), (300, 5, 0.72, 0.5)]


@pytest.mark.parametrize("shape", sorted(ALL_COVERED_GRAPHS))
@pytest.mark.parametrize("model", ["IC", "LT"])
@pytest.mark.parametrize("n,k,eps,ell", ALL_COVERED_CASES)
def test_imm_stop_test_lb_theta_closed_form(shape, model, n, k, eps, ell):
    off, nbr = ALL_COVERED_GRAPHS[shape](n)
    want = closed_form_all_covered(n, k, eps, ell)
    r = oracle.imm(off, nbr, k, eps, ell, model, 11)
    assert r["theta_i"] == want["theta_i"]
    assert r["cov_i"] == want["theta_i"]        # the first pick covers every set
    assert r["rounds"] == len(want["theta_i"])
    if want["lb"] is None:
        assert r["lb"] == 1.0
    else:
        assert abs(r["lb"] - float(want["lb"])) <= 1e-12 * float(want["lb"])
    assert r["theta"] == want["theta"]
    assert r["cov"] == r["theta"] and r["spread"] == float(n)
    # vertex 0 first; every later pick has gain 0 and is the lowest unselected id (R10)
    assert r["seeds"].tolist() == list(range(k))


def test_closed_form_reaches_both_break_rounds():
    # the case table exercises a break at i = 1, a break at i = 2, the loop
    # bound (i < log2 n) and the empty loop -- keep it that way
    kinds = set()
    for n, k, eps, ell in ALL_COVERED_CASES:
        w = closed_form_all_covered(n, k, eps, ell)
        kinds.add((len(w["theta_i"]), w["lb"] is None))
    assert {(1, False), (2, False), (1, True), (0, True)} <= kinds


# Coverage counts C[v] = #sets containing v (Alg. 2 l.25).
def test_coverage_closed_forms():
    n, cnt = 40, 3000
    for model in ("IC", "LT"):
        # path 0 -> ... -> n-1 with p = 1: RR(root) = {0..root}, so C[j] = #{s : root_s >= j}
        off, nbr = inputs.path_graph(n)
        o, m, _ = oracle.sample(off, nbr, model, 3, 0, cnt)
        roots = np.array([oracle.root(3, s, n) for s in range(cnt)])
        want = np.array([(roots >= j).sum() for j in range(n)])
        assert np.array_equal(oracle.coverage(n, o, m), want)
        # cycle: every set is V
        off, nbr = inputs.cycle_graph(n)
        o, m, _ = oracle.sample(off, nbr, model, 3, 0, cnt)
        assert np.array_equal(oracle.coverage(n, o, m), np.full(n, cnt))
    # no edges: singleton sets, C = root frequencies
    off, nbr = inputs.empty_graph(n)
    o, m, _ = oracle.sample(off, nbr, "IC", 4, 0, cnt)
    roots = [oracle.root(4, s, n) for s in range(cnt)]
    assert np.array_equal(oracle.coverage(n, o, m), np.bincount(roots, minlength=n))


def test_coverage_brute_force_random_arenas():
    rng = np.random.default_rng(5)
    for _ in range(20):
        n = int(rng.integers(1, 60))
        sets = [rng.choice(n, size=int(rng.integers(0, n + 1)), replace=False) for _ in range(int(rng.integers(0, 40)))]
        offs = np.zeros(len(sets) + 1, dtype=np.uint64)
        offs[1:] = np.cumsum([len(s) for s in sets])
        mem = np.concatenate(sets).astype(np.uint32) if sets and offs[-1] else np.zeros(0, dtype=np.uint32)
        C = oracle.coverage(n, offs, mem)
        for v in range(n):
            assert C[v] == sum(1 for s in sets if v in set(s.tolist()))
        assert int(C.sum()) == int(offs[-1])
