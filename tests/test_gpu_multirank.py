"""Multi-rank IMM on one GPU: the library's own multi-rank code path.

eim_create_group makes p contexts in one process ("virtual ranks" sharing
cuda:0) with an in-process communicator in place of NCCL; each rank is driven
by its own host thread, exactly like one process per GPU.  Every rank runs
the sharded sampling (eim_shard_range shares of every round, lookahead
launches included), compacts its part, exchanges it (all-gather of counts,
one broadcast per share), appends the others' parts in rank (= sample-id)
order, histograms and runs the greedy.  Bar (BASELINE north_star): every
rank's seeds, theta, theta_i, cov_i, LB, spread, arena size and coverage
counts C equal the CPU oracle bit-exactly, and the examined edges summed over
the ranks equal the oracle's -- for p in {2, 3, 8}, IC and LT, with source
elimination (the cut of the first theta non-empty sets can fall in any
rank's share) and the fresh final phase.
"""
import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np
import pytest

import inputs
import oracle

pytestmark = pytest.mark.gpu

NT = max(1, min(64, os.cpu_count() or 1))
ELIM, FRESH = oracle.SOURCE_ELIM, oracle.FRESH_FINAL


@pytest.fixture(scope="module")
def eim():
    from paper_conf_sc_doneyhl25_b200 import _build
    _build.build()
    import paper_conf_sc_doneyhl25_b200 as E
    return E


class Group:
    def __init__(self, eim, p, off, nbr, gflags=0):
        self.eim = eim
        self.ctxs = eim.eim_create_group([0] * p)
        self.graphs = [eim.eim_load_graph_csr(c, off, nbr, gflags=gflags) for c in self.ctxs]
        self.pool = ThreadPoolExecutor(p)

    def imm(self, *args, flags=0, per_rank_args=None):
        futs = []
        for r, (c, g) in enumerate(zip(self.ctxs, self.graphs)):
            a = per_rank_args[r] if per_rank_args else args
            futs.append(self.pool.submit(self.eim.eim_imm_run, c, g, *a, flags=flags))
        out = []
        for f in futs:
            try:
                out.append(f.result())
            except Exception as e:  # noqa: BLE001 -- collected per rank
                out.append(e)
        return out

    def close(self):
        self.pool.shutdown()
        for c, g in zip(self.ctxs, self.graphs):
            self.eim.eim_graph_free(g)
            self.eim.eim_destroy(c)


def _check(eim, grp, off, nbr, k, eps, ell, model, seed, flags=0, coverage=True):
    res = grp.imm(k, eps, ell, model, seed, flags=flags)
    ref = oracle.imm(off, nbr, k, eps, ell, model, seed, nthreads=NT, flags=flags)
    n = off.size - 1
    edges = 0
    for r, x in enumerate(res):
        assert not isinstance(x, Exception), (r, x)
        seeds, theta, spread, st = x
        assert np.array_equal(seeds, ref["seeds"]), (r, model, flags)
        assert theta == ref["theta"] and spread == ref["spread"], r
        for key in ("theta_i", "cov_i", "lb", "cov", "arena_elems", "ids_sampled", "lambda_p", "lambda_s"):
            assert st[key] == ref[key], (r, key, st[key], ref[key])
        edges += st["edges_examined"]
    assert edges == ref["edges_examined"]
    if coverage and not flags & ELIM:
        first = oracle.FRESH_BASE if flags & FRESH else 0
        ro, rm, _ = oracle.sample(off, nbr, model, seed, first, ref["theta"], nthreads=NT)
        want = oracle.coverage(n, ro, rm)
        for c in grp.ctxs:
            assert np.array_equal(eim.eim_get_coverage(c, n), want)
    return res


@pytest.mark.parametrize("p", [2, 3, 8])
@pytest.mark.parametrize("model", ["IC", "LT"])
def test_multirank_imm_C1(eim, p, model):
    off, nbr = inputs.config_graph("C1")
    grp = Group(eim, p, off, nbr)
    try:
        for seed in (1, 2):
            for k, eps in ((5, 0.5), (50, 0.2), (1024, 0.5)):
                _check(eim, grp, off, nbr, k, eps, 1.0, model, seed)
        for flags in (ELIM, FRESH, ELIM | FRESH):
            for seed in (1, 3):
                _check(eim, grp, off, nbr, 20, 0.3, 1.0, model, seed, flags=flags)
    finally:
        grp.close()


@pytest.mark.parametrize("p", [2, 5])
def test_multirank_special_graphs(eim, p):
    # tiny rounds (fewer sets than ranks in the first round of a 3-vertex
    # graph), every set = V (cycle), singletons (no edges), a packed store
    cases = [(inputs.path_graph(32), 0), (inputs.cycle_graph(700), 0), (inputs.star_out(90), 0),
             (inputs.from_edges(3, [(0, 1), (0, 2)]), 0), (inputs.rmat(600, 60000, seed=4), 1)]
    for (off, nbr), gflags in cases:
        grp = Group(eim, p, off, nbr, gflags=gflags)
        try:
            for model in ("IC", "LT"):
                _check(eim, grp, off, nbr, 3, 0.5, 1.0, model, 7)
                _check(eim, grp, off, nbr, 2, 0.5, 1.0, model, 7, flags=ELIM)
        finally:
            grp.close()
    off, nbr = inputs.empty_graph(64)
    grp = Group(eim, p, off, nbr)
    try:
        _check(eim, grp, off, nbr, 3, 0.5, 1.0, "IC", 5)
    finally:
        grp.close()


def test_multirank_C2(eim):
    c = inputs.CONFIGS["C2"]
    off, nbr = inputs.config_graph("C2")
    for p in (2, 8):
        grp = Group(eim, p, off, nbr)
        try:
            _check(eim, grp, off, nbr, c["k"], c["eps"], c["ell"], "IC", 1)
            if p == 8:
                _check(eim, grp, off, nbr, c["k"], c["eps"], c["ell"], "IC", 1, flags=ELIM)
        finally:
            grp.close()


def test_multirank_C3(eim):
    c = inputs.CONFIGS["C3"]
    off, nbr = inputs.config_graph("C3")
    grp = Group(eim, 3, off, nbr)
    try:
        _check(eim, grp, off, nbr, c["k"], c["eps"], c["ell"], "LT", 1)
        _check(eim, grp, off, nbr, c["k"], c["eps"], c["ell"], "LT", 1, flags=ELIM | FRESH, coverage=False)
    finally:
        grp.close()


def test_multirank_split_launches(eim, monkeypatch):
    # several launches per range on every rank (table budget), plain and
    # with source elimination; the launch sizes of all ranks must agree
    monkeypatch.setenv("EIM_MAX_LAUNCH_IDS", "300")
    off, nbr = inputs.config_graph("C1")
    grp = Group(eim, 3, off, nbr)
    try:
        for model in ("IC", "LT"):
            _check(eim, grp, off, nbr, 10, 0.3, 1.0, model, 4)
            _check(eim, grp, off, nbr, 10, 0.3, 1.0, model, 4, flags=ELIM)
    finally:
        grp.close()


def test_multirank_failure_releases_peers(eim):
    # one rank fails its argument check: the others must not wait for it
    off, nbr = inputs.config_graph("C1")
    grp = Group(eim, 3, off, nbr)
    try:
        good = (5, 0.5, 1.0, "IC", 1)
        res = grp.imm(per_rank_args=[good, (0, 0.5, 1.0, "IC", 1), good])
        assert isinstance(res[1], eim.EimError) and res[1].status == eim.EIM_E_INVAL
        for r in (0, 2):
            assert isinstance(res[r], eim.EimError) and res[r].status == eim.EIM_E_NCCL, res[r]
        # local calls still work on every rank
        for c, g in zip(grp.ctxs, grp.graphs):
            o, m = eim.eim_sample_rrr(c, g, "IC", 1, 0, 100)
            ro, rm, _ = oracle.sample(off, nbr, "IC", 1, 0, 100)
            assert np.array_equal(o, ro) and np.array_equal(m, rm)
    finally:
        grp.close()


def test_group_single_rank_is_plain_context(eim):
    off, nbr = inputs.config_graph("C1")
    grp = Group(eim, 1, off, nbr)
    try:
        _check(eim, grp, off, nbr, 5, 0.5, 1.0, "IC", 2)
    finally:
        grp.close()
