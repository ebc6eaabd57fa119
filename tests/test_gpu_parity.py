"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bar (BASELINE north_star): RRR sets, coverage, theta and seed sets
bit-exact; spread (a double computed from the same integers) identical.
Sizes span several tiles and ragged tails; the full-size configs run the
launch configuration bench.py times (eim_imm_run on C2), with the oracle
multi-threaded over sample ids (identical results by construction).
"""
import os

import numpy as np
import pytest

import inputs
import oracle

pytestmark = pytest.mark.gpu

NT = max(1, min(64, os.cpu_count() or 1))


@pytest.fixture(scope="module")
def eim():
    from paper_conf_sc_doneyhl25_b200 import _build
    _build.build()
    import paper_conf_sc_doneyhl25_b200 as E
    return E


@pytest.fixture(scope="module")
def ctx(eim):
    c = eim.eim_create(0)
    yield c
    eim.eim_destroy(c)


@pytest.fixture(scope="module")
def graphs():
    cache = {}

    def get(name):
        if name not in cache:
            cache[name] = inputs.config_graph(name)
        return cache[name]
    return get


def _sets_equal(eim, ctx, g, off, nbr, model, seed, first, count):
    go, gm = eim.eim_sample_rrr(ctx, g, model, seed, first, count)
    ro, rm, _ = oracle.sample(off, nbr, model, seed, first, count, nthreads=NT)
    assert np.array_equal(go, ro), (model, first, count)
    assert np.array_equal(gm, rm), (model, first, count)
    return ro


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_sample_rrr_C1_all_ids(eim, ctx, graphs, model):
    off, nbr = graphs("C1")
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        for seed in (1, 2, 3):
            _sets_equal(eim, ctx, g, off, nbr, model, seed, 0, 30000)
        # ragged tails, far ids, composability
        _sets_equal(eim, ctx, g, off, nbr, model, 1, 2**40 + 17, 1)
        _sets_equal(eim, ctx, g, off, nbr, model, 1, 2**61, 777)
        a = eim.eim_sample_rrr(ctx, g, model, 5, 100, 33)
        b = eim.eim_sample_rrr(ctx, g, model, 5, 133, 90)
        c = eim.eim_sample_rrr(ctx, g, model, 5, 100, 123)
        assert np.array_equal(np.concatenate([a[1], b[1]]), c[1])
        o, m = eim.eim_sample_rrr(ctx, g, model, 5, 0, 0)
        assert o.tolist() == [0] and m.size == 0
    finally:
        eim.eim_graph_free(g)


# Split modes of the IC sampler (sample.cu): default threshold; a 64-entry
# ring that splits its backlog into 32-vertex tasks after every batch; no
# splits, a 32-entry ring whose overflow leaves as one-vertex tasks; the
# un-hoisted Philox path.
SPILL_MODES = {"default": {}, "spill_all": {"EIM_SPILL_QUADS": "1", "EIM_TASK_QUADS": "1", "EIM_RING_W": "64"},
               "ring32": {"EIM_SPILL_QUADS": "0", "EIM_RING_W": "32"},
               # general Philox path (the hoisted edge draws need quad ids < 2^32)
               "nohoist": {"EIM_NO_HOIST": "1"},
               # probe-first rounds: nearly every root traversal is suspended into tasks;
               # and the id-order policy without probing
               "probe": {"EIM_PROBE_QUADS": "2"}, "noprobe": {"EIM_PROBE_QUADS": "0", "EIM_NO_PREPASS": "1"},
               # the chunked argmax of the greedy for every candidate count, 8 per chunk
               "chunked": {"EIM_GREEDY_CHUNK_MIN": "0", "EIM_GREEDY_CHUNK_SHIFT": "3"}}


@pytest.fixture(params=list(SPILL_MODES))
def spill_mode(request, monkeypatch):
    for k, v in SPILL_MODES[request.param].items():
        monkeypatch.setenv(k, v)
    return request.param


def test_spill_modes_C1(eim, ctx, graphs, spill_mode):
    off, nbr = graphs("C1")
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        _sets_equal(eim, ctx, g, off, nbr, "IC", 4, 0, 20000)
        st = eim.eim_get_stats(ctx)
        if spill_mode == "spill_all":
            assert st["spilled_samples"] > 0, st["spilled_samples"]
        _sets_equal(eim, ctx, g, off, nbr, "IC", 4, 2**50 + 3, 333)
        _imm_equal(eim, ctx, g, off, nbr, 20, 0.3, 1.0, "IC", 4)
    finally:
        eim.eim_graph_free(g)


@pytest.mark.parametrize("model", ["IC", "LT"])
@pytest.mark.parametrize("shape", ["empty", "path", "star", "cycle", "bigcycle", "longpath", "rmat_dense"])
def test_sample_rrr_special_graphs(eim, ctx, model, shape, spill_mode):
    # bigcycle (every set = V, 3000 > the shared-memory ring) and longpath
    # spill to the shared queue; rmat_dense has heavy rows and many live edges.
    off, nbr = {
        "empty": lambda: inputs.empty_graph(100),
        "path": lambda: inputs.path_graph(50),
        "star": lambda: inputs.star_out(70),
        "cycle": lambda: inputs.cycle_graph(40),
        "bigcycle": lambda: inputs.cycle_graph(3000),
        "longpath": lambda: inputs.path_graph(5000),
        "rmat_dense": lambda: inputs.rmat(600, 60000, seed=4),
    }[shape]()
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        _sets_equal(eim, ctx, g, off, nbr, model, 9, 0, 700)
    finally:
        eim.eim_graph_free(g)


@pytest.mark.parametrize("mode", ["-", "chunk2", "chunk5"])
def test_select_seeds_on_oracle_arenas(eim, ctx, graphs, mode, monkeypatch):
    if mode.startswith("chunk"):  # chunked argmax with 4 / 32 candidates per chunk
        monkeypatch.setenv("EIM_GREEDY_CHUNK_MIN", "0")
        monkeypatch.setenv("EIM_GREEDY_CHUNK_SHIFT", mode[5:])
    rng = np.random.default_rng(0)
    for trial in range(30):
        n = int(rng.integers(2, 300))
        num = int(rng.integers(0, 500))
        lens = rng.integers(1, min(n, 12) + 1, size=num)
        offs = np.zeros(num + 1, dtype=np.uint64)
        offs[1:] = np.cumsum(lens)
        mem = np.concatenate([rng.choice(n, size=int(L), replace=False) for L in lens]).astype(np.uint32) \
            if num else np.zeros(0, dtype=np.uint32)
        k = int(rng.integers(1, n + 1))
        s, gn = eim.eim_select_seeds(ctx, n, offs, mem, k)
        rs, rg, _ = oracle.greedy(n, offs, mem, k)
        assert np.array_equal(s, rs) and np.array_equal(gn, rg), trial
    off, nbr = graphs("C1")
    ro, rm, _ = oracle.sample(off, nbr, "IC", 3, 0, 5000, nthreads=NT)
    s, gn = eim.eim_select_seeds(ctx, 1024, ro, rm, 40)
    rs, rg, _ = oracle.greedy(1024, ro, rm, 40)
    assert np.array_equal(s, rs) and np.array_equal(gn, rg)


def _imm_equal(eim, ctx, g, off, nbr, k, eps, ell, model, seed):
    seeds, theta, spread, st = eim.eim_imm_run(ctx, g, k, eps, ell, model, seed)
    ref = oracle.imm(off, nbr, k, eps, ell, model, seed, nthreads=NT)
    assert np.array_equal(seeds, ref["seeds"]), (model, seed)
    assert theta == ref["theta"]
    assert spread == ref["spread"]
    assert st["theta_i"] == ref["theta_i"] and st["cov_i"] == ref["cov_i"]
    assert st["lb"] == ref["lb"] and st["cov"] == ref["cov"]
    assert st["lambda_p"] == ref["lambda_p"] and st["lambda_s"] == ref["lambda_s"]
    assert st["edges_examined"] == ref["edges_examined"]
    assert st["arena_elems"] == ref["arena_elems"]
    return st


@pytest.mark.parametrize("model", ["IC", "LT"])
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_imm_C1(eim, ctx, graphs, model, seed):
    off, nbr = graphs("C1")
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        for k, eps in ((5, 0.5), (1, 0.9), (50, 0.2), (1024, 0.5)):
            _imm_equal(eim, ctx, g, off, nbr, k, eps, 1.0, model, seed)
    finally:
        eim.eim_graph_free(g)


def test_imm_degenerate_graphs(eim, ctx):
    for off, nbr in (inputs.empty_graph(64), inputs.path_graph(32), inputs.cycle_graph(700), inputs.star_out(90)):
        g = eim.eim_load_graph_csr(ctx, off, nbr)
        try:
            for model in ("IC", "LT"):
                _imm_equal(eim, ctx, g, off, nbr, 3, 0.5, 1.0, model, 7)
        finally:
            eim.eim_graph_free(g)


def test_invalid_graphs_rejected(eim, ctx):
    off, nbr = inputs.path_graph(10)
    bad_nbr = nbr.copy()
    bad_nbr[3] = 10
    bad_off = off.copy()
    bad_off[4], bad_off[5] = bad_off[5], bad_off[4]
    for o, m in ((off, bad_nbr), (bad_off, nbr)):
        with pytest.raises(eim.EimError) as ei:
            eim.eim_load_graph_csr(ctx, o, m)
        assert ei.value.status == eim.EIM_E_INVAL
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    with pytest.raises(eim.EimError):
        eim.eim_imm_run(ctx, g, 0, 0.5, 1.0, "IC", 1)
    with pytest.raises(eim.EimError):
        eim.eim_imm_run(ctx, g, 3, 1.5, 1.0, "IC", 1)
    eim.eim_graph_free(g)
    assert eim.lib().eim_graph_free(g) == eim.EIM_E_STATE


# ---------------------------------------------------------------- full size
def _coverage_equal(eim, ctx, n, ro, rm):
    """C after the last eim_imm_run == the oracle's counts over the same R."""
    C = eim.eim_get_coverage(ctx, n)
    assert np.array_equal(C, oracle.coverage(n, ro, rm))
    return C


def _exhaustive(eim, ctx, g, off, nbr, model, seed, theta, chunk=1 << 15):
    """Every set of ids [0, theta) against the oracle (in chunks); returns the oracle arena."""
    ro_all, rm_all = [np.zeros(1, dtype=np.uint64)], []
    base = 0
    for first in range(0, theta, chunk):
        cnt = min(chunk, theta - first)
        ro = _sets_equal(eim, ctx, g, off, nbr, model, seed, first, cnt)
        ro_all.append(ro[1:] + np.uint64(base))
        base += int(ro[-1])
    ro = np.concatenate(ro_all)
    rm = oracle.sample(off, nbr, model, seed, 0, theta, nthreads=NT)[1]
    assert int(ro[-1]) == rm.size
    return ro, rm


def test_C2_sets_exhaustive_coverage_and_imm(eim, ctx, graphs, monkeypatch):
    # every RRR set of the IMM's R (ids [0, theta) = [0, 101294)), the
    # per-vertex coverage counts C and the full IMM (the bench workload)
    c = inputs.CONFIGS["C2"]
    off, nbr = graphs("C2")
    n = off.size - 1
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        st = _imm_equal(eim, ctx, g, off, nbr, c["k"], c["eps"], c["ell"], "IC", 1)
        assert st["theta"] == 101294
        C_gpu = eim.eim_get_coverage(ctx, n)
        ro, rm = _exhaustive(eim, ctx, g, off, nbr, "IC", 1, st["theta"])
        assert np.array_equal(C_gpu, oracle.coverage(n, ro, rm))
        assert int(C_gpu.sum()) == st["arena_elems"]
        with monkeypatch.context() as mp:
            mp.setenv("EIM_SPILL_QUADS", "1")
            mp.setenv("EIM_TASK_QUADS", "1")
            _sets_equal(eim, ctx, g, off, nbr, "IC", 1, 98765, 1500)
            assert eim.eim_get_stats(ctx)["spilled_samples"] > 0
        with monkeypatch.context() as mp:  # ring overflow: one-vertex tasks
            mp.setenv("EIM_SPILL_QUADS", "0")
            mp.setenv("EIM_RING_W", "32")
            _sets_equal(eim, ctx, g, off, nbr, "IC", 1, 5555, 1000)
            assert eim.eim_get_stats(ctx)["spilled_samples"] > 0
    finally:
        eim.eim_graph_free(g)


def test_C3_sets_exhaustive_coverage_and_imm(eim, ctx, graphs, monkeypatch):
    c = inputs.CONFIGS["C3"]
    off, nbr = graphs("C3")
    n = off.size - 1
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        for env in ({"EIM_GREEDY_CHUNK_MIN": "0"},):  # the chunked argmax on a full-size selection
            with monkeypatch.context() as mp:
                for kk, vv in env.items():
                    mp.setenv(kk, vv)
                _imm_equal(eim, ctx, g, off, nbr, c["k"], c["eps"], c["ell"], "LT", 1)
        st = _imm_equal(eim, ctx, g, off, nbr, c["k"], c["eps"], c["ell"], "LT", 1)
        assert st["theta"] == 58277
        C_gpu = eim.eim_get_coverage(ctx, n)
        ro, rm = _exhaustive(eim, ctx, g, off, nbr, "LT", 1, st["theta"])
        assert np.array_equal(C_gpu, oracle.coverage(n, ro, rm))
    finally:
        eim.eim_graph_free(g)


def test_C4_sets_and_imm(eim, ctx, graphs):
    # Twitter-shaped (1.47e9 edges, max in-degree ~4e5): the full IMM against
    # one full oracle IMM, the largest sets of R and a random id sample set by
    # set, and C over a 20,000-id prefix (the IMM's full C needs every set).
    c = inputs.CONFIGS["C4"]
    off, nbr = graphs("C4")
    n = off.size - 1
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        st = _imm_equal(eim, ctx, g, off, nbr, c["k"], c["eps"], c["ell"], "IC", 1)
        go, gm = eim.eim_sample_rrr(ctx, g, "IC", 1, 0, 20000)
        ro, rm, _ = oracle.sample(off, nbr, "IC", 1, 0, 20000, nthreads=NT)
        assert np.array_equal(go, ro) and np.array_equal(gm, rm)
        sizes = np.diff(ro)
        big = np.argsort(-sizes.astype(np.int64), kind="stable")[:200]
        rng = np.random.default_rng(4)
        for s in sorted(set(big.tolist()) | set(rng.integers(20000, st["theta"], size=300).tolist())):
            _sets_equal(eim, ctx, g, off, nbr, "IC", 1, int(s), 1)
        s, gains = eim.eim_select_seeds(ctx, n, ro, rm, c["k"])
        rs, rg, _ = oracle.greedy(n, ro, rm, c["k"])
        assert np.array_equal(s, rs) and np.array_equal(gains, rg)
        _coverage_equal(eim, ctx, n, ro, rm)
    finally:
        eim.eim_graph_free(g)


# The martingale loop's stop test, LB and theta against their closed forms
# (tests/test_oracle_imm.py: one vertex in every RRR set => cov_i = |R|),
# evaluated in mpmath -- independent of the oracle.
@pytest.mark.parametrize("shape", ["path", "star", "cycle"])
def test_imm_stop_test_closed_form_gpu(eim, ctx, shape):
    from test_oracle_imm import ALL_COVERED_CASES, ALL_COVERED_GRAPHS, closed_form_all_covered
    for n, k, eps, ell in ALL_COVERED_CASES:
        off, nbr = ALL_COVERED_GRAPHS[shape](n)
        want = closed_form_all_covered(n, k, eps, ell)
        g = eim.eim_load_graph_csr(ctx, off, nbr)
        try:
            for model in ("IC", "LT"):
                seeds, theta, spread, st = eim.eim_imm_run(ctx, g, k, eps, ell, model, 11)
                assert st["theta_i"] == want["theta_i"] and st["cov_i"] == want["theta_i"], (n, k, eps)
                if want["lb"] is None:
                    assert st["lb"] == 1.0
                else:
                    assert abs(st["lb"] - float(want["lb"])) <= 1e-12 * float(want["lb"])
                assert theta == want["theta"] and st["cov"] == theta and spread == float(n)
                assert seeds.tolist() == list(range(k))
                C = eim.eim_get_coverage(ctx, n)
                if shape == "cycle":
                    assert np.array_equal(C, np.full(n, theta))
                else:
                    assert C[0] == theta
        finally:
            eim.eim_graph_free(g)


def test_coverage_counts_C1_and_select(eim, ctx, graphs):
    off, nbr = graphs("C1")
    n = off.size - 1
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        for model in ("IC", "LT"):
            for seed in (1, 2):
                _, theta, _, _ = eim.eim_imm_run(ctx, g, 5, 0.5, 1.0, model, seed)
                ro, rm, _ = oracle.sample(off, nbr, model, seed, 0, theta, nthreads=NT)
                _coverage_equal(eim, ctx, n, ro, rm)
            _, theta, _, _ = eim.eim_imm_run(ctx, g, 5, 0.5, 1.0, model, 3, flags=oracle.FRESH_FINAL)
            ro, rm, _ = oracle.sample(off, nbr, model, 3, oracle.FRESH_BASE, theta, nthreads=NT)
            _coverage_equal(eim, ctx, n, ro, rm)
        eim.eim_sample_rrr(ctx, g, "IC", 1, 0, 10)
        with pytest.raises(eim.EimError) as ei:
            eim.eim_get_coverage(ctx, n)
        assert ei.value.status == eim.EIM_E_STATE
        ro, rm, _ = oracle.sample(off, nbr, "IC", 3, 0, 3000, nthreads=NT)
        eim.eim_select_seeds(ctx, n, ro, rm, 7)
        _coverage_equal(eim, ctx, n, ro, rm)
        with pytest.raises(eim.EimError) as ei:
            eim.eim_get_coverage(ctx, n + 1)
        assert ei.value.status == eim.EIM_E_INVAL
    finally:
        eim.eim_graph_free(g)


# ---------------------------------------------------------------- NEXT rows
# NEXT-1 source elimination (R22), NEXT-4 fresh final phase (R23): same bar.
ELIM, FRESH = oracle.SOURCE_ELIM, oracle.FRESH_FINAL
assert (ELIM, FRESH) == (1, 2)  # == EIM_F_SOURCE_ELIM, EIM_F_FRESH_FINAL


def _imm_equal_flags(eim, ctx, g, off, nbr, k, eps, ell, model, seed, flags):
    seeds, theta, spread, st = eim.eim_imm_run(ctx, g, k, eps, ell, model, seed, flags=flags)
    ref = oracle.imm(off, nbr, k, eps, ell, model, seed, nthreads=NT, flags=flags)
    assert np.array_equal(seeds, ref["seeds"]), (model, seed, flags)
    for key in ("theta_i", "cov_i", "lb", "cov", "edges_examined", "arena_elems", "ids_sampled"):
        assert st[key] == ref[key], (key, st[key], ref[key])
    assert theta == ref["theta"] and spread == ref["spread"]
    return st


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_sample_rrr_source_elim(eim, ctx, graphs, model, spill_mode):
    off, nbr = graphs("C1")
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        for first, count in ((0, 20000), (2**45 + 5, 301), (oracle.FRESH_BASE, 999)):
            go, gm = eim.eim_sample_rrr(ctx, g, model, 6, first, count, flags=ELIM)
            ro, rm, _ = oracle.sample(off, nbr, model, 6, first, count, nthreads=NT, flags=ELIM)
            assert np.array_equal(go, ro) and np.array_equal(gm, rm), (first, count)
            assert eim.eim_get_stats(ctx)["edges_examined"] == oracle.sample(
                off, nbr, model, 6, first, count, nthreads=NT)[2]
    finally:
        eim.eim_graph_free(g)


@pytest.mark.parametrize("model", ["IC", "LT"])
@pytest.mark.parametrize("flags", [ELIM, FRESH, ELIM | FRESH])
def test_imm_flags_C1(eim, ctx, graphs, model, flags):
    off, nbr = graphs("C1")
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        for seed in (1, 2, 3):
            for k, eps in ((5, 0.5), (50, 0.2), (1024, 0.5)):
                _imm_equal_flags(eim, ctx, g, off, nbr, k, eps, 1.0, model, seed, flags)
    finally:
        eim.eim_graph_free(g)


def test_imm_flags_special_graphs(eim, ctx):
    for off, nbr in (inputs.path_graph(32), inputs.cycle_graph(700), inputs.star_out(90),
                     inputs.from_edges(6, [(0, 0), (4, 5)])):
        g = eim.eim_load_graph_csr(ctx, off, nbr)
        try:
            for model in ("IC", "LT"):
                for flags in (ELIM, FRESH | ELIM):
                    _imm_equal_flags(eim, ctx, g, off, nbr, 3, 0.5, 1.0, model, 7, flags)
        finally:
            eim.eim_graph_free(g)
    for off, nbr in (inputs.empty_graph(64), inputs.from_edges(4, [(0, 0), (2, 2)])):
        g = eim.eim_load_graph_csr(ctx, off, nbr)
        try:
            with pytest.raises(eim.EimError) as ei:
                eim.eim_imm_run(ctx, g, 1, 0.5, 1.0, "IC", 1, flags=ELIM)
            assert ei.value.status == eim.EIM_E_INVAL
            _imm_equal_flags(eim, ctx, g, off, nbr, 2, 0.5, 1.0, "IC", 1, FRESH)
        finally:
            eim.eim_graph_free(g)


@pytest.mark.parametrize("flags", [ELIM, FRESH | ELIM])
def test_C2_imm_flags(eim, ctx, graphs, flags):
    c = inputs.CONFIGS["C2"]
    off, nbr = graphs("C2")
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        go, gm = eim.eim_sample_rrr(ctx, g, "IC", 1, 0, 2000, flags=ELIM)
        ro, rm, _ = oracle.sample(off, nbr, "IC", 1, 0, 2000, nthreads=NT, flags=ELIM)
        assert np.array_equal(go, ro) and np.array_equal(gm, rm)
        st = _imm_equal_flags(eim, ctx, g, off, nbr, c["k"], c["eps"], c["ell"], "IC", 1, flags)
        assert st["ids_sampled"] > st["theta"]
    finally:
        eim.eim_graph_free(g)


def test_C3_imm_source_elim(eim, ctx, graphs):
    c = inputs.CONFIGS["C3"]
    off, nbr = graphs("C3")
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        _imm_equal_flags(eim, ctx, g, off, nbr, c["k"], c["eps"], c["ell"], "LT", 1, ELIM)
    finally:
        eim.eim_graph_free(g)


# NEXT-2: log-encoded graph store (R24).  Results must equal the plain store's
# oracle outputs; the store's size must equal the containers R24 defines.
LOGENC = 1  # EIM_G_LOG_ENCODE


def _packed_bytes(off, nbr):
    n, m = off.size - 1, nbr.size
    boff = oracle.log_bits(m)
    bnbr = oracle.log_bits(int(nbr.max()) if m else 0)
    return 4 * ((((n + 1) * boff + 31) // 32 + 2) + ((m * bnbr + 31) // 32 + 2))


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_log_encoded_graph_C1(eim, ctx, graphs, model, spill_mode):
    off, nbr = graphs("C1")
    g = eim.eim_load_graph_csr(ctx, off, nbr, gflags=LOGENC)
    try:
        assert eim.eim_graph_bytes(g) == _packed_bytes(off, nbr)
        _sets_equal(eim, ctx, g, off, nbr, model, 2, 0, 20000)
        _sets_equal(eim, ctx, g, off, nbr, model, 2, 2**50 + 9, 500)
        _imm_equal(eim, ctx, g, off, nbr, 20, 0.3, 1.0, model, 4)
        _imm_equal_flags(eim, ctx, g, off, nbr, 5, 0.5, 1.0, model, 4, ELIM | FRESH)
    finally:
        eim.eim_graph_free(g)


def test_log_encoded_special_graphs(eim, ctx):
    for off, nbr in (inputs.empty_graph(64), inputs.path_graph(32), inputs.cycle_graph(3000), inputs.star_out(90),
                     inputs.from_edges(3, [(0, 1), (0, 2)]), inputs.rmat(600, 60000, seed=4)):
        g = eim.eim_load_graph_csr(ctx, off, nbr, gflags=LOGENC)
        try:
            assert eim.eim_graph_bytes(g) == _packed_bytes(off, nbr)
            for model in ("IC", "LT"):
                _sets_equal(eim, ctx, g, off, nbr, model, 9, 0, 700)
                _imm_equal(eim, ctx, g, off, nbr, 3, 0.5, 1.0, model, 7)
        finally:
            eim.eim_graph_free(g)


def test_log_encoded_C2_imm(eim, ctx, graphs):
    c = inputs.CONFIGS["C2"]
    off, nbr = graphs("C2")
    g = eim.eim_load_graph_csr(ctx, off, nbr, gflags=LOGENC)
    try:
        packed = eim.eim_graph_bytes(g)
        assert packed == _packed_bytes(off, nbr)
        assert packed < 0.7 * (8 * off.size + 4 * nbr.size + 4 * (off.size - 1))
        _sets_equal(eim, ctx, g, off, nbr, "IC", 1, 0, 2000)
        _imm_equal(eim, ctx, g, off, nbr, c["k"], c["eps"], c["ell"], "IC", 1)
    finally:
        eim.eim_graph_free(g)


# NEXT-3: general edge probabilities (R25), thresholds streamed per edge.
def _random_x(off, model, seed, frac_sum=0.9):
    """Random per-edge x: IC p uniform in (0, 1]; LT a random split of mass <= 1 per row."""
    rng = np.random.default_rng(seed)
    m = int(off[-1])
    if model == "IC":
        return rng.integers(0, 2**32, size=m, dtype=np.uint64).astype(np.uint32)
    d = np.diff(off).astype(np.int64)
    row = np.repeat(np.arange(d.size), d)
    r = rng.random(m) + 1e-3
    rowsum = np.bincount(row, weights=r, minlength=d.size)
    total = np.where(np.arange(d.size) % 3 != 0, np.floor(frac_sum * 2**32), 2.0**32)
    w = np.floor(r / rowsum[row] * (total[row] - d[row])).astype(np.int64) + 1   # row sum <= total
    x = (w - 1).astype(np.uint32)
    return x


def _weighted_equal(eim, ctx, off, nbr, x, model, seed, first, count, imm_args=None):
    g = eim.eim_load_graph_csr(ctx, off, nbr, edge_x=x)
    try:
        go, gm = eim.eim_sample_rrr(ctx, g, model, seed, first, count)
        ro, rm, rex = oracle.sample(off, nbr, model, seed, first, count, nthreads=NT, x=x)
        assert np.array_equal(go, ro) and np.array_equal(gm, rm), (model, first, count)
        assert eim.eim_get_stats(ctx)["edges_examined"] == rex
        if imm_args:
            k, eps, flags = imm_args
            seeds, theta, spread, st = eim.eim_imm_run(ctx, g, k, eps, 1.0, model, seed, flags=flags)
            ref = oracle.imm(off, nbr, k, eps, 1.0, model, seed, nthreads=NT, flags=flags, x=x)
            assert np.array_equal(seeds, ref["seeds"]) and theta == ref["theta"] and spread == ref["spread"]
            for key in ("theta_i", "cov_i", "edges_examined", "arena_elems", "ids_sampled"):
                assert st[key] == ref[key], key
    finally:
        eim.eim_graph_free(g)


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_weighted_C1(eim, ctx, graphs, model, spill_mode):
    off, nbr = graphs("C1")
    for seed in (1, 2):
        x = _random_x(off, model, seed)
        if model == "IC":
            x = (x >> np.uint32(4)).astype(np.uint32)  # p ~ U(0, 1/16): sets of moderate size
        _weighted_equal(eim, ctx, off, nbr, x, model, seed, 0, 6000, (5, 0.5, 0))
    _weighted_equal(eim, ctx, off, nbr, _random_x(off, model, 3) >> np.uint32(5), model, 3, 2**44 + 1, 333,
                    (3, 0.3, ELIM))


def test_weighted_special_cases(eim, ctx):
    # p = 1 on a path: every set is a prefix; WC-derived weights on C1 reproduce the WC sets
    off, nbr = inputs.path_graph(300)
    x = np.full(nbr.size, 2**32 - 1, dtype=np.uint32)
    for model in ("IC", "LT"):
        _weighted_equal(eim, ctx, off, nbr, x, model, 4, 0, 500, (2, 0.5, 0))
    off, nbr = inputs.config_graph("C1")
    d = np.diff(off).astype(np.uint64)
    row = np.repeat(np.arange(off.size - 1), d.astype(np.int64))
    x_ic = (np.uint64(2**32 - 1) // d[row]).astype(np.uint32)
    g = eim.eim_load_graph_csr(ctx, off, nbr, edge_x=x_ic)
    try:
        a = eim.eim_sample_rrr(ctx, g, "IC", 5, 0, 4000)
        b = oracle.sample(off, nbr, "IC", 5, 0, 4000, nthreads=NT)
        assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    finally:
        eim.eim_graph_free(g)
    # LT weights summing above 1 are rejected for LT, accepted for IC
    off, nbr = inputs.from_edges(3, [(0, 2), (1, 2)])
    g = eim.eim_load_graph_csr(ctx, off, nbr, edge_x=np.array([2**31, 2**31 - 1], dtype=np.uint32))
    try:
        with pytest.raises(eim.EimError) as ei:
            eim.eim_imm_run(ctx, g, 1, 0.5, 1.0, "LT", 1)
        assert ei.value.status == eim.EIM_E_INVAL
        eim.eim_imm_run(ctx, g, 1, 0.5, 1.0, "IC", 1)
    finally:
        eim.eim_graph_free(g)
    # the packed weighted store (NEXT-2 x NEXT-3) keeps the LT rejection
    g = eim.eim_load_graph_csr(ctx, off, nbr, gflags=LOGENC, edge_x=np.array([2**31, 2**31 - 1], dtype=np.uint32))
    try:
        with pytest.raises(eim.EimError) as ei:
            eim.eim_imm_run(ctx, g, 1, 0.5, 1.0, "LT", 1)
        assert ei.value.status == eim.EIM_E_INVAL
    finally:
        eim.eim_graph_free(g)


# NEXT-2 x NEXT-3: log-encoded offsets/neighbours with per-edge probabilities
# ("applied to both the network data and the RRR sets").
@pytest.mark.parametrize("model", ["IC", "LT"])
def test_weighted_log_encoded(eim, ctx, graphs, model, spill_mode):
    off, nbr = graphs("C1")
    x = _random_x(off, model, 11)
    if model == "IC":
        x = (x >> np.uint32(4)).astype(np.uint32)
    g = eim.eim_load_graph_csr(ctx, off, nbr, gflags=LOGENC, edge_x=x)
    try:
        m = nbr.size
        assert eim.eim_graph_bytes(g) == _packed_bytes(off, nbr) + 4 * ((m + 3) // 4 * 4 + 4) + 4 * max(m, 1)
        go, gm = eim.eim_sample_rrr(ctx, g, model, 2, 0, 6000)
        ro, rm, rex = oracle.sample(off, nbr, model, 2, 0, 6000, nthreads=NT, x=x)
        assert np.array_equal(go, ro) and np.array_equal(gm, rm)
        assert eim.eim_get_stats(ctx)["edges_examined"] == rex
        for flags in (0, ELIM | FRESH):
            seeds, theta, spread, st = eim.eim_imm_run(ctx, g, 5, 0.5, 1.0, model, 2, flags=flags)
            ref = oracle.imm(off, nbr, 5, 0.5, 1.0, model, 2, nthreads=NT, flags=flags, x=x)
            assert np.array_equal(seeds, ref["seeds"]) and theta == ref["theta"] and spread == ref["spread"]
            for key in ("theta_i", "cov_i", "edges_examined", "arena_elems", "ids_sampled"):
                assert st[key] == ref[key], key
    finally:
        eim.eim_graph_free(g)


@pytest.mark.parametrize("model", ["IC", "LT"])
def test_weighted_C2(eim, ctx, graphs, model):
    off, nbr = graphs("C2")
    x = _random_x(off, model, 7)
    if model == "IC":  # trivalency-like small probabilities keep the sets moderate
        x = (x >> np.uint32(6)).astype(np.uint32)
    _weighted_equal(eim, ctx, off, nbr, x, model, 1, 0, 3000 if model == "IC" else 20000)


def test_task_pool_layout_change_between_rounds(eim, ctx, graphs, monkeypatch):
    # Regression: a round with a smaller task pool than the previous one (same
    # buffer) must not read the previous pool's seed ids as task descriptors.
    off, nbr = graphs("C2")
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        with monkeypatch.context() as mp:
            mp.setenv("EIM_TABLE_BITS", "26")
            mp.setenv("EIM_SPILL_QUADS", "1")
            mp.setenv("EIM_TASK_QUADS", "1")
            _sets_equal(eim, ctx, g, off, nbr, "IC", 1, 0, 3000)
        with monkeypatch.context() as mp:
            mp.setenv("EIM_SPILL_QUADS", "1")
            mp.setenv("EIM_TASK_QUADS", "1")
            _sets_equal(eim, ctx, g, off, nbr, "IC", 1, 7000, 2000)
        _sets_equal(eim, ctx, g, off, nbr, "IC", 1, 20000, 1000)
    finally:
        eim.eim_graph_free(g)


# LT walk store (lt_aug_kernel, default on the plain store) and the
# row-offset walk (lt_kernel, EIM_NO_LT_AUG=1) against the oracle.  Cycles
# make every walk end at a revisit (the speculative insert past it is
# tombstoned), bigcycle gives 3000-step walks, the path graph ends walks at
# d = 0, dense R-MAT mixes both; the same graph object serves both switches.
@pytest.mark.parametrize("store", ["walk_store", "row_offsets"])
def test_lt_walk_store_vs_row_offsets(eim, ctx, graphs, store, monkeypatch):
    if store == "row_offsets":
        monkeypatch.setenv("EIM_NO_LT_AUG", "1")
    cases = [inputs.cycle_graph(40), inputs.cycle_graph(3000), inputs.path_graph(500),
             inputs.rmat(600, 60000, seed=4), graphs("C1")]
    for off, nbr in cases:
        g = eim.eim_load_graph_csr(ctx, off, nbr)
        try:
            _sets_equal(eim, ctx, g, off, nbr, "LT", 5, 0, 1500)
            _sets_equal(eim, ctx, g, off, nbr, "LT", 5, 2**40 + 7, 257)
        finally:
            eim.eim_graph_free(g)


# Ranges above the membership-table budget are sampled in several launches
# (ADVICE r1): forced tiny launches give the same sets and IMM results.
@pytest.mark.parametrize("model", ["IC", "LT"])
def test_launches_split_by_table_budget(eim, ctx, graphs, model, monkeypatch):
    off, nbr = graphs("C1")
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    try:
        monkeypatch.setenv("EIM_MAX_LAUNCH_IDS", "777")
        _sets_equal(eim, ctx, g, off, nbr, model, 3, 5, 5000)
        assert eim.eim_get_stats(ctx)["sample_launches"] >= 7
        for flags in (0, ELIM, FRESH):
            _imm_equal_flags(eim, ctx, g, off, nbr, 10, 0.3, 1.0, model, 2, flags)
    finally:
        eim.eim_graph_free(g)


def test_select_seeds_rejects_duplicates(eim, ctx):
    offs = np.array([0, 3, 5], dtype=np.uint64)
    with pytest.raises(eim.EimError) as ei:
        eim.eim_select_seeds(ctx, 10, offs, np.array([1, 2, 1, 4, 5], dtype=np.uint32), 2)
    assert ei.value.status == eim.EIM_E_INVAL
    # the same member in two different sets is fine
    s, gn = eim.eim_select_seeds(ctx, 10, offs, np.array([1, 2, 3, 1, 5], dtype=np.uint32), 2)
    assert s.tolist() == [1, 0] and gn.tolist() == [2, 0]  # all covered after the first pick: lowest id (R10)
