"""Multi-rank protocol of eim_imm_run on CPU (gloo, world size 2 and 3).

The library's N>1 path (imm.cpp sample_round) is: every round's new sample
ids [|R|, theta_i) are split with eim_shard_range (the library's own host
function, called here), each rank samples its share, the shares are
exchanged in rank order (= sample-id order) and the greedy runs replicated
(also with the fresh final phase, whose ids start at EIM_FRESH_BASE).
Here each rank samples with the oracle and exchanges over gloo; the result
must equal the single-process oracle IMM bit for bit on every rank.
"""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

import inputs
import oracle
import paper_conf_sc_doneyhl25_b200 as eim
from paper_conf_sc_doneyhl25_b200 import _build


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _dist_imm(rank, world, off, nbr, k, eps, ell, model, seed, fresh=False):
    """Mirror of imm.cpp's control flow with the exchange done over gloo.
    fresh: the final phase draws theta sets from ids FRESH_BASE.. (R23),
    sharded the same way (set index i = sample id FRESH_BASE + i)."""
    n = off.size - 1
    p = eim.eim_imm_params(n, k, eps, ell)
    offsets = [np.zeros(1, dtype=np.uint64)]
    members = []
    R, cov, total = 0, 0, 0
    LB = 1.0
    rounds = []
    id_base = 0

    def sample_round(R, R_new):
        nonlocal total
        lo, hi = eim.eim_shard_range(R, R_new - R, rank, world)
        o, m, _ = oracle.sample(off, nbr, model, seed, id_base + lo, hi - lo)
        gathered = [None] * world
        dist.all_gather_object(gathered, (lo, hi, o, m))
        for q in range(world):  # rank order == sample-id order
            lo_q, hi_q, o_q, m_q = gathered[q]
            assert lo_q == (R if q == 0 else gathered[q - 1][1])
            offsets.append(o_q[1:] + total)
            members.append(m_q)
            total += int(o_q[-1])
        assert gathered[-1][1] == R_new

    def select():
        O = np.concatenate(offsets)
        M = np.concatenate(members) if members else np.zeros(0, dtype=np.uint32)
        return oracle.greedy(n, O, M, k)

    i = 1
    S = None
    R_sel = None
    while i < p.log2n:
        th = int(np.ceil(np.ldexp(p.lambda_p, i) / n))
        if th > R:
            sample_round(R, th)
            R = th
        S, _, cov = select()
        R_sel = R
        rounds.append((R, cov))
        if cov * 2.0**i >= (1.0 + p.eps_p) * R:
            LB = (n * cov) / ((1.0 + p.eps_p) * R)
            break
        i += 1
    theta = int(np.ceil(p.lambda_s / LB))
    if fresh:
        offsets[:] = [np.zeros(1, dtype=np.uint64)]
        members.clear()
        total, R, R_sel, id_base = 0, 0, None, eim.EIM_FRESH_BASE
    if theta > R:
        sample_round(R, theta)
        R = theta
    if R != R_sel:
        S, _, cov = select()
    return S, R, n * cov / R, rounds


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        out = []
        off, nbr = inputs.config_graph("C1")
        for model in ("IC", "LT"):
            for seed in (1, 2):
                for fresh in (False, True):
                    S, theta, spread, rounds = _dist_imm(rank, world, off, nbr, 5, 0.5, 1.0, model, seed, fresh)
                    out.append((model, seed, fresh, S.tolist(), theta, spread, rounds))
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_multi_rank_protocol_matches_single_process(world):
    _build.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p_ in procs:
        p_.start()
    results = dict(q.get(timeout=300) for _ in range(world))
    for p_ in procs:
        p_.join(timeout=60)
        assert p_.exitcode == 0
    off, nbr = inputs.config_graph("C1")
    for r in range(world):
        for (model, seed, fresh, S, theta, spread, rounds) in results[r]:
            ref = oracle.imm(off, nbr, 5, 0.5, 1.0, model, seed, flags=oracle.FRESH_FINAL if fresh else 0)
            assert S == ref["seeds"].tolist(), (r, model, seed)
            assert theta == ref["theta"] and spread == ref["spread"]
            assert [x for x, _ in rounds] == ref["theta_i"] and [c for _, c in rounds] == ref["cov_i"]
