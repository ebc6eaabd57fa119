"""ctypes wrapper of the CPU oracle (eim_oracle.c).

TEST INFRASTRUCTURE ONLY: importable from tests/, __graft_entry__.smoke()
and bench.py's cpu_baseline / --impl reference legs.  The product package
(paper_conf_sc_doneyhl25_b200) never imports this module.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "eim_oracle.c")
_HDR = os.path.join(_HERE, "eim_oracle.h")

IC, LT = 0, 1
# run flags (eim_oracle.h): source-vertex elimination (NEXT-1), fresh final phase (NEXT-4)
SOURCE_ELIM, FRESH_FINAL = 1, 2
FRESH_BASE = 1 << 61
MODELS = {"IC": IC, "LT": LT, IC: IC, LT: LT}

# -ffp-contract=off / no fast-math: the theta schedule must be evaluated as written.
CFLAGS = ["-O2", "-std=c11", "-fPIC", "-shared", "-pthread", "-ffp-contract=off", "-fno-fast-math"]


def build(force: bool = False) -> str:
    newest = max(os.path.getmtime(_SRC), os.path.getmtime(_HDR))
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < newest:
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", _SO, "-lm"])
    return _SO


class _Arena(ctypes.Structure):
    _fields_ = [
        ("num_sets", ctypes.c_uint64),
        ("total", ctypes.c_uint64),
        ("offsets", ctypes.POINTER(ctypes.c_uint64)),
        ("members", ctypes.POINTER(ctypes.c_uint32)),
        ("edges_examined", ctypes.c_uint64),
        ("set_edges", ctypes.POINTER(ctypes.c_uint64)),
    ]


class Params(ctypes.Structure):
    _fields_ = [(f, ctypes.c_double) for f in ("ell_p", "eps_p", "lnC", "lambda_p", "lambda_s", "log2n")]


class ImmStats(ctypes.Structure):
    _fields_ = [
        ("rounds", ctypes.c_uint32),
        ("theta_i", ctypes.c_uint64 * 64),
        ("cov_i", ctypes.c_uint64 * 64),
        ("lambda_p", ctypes.c_double),
        ("lambda_s", ctypes.c_double),
        ("lb", ctypes.c_double),
        ("theta", ctypes.c_uint64),
        ("cov", ctypes.c_uint64),
        ("edges_examined", ctypes.c_uint64),
        ("arena_elems", ctypes.c_uint64),
        ("ids_sampled", ctypes.c_uint64),
    ]


_lib = None
P = ctypes.c_void_p
U32, U64, I32, D = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int, ctypes.c_double


def _load():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        sig = {
            "orc_philox4x32_10": (None, [P, P, P]),
            "orc_draw": (U32, [U64, U64, U32, U64, U32]),
            "orc_edge_draw": (U32, [U64, U64, U64]),
            "orc_lt_draw": (U32, [U64, U64, U32]),
            "orc_root": (U32, [U64, U64, U32]),
            "orc_ic_live": (I32, [U32, U64]),
            "orc_lt_choice": (U32, [U32, U64]),
            "orc_rrr_set": (U32, [U32, P, P, I32, U64, U64, P, P]),
            "orc_sample": (ctypes.POINTER(_Arena), [U32, P, P, I32, U64, U64, U64, I32]),
            "orc_sample_ex": (ctypes.POINTER(_Arena), [U32, P, P, I32, U64, U64, U64, U32, I32]),
            "orc_arena_free": (None, [ctypes.POINTER(_Arena)]),
            "orc_greedy": (U64, [U32, U64, P, P, U32, P, P]),
            "orc_coverage": (None, [U32, U64, P, P, P]),
            "orc_imm_params": (I32, [U32, U32, D, D, ctypes.POINTER(Params)]),
            "orc_imm": (I32, [U32, P, P, U32, D, D, I32, U64, I32, P, P, P, ctypes.POINTER(ImmStats)]),
            "orc_imm_ex": (I32, [U32, P, P, U32, D, D, I32, U64, U32, I32, P, P, P, ctypes.POINTER(ImmStats)]),
            "orc_ic_live_w": (I32, [U32, U32]),
            "orc_lt_choice_w": (U32, [U32, P, U64]),
            "orc_lt_weights_ok": (I32, [U32, P, P]),
            "orc_sample_w": (ctypes.POINTER(_Arena), [U32, P, P, P, I32, U64, U64, U64, U32, I32]),
            "orc_imm_w": (I32, [U32, P, P, P, U32, D, D, I32, U64, U32, I32, P, P, P, ctypes.POINTER(ImmStats)]),
            "orc_log_bits": (U32, [U64]),
            "orc_log_words": (U64, [U64, U32]),
            "orc_log_encode": (None, [P, U64, U32, P]),
            "orc_log_decode": (U64, [P, U64, U32]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data


def philox4x32_10(ctr, key):
    L = _load()
    c = np.asarray(ctr, dtype=np.uint32)
    k = np.asarray(key, dtype=np.uint32)
    out = np.zeros(4, dtype=np.uint32)
    L.orc_philox4x32_10(_ptr(c), _ptr(k), _ptr(out))
    return out


def draw(seed, s, tag, q, word):
    return int(_load().orc_draw(seed, s, tag, q, word))


def edge_draw(seed, s, e):
    return int(_load().orc_edge_draw(seed, s, e))


def lt_draw(seed, s, u):
    return int(_load().orc_lt_draw(seed, s, u))


def root(seed, s, n):
    return int(_load().orc_root(seed, s, n))


def ic_live(draw_, d):
    return bool(_load().orc_ic_live(draw_, d))


def lt_choice(tau, d):
    return int(_load().orc_lt_choice(tau, d))


def _graph(off, nbr):
    off = np.ascontiguousarray(off, dtype=np.uint64)
    nbr = np.ascontiguousarray(nbr, dtype=np.uint32)
    if nbr.size == 0:
        nbr = np.zeros(1, dtype=np.uint32)
    return off, nbr


def rrr_set(off, nbr, model, seed, s):
    off, nbr = _graph(off, nbr)
    n = off.size - 1
    out = np.zeros(n, dtype=np.uint32)
    stamp = np.zeros(n, dtype=np.uint64)
    sz = _load().orc_rrr_set(n, _ptr(off), _ptr(nbr), MODELS[model], seed, s, _ptr(out), _ptr(stamp))
    return out[:sz].copy()


def sample(off, nbr, model, seed, first, count, nthreads=1, flags=0, per_set_edges=False, x=None):
    """Returns (offsets u64[count+1], members u32[total], edges_examined)
    (edges_examined as u64[count], one per set, when per_set_edges).
    x: per-edge u32 probabilities p_e = (x_e + 1) / 2^32 (NEXT-3), None = WC."""
    off, nbr = _graph(off, nbr)
    n = off.size - 1
    L = _load()
    if x is not None:
        xa = _weights(x, nbr)
        a = L.orc_sample_w(n, _ptr(off), _ptr(nbr), _ptr(xa), MODELS[model], seed, first, count, flags, nthreads)
    elif flags:
        a = L.orc_sample_ex(n, _ptr(off), _ptr(nbr), MODELS[model], seed, first, count, flags, nthreads)
    else:
        a = L.orc_sample(n, _ptr(off), _ptr(nbr), MODELS[model], seed, first, count, nthreads)
    A = a.contents
    offsets = np.ctypeslib.as_array(A.offsets, shape=(count + 1,)).copy()
    members = (np.ctypeslib.as_array(A.members, shape=(A.total,)).copy()
               if A.total else np.zeros(0, dtype=np.uint32))
    if per_set_edges:
        ex = (np.ctypeslib.as_array(A.set_edges, shape=(count,)).copy()
              if count else np.zeros(0, dtype=np.uint64))
    else:
        ex = int(A.edges_examined)
    L.orc_arena_free(a)
    return offsets, members, ex


def greedy(n, offsets, members, k):
    """Returns (seeds u32[k], gains u64[k], cov)."""
    offsets = np.ascontiguousarray(offsets, dtype=np.uint64)
    members = np.ascontiguousarray(members, dtype=np.uint32)
    if members.size == 0:
        members = np.zeros(1, dtype=np.uint32)
    seeds = np.zeros(k, dtype=np.uint32)
    gains = np.zeros(k, dtype=np.uint64)
    cov = _load().orc_greedy(n, offsets.size - 1, _ptr(offsets), _ptr(members), k, _ptr(seeds), _ptr(gains))
    return seeds, gains, int(cov)


def coverage(n, offsets, members):
    """C u32[n]: number of sets containing each vertex."""
    offsets = np.ascontiguousarray(offsets, dtype=np.uint64)
    members = np.ascontiguousarray(members, dtype=np.uint32)
    if members.size == 0:
        members = np.zeros(1, dtype=np.uint32)
    C = np.zeros(n, dtype=np.uint32)
    _load().orc_coverage(n, offsets.size - 1, _ptr(offsets), _ptr(members), _ptr(C))
    return C


def imm_params(n, k, eps, ell):
    p = Params()
    rc = _load().orc_imm_params(n, k, eps, ell, ctypes.byref(p))
    if rc != 0:
        raise ValueError("invalid IMM parameters")
    return p


def _weights(x, nbr):
    xa = np.ascontiguousarray(x, dtype=np.uint32)
    return xa if xa.size else np.zeros(1, dtype=np.uint32)


def ic_live_w(draw_, x):
    return bool(_load().orc_ic_live_w(draw_, x))


def lt_choice_w(tau, x_row):
    """First j with sum_{i<=j}(x_i + 1) > tau, or None."""
    xr = np.ascontiguousarray(x_row, dtype=np.uint32)
    j = int(_load().orc_lt_choice_w(tau, _ptr(xr) if xr.size else None, xr.size))
    return None if j == 0xFFFFFFFF else j


def lt_weights_ok(off, x):
    off = np.ascontiguousarray(off, dtype=np.uint64)
    xa = np.ascontiguousarray(x, dtype=np.uint32)
    return bool(_load().orc_lt_weights_ok(off.size - 1, _ptr(off), _ptr(xa) if xa.size else None))


def imm(off, nbr, k, eps, ell, model, seed, nthreads=1, flags=0, x=None):
    """Returns dict(seeds, theta, spread, stats).  flags: SOURCE_ELIM | FRESH_FINAL.
    x: per-edge probabilities (NEXT-3), None = WC."""
    off, nbr = _graph(off, nbr)
    n = off.size - 1
    seeds = np.zeros(k, dtype=np.uint32)
    theta = ctypes.c_uint64()
    spread = ctypes.c_double()
    st = ImmStats()
    xa = _weights(x, nbr) if x is not None else None
    rc = _load().orc_imm_w(n, _ptr(off), _ptr(nbr), _ptr(xa) if xa is not None else None, k, eps, ell,
                           MODELS[model], seed, flags, nthreads,
                           _ptr(seeds), ctypes.addressof(theta), ctypes.addressof(spread), ctypes.byref(st))
    if rc != 0:
        raise RuntimeError(f"orc_imm failed rc={rc}")
    rounds = min(st.rounds, 64)
    return dict(
        seeds=seeds, theta=int(theta.value), spread=float(spread.value),
        rounds=int(st.rounds), theta_i=[int(x) for x in st.theta_i[:rounds]],
        cov_i=[int(x) for x in st.cov_i[:rounds]], lambda_p=st.lambda_p, lambda_s=st.lambda_s,
        lb=st.lb, cov=int(st.cov), edges_examined=int(st.edges_examined),
        arena_elems=int(st.arena_elems), ids_sampled=int(st.ids_sampled),
    )


def log_bits(x_max):
    return int(_load().orc_log_bits(int(x_max)))


def log_encode(x, b=None):
    """Log-encode (bit-pack) x: returns (u32 containers, n_b)."""
    x = np.ascontiguousarray(x, dtype=np.uint64)
    if b is None:
        b = log_bits(int(x.max()) if x.size else 0)
    L = _load()
    nw = int(L.orc_log_words(x.size, b))
    w = np.zeros(max(nw, 1), dtype=np.uint32)
    L.orc_log_encode(_ptr(x) if x.size else None, x.size, b, _ptr(w))
    return w[:nw], b


def log_decode(words, count, b):
    words = np.ascontiguousarray(words, dtype=np.uint32)
    if words.size == 0:
        words = np.zeros(1, dtype=np.uint32)
    L = _load()
    return np.array([L.orc_log_decode(_ptr(words), j, b) for j in range(count)], dtype=np.uint64)
