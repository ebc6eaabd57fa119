"""Thin ctypes binding of libeim.so (include/eim.h): argument marshalling only.

Every step of the hot path runs in the library's CUDA kernels.  There is no
CPU fallback: importing this package on a machine without the built library
raises, and calls on a machine without a GPU fail with EIM_E_CUDA.
Names follow the C ABI.  Arrays are numpy (host) or integers (device
pointers, streams).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libeim.so")

EIM_OK, EIM_E_INVAL, EIM_E_NOMEM, EIM_E_CUDA, EIM_E_NCCL, EIM_E_CAPACITY, EIM_E_STATE = 0, -1, -2, -3, -4, -5, -6
EIM_IC, EIM_LT = 0, 1
MODELS = {"IC": EIM_IC, "LT": EIM_LT, EIM_IC: EIM_IC, EIM_LT: EIM_LT}
NCCL_ID_BYTES = 128
# run flags (include/eim.h)
EIM_F_SOURCE_ELIM, EIM_F_FRESH_FINAL = 1, 2
EIM_FRESH_BASE = 1 << 61
EIM_G_LOG_ENCODE = 1

STATUS_NAMES = {0: "EIM_OK", -1: "EIM_E_INVAL", -2: "EIM_E_NOMEM", -3: "EIM_E_CUDA", -4: "EIM_E_NCCL",
                -5: "EIM_E_CAPACITY", -6: "EIM_E_STATE"}

# Every symbol include/eim.h declares (checked by tests/test_abi.py).
EXPORTS = ["eim_create", "eim_create_group", "eim_nccl_get_id", "eim_destroy", "eim_last_error", "eim_version",
           "eim_load_graph_csr", "eim_load_graph_csr_ex", "eim_load_graph_csr_weighted", "eim_graph_bytes",
           "eim_graph_free", "eim_imm_run", "eim_imm_run_ex", "eim_sample_rrr",
           "eim_sample_rrr_ex", "eim_select_seeds",
           "eim_imm_params", "eim_shard_range", "eim_get_stats", "eim_get_coverage"]


class EimError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


class Stats(ctypes.Structure):
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
        ("spilled_samples", ctypes.c_uint64),
        ("kernel_launches", ctypes.c_uint64),
        ("sample_launches", ctypes.c_uint32),
        ("ms_total", ctypes.c_double),
        ("ms_sample", ctypes.c_double),
        ("ms_select", ctypes.c_double),
        ("ms_comm", ctypes.c_double),
        ("ms_sample_kernel", ctypes.c_double),
        ("ids_sampled", ctypes.c_uint64),
        ("arena_bytes", ctypes.c_uint64),
        ("ms_select_kernel", ctypes.c_double),
        ("select_launches", ctypes.c_uint32),
        ("select_picks", ctypes.c_uint64),
    ]

    def as_dict(self):
        r = int(min(self.rounds, 64))
        d = {f: getattr(self, f) for f, _ in self._fields_ if f not in ("theta_i", "cov_i")}
        d["theta_i"] = [int(x) for x in self.theta_i[:r]]
        d["cov_i"] = [int(x) for x in self.cov_i[:r]]
        return d


class ImmParams(ctypes.Structure):
    _fields_ = [(f, ctypes.c_double) for f in ("ell_p", "eps_p", "lnC", "lambda_p", "lambda_s", "log2n")]


_lib = None
_P = ctypes.c_void_p
_U32, _U64, _I, _D = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int, ctypes.c_double


def lib():
    """Load libeim.so (fails loudly if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = ctypes.CDLL(LIB_PATH)
    sig = {
        "eim_create": (_I, [_I, _I, _I, _P, _U64, ctypes.POINTER(_P)]),
        "eim_nccl_get_id": (_I, [_P]),
        "eim_create_group": (_I, [_P, _I, _P]),
        "eim_destroy": (None, [_P]),
        "eim_last_error": (ctypes.c_char_p, [_P]),
        "eim_version": (ctypes.c_char_p, []),
        "eim_load_graph_csr": (_I, [_P, _U32, _U64, _P, _P, ctypes.POINTER(_P)]),
        "eim_graph_free": (_I, [_P]),
        "eim_load_graph_csr_ex": (_I, [_P, _U32, _U64, _P, _P, _U32, ctypes.POINTER(_P)]),
        "eim_graph_bytes": (_I, [_P, ctypes.POINTER(_U64)]),
        "eim_load_graph_csr_weighted": (_I, [_P, _U32, _U64, _P, _P, _P, _U32, ctypes.POINTER(_P)]),
        "eim_imm_run": (_I, [_P, _P, _U32, _D, _D, _I, _U64, _P, _P, _P, _P]),
        "eim_imm_run_ex": (_I, [_P, _P, _U32, _D, _D, _I, _U64, _U32, _P, _P, _P, _P]),
        "eim_sample_rrr": (_I, [_P, _P, _I, _U64, _U64, _U64, _P, _P, _U64, _P]),
        "eim_sample_rrr_ex": (_I, [_P, _P, _I, _U64, _U64, _U64, _U32, _P, _P, _U64, _P]),
        "eim_select_seeds": (_I, [_P, _U32, _U64, _P, _P, _U32, _P, _P]),
        "eim_imm_params": (_I, [_U32, _U32, _D, _D, ctypes.POINTER(ImmParams)]),
        "eim_shard_range": (_I, [_U64, _U64, _I, _I, ctypes.POINTER(_U64), ctypes.POINTER(_U64)]),
        "eim_get_stats": (_I, [_P, _P]),
        "eim_get_coverage": (_I, [_P, _U32, _P]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


def _check(status, ctx=None):
    if status != EIM_OK:
        msg = lib().eim_last_error(ctx)
        raise EimError(status, (msg or b"").decode(errors="replace"))


def _host(a, dtype):
    a = np.ascontiguousarray(a, dtype=dtype)
    return a


# ------------------------------------------------------------------ context
def eim_version():
    return lib().eim_version().decode()


def eim_nccl_get_id() -> bytes:
    buf = ctypes.create_string_buffer(NCCL_ID_BYTES)
    _check(lib().eim_nccl_get_id(buf))
    return buf.raw


def eim_create(device=0, rank=0, world=1, nccl_id: bytes | None = None, stream: int = 0):
    out = _P()
    idbuf = ctypes.create_string_buffer(nccl_id, NCCL_ID_BYTES) if nccl_id is not None else None
    _check(lib().eim_create(device, rank, world, idbuf, stream, ctypes.byref(out)))
    return out.value


def eim_create_group(devices):
    """In-process ranks (one context per entry of devices; devices may repeat).
    Returns the list of contexts, rank order."""
    devs = np.ascontiguousarray(list(devices), dtype=np.int32)
    out = (_P * len(devs))()
    _check(lib().eim_create_group(devs.ctypes.data, len(devs), out))
    return [out[r] for r in range(len(devs))]


def eim_destroy(ctx):
    lib().eim_destroy(ctx)


def eim_last_error(ctx=None):
    return (lib().eim_last_error(ctx) or b"").decode()


# ------------------------------------------------------------------ graph
def eim_load_graph_csr(ctx, in_offsets, in_neighbors, gflags=0, edge_x=None):
    """in_offsets: u64[n+1] (numpy or pinned torch tensor .numpy()), in_neighbors: u32[m].
    gflags != 0 (EIM_G_LOG_ENCODE) calls eim_load_graph_csr_ex; edge_x (u32[m], p = (x+1)/2^32)
    calls eim_load_graph_csr_weighted."""
    off = _host(in_offsets, np.uint64)
    nbr = _host(in_neighbors, np.uint32)
    n = off.size - 1
    out = _P()
    args = (ctx, n, nbr.size, off.ctypes.data, nbr.ctypes.data if nbr.size else None)
    if edge_x is not None:
        x = _host(edge_x, np.uint32)
        if x.size != nbr.size:
            raise ValueError("edge_x must have one entry per edge")
        _check(lib().eim_load_graph_csr_weighted(*args, x.ctypes.data if x.size else None, gflags,
                                                 ctypes.byref(out)), ctx)
    elif gflags:
        _check(lib().eim_load_graph_csr_ex(*args, gflags, ctypes.byref(out)), ctx)
    else:
        _check(lib().eim_load_graph_csr(*args, ctypes.byref(out)), ctx)
    return out.value


def eim_graph_bytes(g):
    b = _U64()
    _check(lib().eim_graph_bytes(g, ctypes.byref(b)))
    return int(b.value)


def eim_load_graph_csr_ptr(ctx, n, m, off_ptr, nbr_ptr):
    """Same call with raw host pointers (e.g. pinned torch tensors)."""
    out = _P()
    _check(lib().eim_load_graph_csr(ctx, n, m, off_ptr, nbr_ptr, ctypes.byref(out)), ctx)
    return out.value


def eim_graph_free(g):
    _check(lib().eim_graph_free(g))


# ------------------------------------------------------------------ hot path
def eim_imm_run(ctx, g, k, eps, ell, model, seed, with_stats=True, flags=0):
    """Returns (seeds u32[k], theta, spread, stats dict or None).  flags != 0 calls eim_imm_run_ex."""
    seeds = np.zeros(k, dtype=np.uint32)
    theta = ctypes.c_uint64()
    spread = ctypes.c_double()
    st = Stats() if with_stats else None
    outs = (seeds.ctypes.data, ctypes.addressof(theta), ctypes.addressof(spread),
            ctypes.addressof(st) if st is not None else None)
    if flags:
        _check(lib().eim_imm_run_ex(ctx, g, k, eps, ell, MODELS[model], seed, flags, *outs), ctx)
    else:
        _check(lib().eim_imm_run(ctx, g, k, eps, ell, MODELS[model], seed, *outs), ctx)
    return seeds, int(theta.value), float(spread.value), (st.as_dict() if st is not None else None)


def eim_sample_rrr(ctx, g, model, seed, first_id, count, members_cap=None, flags=0):
    """Returns (offsets u64[count+1], members u32[total]); sets ascending, in sample-id order.
    flags != 0 (EIM_F_SOURCE_ELIM) calls eim_sample_rrr_ex."""
    offsets = np.zeros(count + 1, dtype=np.uint64)
    total = ctypes.c_uint64()
    cap = members_cap if members_cap is not None else max(16, count * 64)
    while True:
        members = np.zeros(max(cap, 1), dtype=np.uint32)
        outs = (offsets.ctypes.data, members.ctypes.data, cap, ctypes.addressof(total))
        if flags:
            s = lib().eim_sample_rrr_ex(ctx, g, MODELS[model], seed, first_id, count, flags, *outs)
        else:
            s = lib().eim_sample_rrr(ctx, g, MODELS[model], seed, first_id, count, *outs)
        if s == EIM_E_CAPACITY and members_cap is None:
            cap = int(total.value)
            continue
        _check(s, ctx)
        return offsets, members[: int(total.value)]


def eim_sample_rrr_stats(ctx, g, model, seed, first_id, count, flags=0):
    """Samples ids [first_id, first_id+count) and returns the call's stats
    only (the members stay on the device: members_cap 0 => EIM_E_CAPACITY
    after the sampling, which is the expected outcome here)."""
    offsets = np.zeros(count + 1, dtype=np.uint64)
    total = ctypes.c_uint64()
    s = lib().eim_sample_rrr_ex(ctx, g, MODELS[model], seed, first_id, count, flags, offsets.ctypes.data, None, 0,
                                ctypes.addressof(total))
    if s not in (EIM_OK, EIM_E_CAPACITY):
        _check(s, ctx)
    return eim_get_stats(ctx)


def eim_select_seeds(ctx, n, offsets, members, k):
    """Returns (seeds u32[k], gains u64[k])."""
    off = _host(offsets, np.uint64)
    mem = _host(members, np.uint32)
    seeds = np.zeros(k, dtype=np.uint32)
    gains = np.zeros(k, dtype=np.uint64)
    _check(lib().eim_select_seeds(ctx, n, off.size - 1, off.ctypes.data, mem.ctypes.data if mem.size else None, k,
                                  seeds.ctypes.data, gains.ctypes.data), ctx)
    return seeds, gains


def eim_get_stats(ctx):
    st = Stats()
    _check(lib().eim_get_stats(ctx, ctypes.addressof(st)), ctx)
    return st.as_dict()


def eim_get_coverage(ctx, n):
    """Coverage counts C u32[n] of the R of the last eim_imm_run / eim_select_seeds."""
    C = np.zeros(n, dtype=np.uint32)
    _check(lib().eim_get_coverage(ctx, n, C.ctypes.data), ctx)
    return C


# ------------------------------------------------------------------ host-only
def eim_imm_params(n, k, eps, ell):
    p = ImmParams()
    _check(lib().eim_imm_params(n, k, eps, ell, ctypes.byref(p)))
    return p


def eim_shard_range(first, count, rank, world):
    lo, hi = _U64(), _U64()
    _check(lib().eim_shard_range(first, count, rank, world, ctypes.byref(lo), ctypes.byref(hi)))
    return int(lo.value), int(hi.value)
