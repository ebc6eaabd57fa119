"""Seeded synthetic inputs shared by the oracle and the CUDA path.

This module holds NO arithmetic of the eIM method: it only produces graphs
(reverse CSR: in_off[n+1] u64, in_nbr[m] u32, rows ascending) and the
benchmark configuration table.  Recipe: DESIGN.md §5.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "librmat.so")
_SRC = os.path.join(_HERE, "rmat.c")

# Graph500 R-MAT parameters (a, b, c); d = 1 - a - b - c.
GRAPH500 = (0.57, 0.19, 0.19)

# BASELINE.json configs[0..4] realised as R-MAT graphs with the SNAP n, m.
CONFIGS = {
    "C1": dict(name="rmat-s10", n=1024, m=16384, model="IC", k=5, eps=0.5, ell=1.0),
    "C2": dict(name="livejournal-shaped", n=4847571, m=68993773, model="IC", k=50, eps=0.5, ell=1.0),
    "C3": dict(name="orkut-shaped", n=3072441, m=117185083, model="LT", k=100, eps=0.3, ell=1.0),
    "C4": dict(name="twitter-shaped", n=41652230, m=1468365182, model="IC", k=50, eps=0.5, ell=1.0),
    "C5": dict(name="friendster-shaped", n=65608366, m=1806067135, model="IC", k=200, eps=0.1, ell=1.0),
}


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-pthread", _SRC, "-o", _SO, "-lm"]
        )
    return _SO


_lib = None


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        lib.rmat_generate.restype = ctypes.c_int
        lib.rmat_generate.argtypes = [
            ctypes.c_uint32, ctypes.c_uint64, ctypes.c_double, ctypes.c_double, ctypes.c_double,
            ctypes.c_uint64, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
        ]
        _lib = lib
    return _lib


def rmat(n: int, m: int, seed: int = 1, abc=GRAPH500, nthreads: int | None = None):
    """Deterministic R-MAT graph as reverse CSR (in_off u64[n+1], in_nbr u32[m])."""
    lib = _load()
    if nthreads is None:
        nthreads = max(1, min(64, os.cpu_count() or 1))
    off = np.zeros(n + 1, dtype=np.uint64)
    nbr = np.zeros(max(m, 1), dtype=np.uint32)
    rc = lib.rmat_generate(n, m, abc[0], abc[1], abc[2], seed, nthreads,
                           off.ctypes.data, nbr.ctypes.data)
    if rc != 0:
        raise RuntimeError(f"rmat_generate failed (n={n}, m={m})")
    return off, nbr[:m]


def config_graph(name: str, seed: int = 1):
    c = CONFIGS[name]
    return rmat(c["n"], c["m"], seed=seed)


def from_edges(n: int, edges):
    """Reverse CSR from a list of directed edges (u -> v): row v lists in-neighbours u ascending."""
    edges = sorted((int(v), int(u)) for (u, v) in edges)
    off = np.zeros(n + 1, dtype=np.uint64)
    nbr = np.zeros(len(edges), dtype=np.uint32)
    for i, (v, u) in enumerate(edges):
        off[v + 1] += 1
        nbr[i] = u
    off = np.cumsum(off, dtype=np.uint64)
    return off, nbr


def path_graph(n: int):
    """0 -> 1 -> ... -> n-1 (in-degree 1 everywhere but vertex 0)."""
    return from_edges(n, [(i, i + 1) for i in range(n - 1)])


def star_out(n: int):
    """hub 0 -> every leaf 1..n-1."""
    return from_edges(n, [(0, i) for i in range(1, n)])


def cycle_graph(n: int):
    return from_edges(n, [(i, (i + 1) % n) for i in range(n)])


def empty_graph(n: int):
    return np.zeros(n + 1, dtype=np.uint64), np.zeros(0, dtype=np.uint32)


def random_small_graph(n: int, m: int, seed: int):
    """Uniform simple digraph with exactly m edges (for enumeration pins)."""
    rng = np.random.default_rng(seed)
    allp = [(u, v) for u in range(n) for v in range(n) if u != v]
    pick = rng.choice(len(allp), size=m, replace=False)
    return from_edges(n, [allp[i] for i in pick])
