"""Sweep-only probe (libeim.so built with -DEIM_SWEEP_BENCH): ns per batch and
quads/ns of one group (and of a full grid) over a staged batch of rows."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

L = eim.lib()
f = L.eim_dev_sweep_bench
f.argtypes = [ctypes.c_int, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.POINTER(ctypes.c_double),
              ctypes.POINTER(ctypes.c_double)]
tag = sys.argv[1] if len(sys.argv) > 1 else ""
for blocks in (1, 148 * 4):
    for nrows, d in ((10, 2300), (1, 23000), (100, 230), (256, 40)):
        ns, q = ctypes.c_double(), ctypes.c_double()
        rc = f(blocks, nrows, d, 200, ctypes.byref(ns), ctypes.byref(q))
        print(f"{tag} blocks={blocks} rows={nrows} d={d} ns/batch={ns.value:.0f} quads/ns={q.value:.2f} rc={rc}")
