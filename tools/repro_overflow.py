"""Table-overflow redo path: sample ids with a forced tiny membership table
(EIM_TABLE_BITS) and compare with the oracle.  Usage: python tools/repro_overflow.py CFG BITS COUNT"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import inputs  # noqa: E402
import oracle  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

cfg, bits, count = sys.argv[1], sys.argv[2], int(sys.argv[3])
os.environ["EIM_TABLE_BITS"] = bits
off, nbr = inputs.config_graph(cfg)
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
for first in (0, 5000):
    go, gm = eim.eim_sample_rrr(ctx, g, "IC", 1, first, count)
    ro, rm, _ = oracle.sample(off, nbr, "IC", 1, first, count, nthreads=16)
    print(cfg, bits, first, count, "equal", np.array_equal(go, ro) and np.array_equal(gm, rm),
          "max set", int(np.diff(ro).max()), flush=True)
