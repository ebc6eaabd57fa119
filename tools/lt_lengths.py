import sys, os, numpy as np
sys.path.insert(0, os.getcwd())
import inputs, paper_conf_sc_doneyhl25_b200 as eim
off, nbr = inputs.config_graph("C3")
ctx = eim.eim_create(0); g = eim.eim_load_graph_csr(ctx, off, nbr)
o, m = eim.eim_sample_rrr(ctx, g, "LT", 1, 0, 58277)
L = np.diff(o.astype(np.int64))
print("mean", L.mean(), "max", L.max(), "p99", np.percentile(L, 99), "p999", np.percentile(L, 99.9), "top", np.sort(L)[-10:])
deg = np.diff(off.astype(np.int64))
print("max indeg", deg.max(), "n0", (deg==0).mean())
