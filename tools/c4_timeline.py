import os, sys
sys.path.insert(0, os.getcwd())
import inputs, paper_conf_sc_doneyhl25_b200 as eim
c = inputs.CONFIGS["C4"]
off, nbr = inputs.config_graph("C4")
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)
os.environ["EIM_DEBUG_TIMELINE"] = "1"
s, th, sp, st = eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)
print("C4 imm", st["ms_total"], st["ms_sample_kernel"], flush=True)
import numpy as np
print("max in-degree", int(np.diff(off).max()), "rows > 100K:", int((np.diff(off) > 100000).sum()))
