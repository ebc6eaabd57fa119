import os, sys
sys.path.insert(0, os.getcwd())
import inputs, paper_conf_sc_doneyhl25_b200 as eim
cfg = sys.argv[1]
c = inputs.CONFIGS[cfg]
off, nbr = inputs.config_graph(cfg)
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
for i in range(3):
    if i == 2: os.environ["EIM_TRACE"] = "1"
    s = eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)[3]
    print("run", i, s["ms_total"], s["ms_sample_kernel"], s["ms_select"], file=sys.stderr)
