"""One warm-up IMM + one profiled IMM on a config (for ncu: -k regex:ic_kernel -s <launches of one IMM>)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C2"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
c = inputs.CONFIGS[name]
off, nbr = inputs.config_graph(name)
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
for rep in range(reps):
    seeds, theta, spread, st = eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)
    print(rep, theta, st["sample_launches"], round(st["ms_sample_kernel"], 3), round(st["ms_select"], 3),
          round(st["ms_total"], 3), flush=True)
eim.eim_graph_free(g)
eim.eim_destroy(ctx)
