"""Per-round sampler timeline (EIM_DEBUG_TIMELINE=1): time until every id is
taken vs the tail until the last task ends, for one IMM run on a config."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["EIM_DEBUG_TIMELINE"] = "1"
import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C2"
c = inputs.CONFIGS[name]
off, nbr = inputs.config_graph(name)
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
for rep in range(2):
    print("run", rep, file=sys.stderr)
    seeds, theta, spread, st = eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)
    print(theta, st["ms_sample_kernel"], st["ms_total"], file=sys.stderr)
