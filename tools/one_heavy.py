"""ncu target: heavy C2 sample 1302 alone (no splitting), after a warm-up."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["EIM_SPILL_QUADS"] = "0"
import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

off, nbr = inputs.config_graph("C2")
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
for rep in range(2):
    eim.eim_sample_rrr(ctx, g, "IC", 1, int(sys.argv[1]) if len(sys.argv) > 1 else 1302, 1)
