"""Development probe: one heavy C2 sample alone on the GPU vs inside its round
(EIM_DEBUG_TIMELINE per-batch phase times), with and without splitting."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["EIM_DEBUG_TIMELINE"] = "1"
import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

off, nbr = inputs.config_graph("C2")
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
ids = [int(x) for x in (sys.argv[1:] or ["321", "1302", "198"])]
for spill in ("8192", "0"):
    os.environ["EIM_SPILL_QUADS"] = spill
    for s in ids:
        for rep in range(2):
            print(f"--- spill={spill} sample {s} rep {rep}", file=sys.stderr, flush=True)
            eim.eim_sample_rrr(ctx, g, "IC", 1, s, 1)
    print(f"--- spill={spill} round ids [0, 6331)", file=sys.stderr, flush=True)
    eim.eim_sample_rrr(ctx, g, "IC", 1, 0, 6331)
