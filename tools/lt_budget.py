"""LT sampler alone on a fixed budget of sample ids (profiling target).
    python tools/lt_budget.py [CFG] [IDS]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
ids = int(sys.argv[2]) if len(sys.argv) > 2 else 1 << 20
off, nbr = inputs.config_graph(cfg)
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
for _ in range(2):
    eim.eim_sample_rrr(ctx, g, "LT", 1, 0, ids)
    st = eim.eim_get_stats(ctx)
    print(cfg, "LT ids", ids, "steps", st["edges_examined"], "kernel_ms", st["ms_sample_kernel"],
          "steps/s", st["edges_examined"] / st["ms_sample_kernel"] * 1e3, flush=True)
