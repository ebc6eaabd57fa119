"""Host timeline of one IMM (EIM_TRACE=1): library stamps after each host
synchronisation (sampler launch done, append read-back, selections enqueued
and collected), in ms since the call started; two warm-up runs first.
    python tools/trace_imm.py CFG"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

cfg = sys.argv[1]
c = inputs.CONFIGS[cfg]
off, nbr = inputs.config_graph(cfg)
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
for i in range(3):
    if i == 2:
        os.environ["EIM_TRACE"] = "1"  # read by the library at the start of each IMM
    s = eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)[3]
    print("run", i, s["ms_total"], s["ms_sample_kernel"], s["ms_select"], file=sys.stderr)
