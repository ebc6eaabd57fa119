"""IMM wall and sampler time on a large IC config (graph generated here).
    python tools/ab_c4.py [CFG]"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
c = inputs.CONFIGS[cfg]
t = time.time()
off, nbr = inputs.config_graph(cfg)
print("gen", time.time() - t, flush=True)
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
for rep in range(3):
    seeds, theta, spread, st = eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)
    print(f"{cfg} rep={rep} imm_ms={st['ms_total']:9.2f} sample_ms={st['ms_sample']:9.2f} "
          f"kernel_ms={st['ms_sample_kernel']:9.2f} select_ms={st['ms_select']:7.2f} theta={theta} "
          f"edges={st['edges_examined']} Gedge/s={st['edges_examined'] / st['ms_sample_kernel'] / 1e6:7.1f}", flush=True)
