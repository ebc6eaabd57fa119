"""A/B of an environment switch of the sampler on a config: median IMM and
sampler-kernel ms over REPS runs for each setting, results identical.
    python tools/ab_env.py CFG REPS VAR VALUE1 VALUE2 ...   (VALUE '-' = unset)"""
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

cfg, reps, var, values = sys.argv[1], int(sys.argv[2]), sys.argv[3], sys.argv[4:]
c = inputs.CONFIGS[cfg]
off, nbr = inputs.config_graph(cfg)
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
ref = None
for val in values * 2:
    if val == "-":
        os.environ.pop(var, None)
    else:
        os.environ[var] = val
    eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)
    tot, ker, sel = [], [], []
    for _ in range(reps):
        seeds, theta, spread, st = eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)
        tot.append(st["ms_total"])
        ker.append(st["ms_sample_kernel"])
        sel.append(st["ms_select"])
    ref = ref or seeds.tolist()
    assert seeds.tolist() == ref
    print(f"{cfg} {var}={val:>6s} imm_ms={statistics.median(tot):8.3f} sample_kernel_ms={statistics.median(ker):8.3f} "
          f"select_ms={statistics.median(sel):8.3f}",
          flush=True)
