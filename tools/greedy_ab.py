"""A/B of the greedy argmax shortlist (EIM_GREEDY_NO_SHORTLIST) on a config:
IMM seconds and select ms per IMM, results checked identical.
    python tools/greedy_ab.py [CFG] [REPS]"""
import os
import statistics
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 8
c = inputs.CONFIGS[cfg]
off, nbr = inputs.config_graph(cfg)
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
res = {}
for mode in ("shortlist", "full", "shortlist", "full"):
    if mode == "full":
        os.environ["EIM_GREEDY_NO_SHORTLIST"] = "1"
    else:
        os.environ.pop("EIM_GREEDY_NO_SHORTLIST", None)
    sel, tot = [], []
    for _ in range(reps):
        seeds, theta, spread, st = eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)
        sel.append(st["ms_select"])
        tot.append(st["ms_total"])
    res.setdefault(mode, []).append((statistics.median(sel), statistics.median(tot), seeds.tolist(), theta))
    print(cfg, mode, "select ms", statistics.median(sel), "total ms", statistics.median(tot), "theta", theta,
          "rounds", st["rounds"], flush=True)
assert res["shortlist"][0][2] == res["full"][0][2], "seeds differ"
print("seeds identical")
