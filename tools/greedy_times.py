"""Per-pick phase times of the greedy kernel (EIM_DEBUG_GREEDY timers): argmax
(to the first grid barrier), cover (to the second), per NodeSelection.
    python tools/greedy_times.py CFG"""
import os
import sys
import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

cfg = sys.argv[1]
c = inputs.CONFIGS[cfg]
off, nbr = inputs.config_graph(cfg)
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)
path = "/tmp/greedy_dbg.bin"
if os.path.exists(path):
    os.remove(path)
os.environ["EIM_DEBUG_GREEDY"] = path
eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)
t = np.fromfile(path, dtype=np.uint64).astype(np.int64).reshape(-1, 3)
k = c["k"]
for r in range(len(t) // k):
    b = t[r * k:(r + 1) * k]
    arg = (b[:, 1] - b[:, 0]) / 1e3
    cov = (b[:, 2] - b[:, 1]) / 1e3
    nxt = (b[1:, 0] - b[:-1, 2]) / 1e3
    print(f"{cfg} selection {r}: picks {k} total {(b[-1, 2] - b[0, 0]) / 1e3:.1f} us; argmax+sync median {np.median(arg):.2f} "
          f"max {arg.max():.2f}; cover median {np.median(cov):.2f} max {cov.max():.2f} (first {cov[0]:.2f}); "
          f"second sync median {np.median(nxt) if len(nxt) else 0:.2f} us")
