"""LT walk-step latency at C3: the longest walks of the bench round timed
alone (one walk per launch: unloaded latency per step) against the whole
round [0, theta_2) (the launch lasts as long as its longest walk).
    python tools/lt_step_latency.py"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

off, nbr = inputs.config_graph("C3")
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
N = 58277
o, _ = eim.eim_sample_rrr(ctx, g, "LT", 1, 0, N)
L = np.diff(o.astype(np.int64))
top = np.argsort(L)[::-1][:5]
for rep in range(3):
    st = eim.eim_sample_rrr_stats(ctx, g, "LT", 1, 0, N)
    print(f"round [0,{N}): kernel {st['ms_sample_kernel']:.3f} ms, longest walk {L.max()} members "
          f"-> {1e3 * st['ms_sample_kernel'] / L.max():.3f} us per step of the longest walk")
for s in top:
    ms = []
    for rep in range(5):
        st = eim.eim_sample_rrr_stats(ctx, g, "LT", 1, int(s), 1)
        ms.append(st["ms_sample_kernel"])
    m = float(np.median(ms))
    print(f"walk {s}: {L[s]} members alone: {m:.3f} ms = {1e3 * m / L[s]:.3f} us per step")
