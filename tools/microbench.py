"""Sampler / greedy micro-benchmarks on one GPU (development tool, not the bench).

    python tools/microbench.py [C2] [--variants fused,group]

Times eim_sample_rrr over IMM-round-shaped id ranges and a large fixed budget,
reporting the sampler's device time (CUDA events inside the library) and
examined edges per second."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 and not sys.argv[1].startswith("--") else "C2"
    variants = ["default"]
    for a in sys.argv:
        if a.startswith("--variants="):
            variants = a.split("=", 1)[1].split(",")
    c = inputs.CONFIGS[cfg]
    off, nbr = inputs.config_graph(cfg)
    ctx = eim.eim_create(0)
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    ranges = [(0, 6331), (6331, 6331), (12662, 12662), (25324, 25323), (50647, 50647), (0, 1 << 18)]
    out = {}
    for var in variants:
        if var != "default":
            os.environ["EIM_IC_KERNEL"] = var
        res = []
        eim.eim_sample_rrr(ctx, g, c["model"], 1, 0, 2000)  # warm-up
        for first, count in ranges:
            t0 = time.perf_counter()
            eim.eim_sample_rrr(ctx, g, c["model"], 1, first, count)
            wall = (time.perf_counter() - t0) * 1e3
            st = eim.eim_get_stats(ctx)
            res.append(dict(first=first, count=count, kernel_ms=round(st["ms_sample_kernel"], 3),
                            sample_ms=round(st["ms_sample"], 3), call_ms=round(wall, 2),
                            gedge_s=round(st["edges_examined"] / st["ms_sample_kernel"] / 1e6, 1),
                            edges=st["edges_examined"], spilled=st["spilled_samples"]))
        out[var] = res
        for r in res:
            print(var, json.dumps(r))
    eim.eim_graph_free(g)
    eim.eim_destroy(ctx)




def greedy_bench():
    """select_seeds on a GPU-sampled C2 arena of 101294 sets (the last IMM round)."""
    c = inputs.CONFIGS["C2"]
    off, nbr = inputs.config_graph("C2")
    ctx = eim.eim_create(0)
    g = eim.eim_load_graph_csr(ctx, off, nbr)
    o, m = eim.eim_sample_rrr(ctx, g, "IC", 1, 0, 101294)
    for _ in range(2):
        eim.eim_select_seeds(ctx, c["n"], o, m, c["k"])
    times = []
    for _ in range(5):
        eim.eim_select_seeds(ctx, c["n"], o, m, c["k"])
        times.append(eim.eim_get_stats(ctx)["ms_select"])
    print("greedy", json.dumps(dict(k=c["k"], sets=101294, members=int(m.size), ms=sorted(times))))


if __name__ == "__main__":
    if "--greedy" in sys.argv:
        greedy_bench()
    else:
        main()
