"""Row-range task size sweep (EIM_ROW_TASK_QUADS) on an IC config: IMM time,
sampler kernel time, fixed-budget sampler rate; results checked identical.
    python tools/ab_rowsplit.py [CFG] [REPS]"""
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import inputs  # noqa: E402
import paper_conf_sc_doneyhl25_b200 as eim  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 6
c = inputs.CONFIGS[cfg]
off, nbr = inputs.config_graph(cfg)
ctx = eim.eim_create(0)
g = eim.eim_load_graph_csr(ctx, off, nbr)
ref = None
for rq in ("0", "8192", "4096", "2048", "1024", "512", "0", "2048"):
    os.environ["EIM_ROW_TASK_QUADS"] = rq
    eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)
    tot, ker = [], []
    for _ in range(reps):
        seeds, theta, spread, st = eim.eim_imm_run(ctx, g, c["k"], c["eps"], c["ell"], c["model"], 1)
        tot.append(st["ms_total"])
        ker.append(st["ms_sample_kernel"])
    if ref is None:
        ref = seeds.tolist()
    assert seeds.tolist() == ref
    eim.eim_sample_rrr(ctx, g, c["model"], 1, 0, 1 << 20)
    sb = eim.eim_get_stats(ctx)
    print(f"{cfg} row_quads={rq:>5s} imm_ms={statistics.median(tot):7.3f} sample_kernel_ms={statistics.median(ker):7.3f} "
          f"budget_kernel_ms={sb['ms_sample_kernel']:7.2f} budget_Gedge/s={sb['edges_examined'] / sb['ms_sample_kernel'] / 1e6:7.1f}",
          flush=True)
