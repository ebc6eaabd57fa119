"""Per-pick phase times of the greedy pick kernel (EIM_DEBUG_GREEDY timers,
record-index kernel greedy2_kernel): argmax + first barrier, cover, second
barrier (block 0's stamps), and the spread of the blocks' arrivals at each
barrier (first to last arrival = how long the barrier waits for the slowest
block), per NodeSelection of slot 0.
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
raw = np.fromfile(path, dtype=np.uint64).astype(np.int64)
pos, r = 0, 0
while pos < len(raw):
    k, nb, pp = int(raw[pos]), int(raw[pos + 1]), int(raw[pos + 2])
    pos += 3
    b = raw[pos:pos + 3 * k].reshape(k, 3)
    pos += 3 * k
    arr = raw[pos:pos + pp * k * nb].reshape(k, pp, nb)
    pos += pp * k * nb
    arg = (b[:, 1] - b[:, 0]) / 1e3
    cov = (b[:, 2] - b[:, 1]) / 1e3
    nxt = (b[1:, 0] - b[:-1, 2]) / 1e3
    s1 = (arr[:, 0].max(1) - arr[:, 0].min(1)) / 1e3   # argmax arrivals spread
    s2 = (arr[:, 1].max(1) - arr[:, 1].min(1)) / 1e3   # cover arrivals spread
    l1 = (b[:, 1] - arr[:, 0].max(1)) / 1e3            # last arrival -> block 0 leaves barrier 1
    l2 = (b[1:, 0] - arr[:-1, 1].max(1)) / 1e3          # last arrival -> block 0 leaves barrier 2
    print(f"{cfg} selection {r} ({nb} blocks): {k} picks in {(b[-1, 2] - b[0, 0]) / 1e3:.1f} us = "
          f"{(b[-1, 2] - b[0, 0]) / 1e3 / k:.2f} us/pick | argmax+B1 med {np.median(arg):.2f} | "
          f"cover med {np.median(cov):.2f} (first {cov[0]:.2f}) | B2 med {np.median(nxt) if len(nxt) else 0:.2f} | "
          f"arrival spread B1 med {np.median(s1):.2f} B2 med {np.median(s2):.2f} | "
          f"last-arrival->exit B1 med {np.median(l1):.2f} B2 med {np.median(l2) if len(l2) else 0:.2f} us")
    if pp == 4:  # per block: B2 exit -> scan done, and the spread of the B2 exits
        sc = (arr[:, 3] - arr[:, 2]) / 1e3
        ex = (arr[:, 2].max(1) - arr[:, 2].min(1)) / 1e3
        print(f"    per-block scan med {np.median(sc):.2f} max-over-blocks med {np.median(sc.max(1)):.2f} | "
              f"B2-exit spread med {np.median(ex):.2f} | scan-done -> B1 arrival med {np.median((arr[:, 0] - arr[:, 3]) / 1e3):.2f} us")
    r += 1
