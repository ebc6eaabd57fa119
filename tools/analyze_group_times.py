"""Summarise the group sampler's EIM_DEBUG_TIMES records:
per sample (t_begin, t_end, batches, stage_ns, sweep_ns, quads)."""
import sys
import numpy as np

data = open(sys.argv[1], "rb").read()
pos = 0
while pos < len(data):
    first, count = (int(x) for x in np.frombuffer(data, dtype=np.uint64, count=2, offset=pos))
    pos += 16
    rec = np.frombuffer(data, dtype=np.uint64, count=6 * count, offset=pos).reshape(-1, 6).astype(np.int64)
    pos += 48 * count
    ok = rec[:, 1] > 0
    t0 = rec[ok, 0].min()
    dur = (rec[:, 1] - rec[:, 0]) / 1e3
    print(f"launch first={first} count={count}: span {(rec[ok,1].max()-t0)/1e3:.0f} us")
    for i in np.argsort(-dur)[:6]:
        b = max(rec[i, 2], 1)
        print(f"   s={first+i} start={(rec[i,0]-t0)/1e3:7.1f} dur={dur[i]:8.1f}us batches={rec[i,2]:4d} "
              f"stage/b={rec[i,3]/b/1e3:6.2f}us sweep/b={rec[i,4]/b/1e3:6.2f}us quads/b={rec[i,5]/b:8.0f}")
