"""Summarise EIM_DEBUG_TIMES records (per-sample start/end ns, levels, edges)."""
import sys
import numpy as np

data = open(sys.argv[1], "rb").read()
pos = 0
while pos < len(data):
    first, count = (int(x) for x in np.frombuffer(data, dtype=np.uint64, count=2, offset=pos))
    pos += 16
    rec = np.frombuffer(data, dtype=np.uint64, count=4 * int(count), offset=pos).reshape(-1, 4)
    pos += 32 * int(count)
    st, en, lev = rec[:, 0].astype(np.int64), rec[:, 1].astype(np.int64), rec[:, 2].astype(np.int64)
    edges = (rec[:, 3] >> np.uint64(20)).astype(np.int64)
    ok = en > 0
    t0 = st[ok].min()
    span = (en[ok].max() - t0) / 1e3
    dur = (en - st) / 1e3
    print(f"launch first={first} count={count}: span {span:.0f} us, done {ok.sum()}")
    idx = np.argsort(-dur)[:8]
    for i in idx:
        print(f"   s={first + i:8d} start={(st[i]-t0)/1e3:8.1f}us dur={dur[i]:8.1f}us levels={lev[i]:4d} "
              f"us/level={dur[i]/max(lev[i],1):6.2f} edges={edges[i]}")
    # when did the last 1% of samples start
    ss = np.sort((st[ok] - t0) / 1e3)
    print(f"   start times: p50 {ss[len(ss)//2]:.0f}us p99 {ss[int(len(ss)*0.99)]:.0f}us max {ss[-1]:.0f}us")
