"""Aggregate an ncu --metrics gpu__time_duration.sum --csv launch list per kernel.
    python tools/launch_table.py launches.csv out.txt "command"   """
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
hdr = rows[start]
idx = {k: j for j, k in enumerate(hdr)}
scale = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}
agg = collections.defaultdict(lambda: [0, 0.0])
for r in rows[start + 1:]:
    if len(r) < len(hdr) or r[idx["Metric Name"]] != "gpu__time_duration.sum":
        continue
    name = r[idx["Kernel Name"]].split("(")[0]
    agg[name][0] += 1
    agg[name][1] += float(r[idx["Metric Value"]].replace(",", "")) * scale[r[idx["Metric Unit"]]]
tot = sum(v[1] for v in agg.values())
with open(sys.argv[2], "w") as f:
    f.write(f"ncu launch list of `{sys.argv[3]}` (cold-cache, serialised: compare shares)\n")
    f.write(f"{'kernel':64s} {'launches':>8s} {'total_us':>12s} {'share':>7s}\n")
    for k, (n, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        f.write(f"{k[:64]:64s} {n:8d} {us:12.1f} {us / tot:7.1%}\n")
