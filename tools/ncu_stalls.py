"""Stall-reason breakdown of an `ncu --page source --csv` export (SASS view):
totals per reason and the top instructions by samples, per profiled launch.

    python tools/ncu_stalls.py gpurun_out/prof_src.csv [launch_index] [top]
"""
import csv
import sys


def main(path, which=None, top=25):
    rows = list(csv.reader(open(path)))
    hdrs = [i for i, r in enumerate(rows) if r and r[0] == "Address"]
    for li, hi in enumerate(hdrs):
        if which is not None and li != which:
            continue
        h = rows[hi]
        end = hdrs[li + 1] - 1 if li + 1 < len(hdrs) else len(rows)
        body = [r for r in rows[hi + 1:end] if len(r) == len(h)]
        reasons = [(i, x) for i, x in enumerate(h) if x.startswith("stall_") and "Not Issued" not in x]
        tot = {x: sum(int(r[i] or 0) for r in body) for i, x in reasons}
        allsamp = sum(int(r[2] or 0) for r in body)
        print(f"launch {li}: samples {allsamp}")
        for k, v in sorted(tot.items(), key=lambda kv: -kv[1])[:10]:
            print(f"   {k:28s} {v:9d} {100.0 * v / max(allsamp, 1):5.1f}%")
        body.sort(key=lambda r: -int(r[2] or 0))
        for r in body[:top]:
            top3 = sorted(((int(r[i] or 0), x) for i, x in reasons), reverse=True)[:3]
            print(f"   {int(r[2]):8d} {r[1].strip()[:60]:60s} " + " ".join(f"{x[6:]}={v}" for v, x in top3 if v))


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else None, int(sys.argv[3]) if len(sys.argv) > 3 else 25)
