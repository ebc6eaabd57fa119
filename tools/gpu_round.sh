#!/bin/bash
# One gpurun call: build, selected GPU tests, short benches.  Usage (under gpurun):
#   bash tools/gpu_round.sh TAG "pytest -k expr" [bench configs...]
TAG=$1; K=$2; shift 2
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/$TAG.build.log 2>&1 || { tail -30 gpurun_out/$TAG.build.log; exit 1; }
nproc > gpurun_out/$TAG.nproc
if [ -n "$K" ]; then
  timeout 2400 python -m pytest tests -m gpu -x -q -k "$K" > gpurun_out/$TAG.tests.log 2>&1
  tail -5 gpurun_out/$TAG.tests.log
fi
for C in "$@"; do
  timeout 600 python bench.py --config $C --steps 10 --warmup 3 --no-cpu-baseline --variant-steps 0 --e2e-steps 1 > gpurun_out/$TAG.bench_$C.json 2> gpurun_out/$TAG.bench_$C.err
  python - "$TAG" "$C" <<'PY'
import json,sys
t,c=sys.argv[1],sys.argv[2]
try:
    d=json.loads(open(f"gpurun_out/{t}.bench_{c}.json").read().strip().splitlines()[-1])
    print(c, "ms/IMM %.3f" % d["ms_per_step"], "phase", {k: round(v,3) for k,v in d["phase_ms"].items()}, "frac", d["roofline"]["frac"])
except Exception as e:
    print(c, "bench failed", e, open(f"gpurun_out/{t}.bench_{c}.err").read()[-2000:])
PY
done
