#!/bin/bash
# sampler scheduling change: quick C2 bench, C4 IMM timing, then the parity suite
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python bench.py --steps 5 --variant-steps 0 --no-cpu-baseline --e2e-steps 0 > $O/bench_c2_quick.json 2>$O/bench_c2_quick.err
python - <<'PY'
import json
d = json.loads(open("gpurun_out/bench_c2_quick.json").read().strip().splitlines()[-1])
print("C2", d["ms_per_step"], d["phase_ms"], "frac", d["roofline"]["frac"], "budget", d["sampler_fixed_budget"]["edges_per_s"] / 1e9, d["sampler_fixed_budget"]["frac"])
PY
timeout 1200 python tools/c4_timeline.py > $O/c4_timeline.log 2>&1; grep -E "timeline|C4 imm" $O/c4_timeline.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/gpu_tests.log 2>&1; tail -3 $O/gpu_tests.log
