#!/bin/bash
# Final round measurement: bench lines (C2, C3, reference), launch list, ncu summaries, smoke.
set -x
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 900 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err; tail -c 400 $O/bench_c2.json
timeout 900 python bench.py --config C3 > $O/bench_c3.json 2> $O/bench_c3.err; tail -c 200 $O/bench_c3.json
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file $O/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 --budget-ids 0 --variant-steps 0 > $O/ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ic_kernel --launch-skip 6 -c 3 -f -o $O/prof_ic \
  python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 --budget-ids 0 --variant-steps 0 > $O/ncu_ic.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:greedy_kernel -c 2 -f -o $O/prof_greedy \
  python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 --budget-ids 0 --variant-steps 0 > $O/ncu_greedy.log 2>&1
timeout 900 python tools/ab_c4.py C4 > $O/c4_imm.log 2>&1; tail -3 $O/c4_imm.log
