#!/bin/bash
# One GPU call (round 2): bench lines (C2, C3, reference arm), the ncu launch
# lists of the bench commands, and ncu --set full captures of the IC sampler,
# the greedy kernel and the LT walk kernel.  Outputs in gpurun_out/r02_*.
set -x
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/r02_build.log 2>&1
timeout 900 python bench.py > $O/r02_bench_c2.json 2> $O/r02_bench_c2.err; tail -c 600 $O/r02_bench_c2.json
timeout 900 python bench.py --config C3 > $O/r02_bench_c3.json 2> $O/r02_bench_c3.err; tail -c 300 $O/r02_bench_c3.json
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/r02_bench_ref.json 2> $O/r02_bench_ref.err; tail -c 300 $O/r02_bench_ref.json
B="--steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 --budget-ids 0 --variant-steps 0"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file $O/r02_launches.csv \
  python bench.py $B > $O/r02_ncu_launch_c2.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file $O/r02_launches_c3.csv \
  python bench.py --config C3 $B > $O/r02_ncu_launch_c3.log 2>&1
B1="--steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 --budget-ids 0 --variant-steps 0"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:ic_kernel --launch-skip 9 -c 3 -f -o $O/r02_prof_ic \
  python bench.py $B1 > $O/r02_ncu_ic.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:greedy_kernel --launch-skip 6 -c 2 -f -o $O/r02_prof_greedy \
  python bench.py --config C3 $B1 > $O/r02_ncu_greedy.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lt_aug_kernel --launch-skip 3 -c 2 -f -o $O/r02_prof_lt \
  python bench.py --config C3 $B1 > $O/r02_ncu_lt.log 2>&1
ls -la $O | grep r02
