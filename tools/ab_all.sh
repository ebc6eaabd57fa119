#!/bin/bash
# row-range tasks + LT step overlap: parity, A/B on C2, C3 bench, C4 A/B
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/gpu_tests.log 2>&1; tail -3 $O/gpu_tests.log
timeout 600 python tools/ab_rowsplit.py C2 6 > $O/ab_rowsplit_c2.log 2>&1; cat $O/ab_rowsplit_c2.log
timeout 600 python bench.py --config C3 --steps 5 --variant-steps 0 --no-cpu-baseline --e2e-steps 0 --budget-ids 0 > $O/bench_c3_quick.json 2>&1; tail -c 700 $O/bench_c3_quick.json
timeout 1200 python tools/ab_c4.py C4 > $O/ab_c4.log 2>&1; cat $O/ab_c4.log
