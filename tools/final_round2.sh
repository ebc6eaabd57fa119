#!/bin/bash
# Round-2 validation on one B200 (one gpurun call): every GPU test, smoke,
# the bench lines + ncu captures (tools/profile_round.sh).  The C5
# full-size parity run is a call of its own (tools/big_parity.py, ~45 min).
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/f_build.log 2>&1 || { tail -20 $O/f_build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q > $O/f_tests.log 2>&1; tail -3 $O/f_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/f_smoke.log 2>&1; tail -2 $O/f_smoke.log
bash tools/profile_round.sh > $O/f_profile.log 2>&1
