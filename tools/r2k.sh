bash tools/gpu_round.sh r2k "not C4_sets" C2 C3
timeout 600 python tools/ab_env.py C2 5 EIM_NO_PAIR - 1 > gpurun_out/r2k.ab_pair_c2.txt 2>&1
EIM_DEBUG_TIMELINE=1 timeout 300 python tools/timeline.py C2 > /dev/null 2> gpurun_out/r2k.timeline.err
