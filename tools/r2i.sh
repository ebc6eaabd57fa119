bash tools/gpu_round.sh r2i "not C4_sets" C2 C3
timeout 600 python tools/ab_env.py C3 5 EIM_NO_PAIR - 1 > gpurun_out/r2i.ab_pair_c3.txt 2>&1
timeout 600 python tools/ab_env.py C2 5 EIM_NO_PAIR - 1 > gpurun_out/r2i.ab_pair_c2.txt 2>&1
