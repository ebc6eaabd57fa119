bash tools/gpu_round.sh r2j "not C4_sets"
for B in - 74 37; do
  echo "blocks $B" >> gpurun_out/r2j.ab.txt
  if [ "$B" != "-" ]; then export EIM_GREEDY_BLOCKS=$B; fi
  timeout 600 python tools/ab_env.py C3 3 EIM_NO_PAIR - 1 >> gpurun_out/r2j.ab.txt 2>&1
done
