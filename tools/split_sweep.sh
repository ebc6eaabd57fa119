for sq in 8192 4096 2048 1024; do for tq in 8192 2048 1024 512; do
  echo "spill=$sq task=$tq $(EIM_SPILL_QUADS=$sq EIM_TASK_QUADS=$tq timeout 120 python tools/prof_imm.py C2 3 2>&1 | tail -1)"
done; done
