# Tuning sweep over compile-time sampler variants (run on the GPU box):
#   bash tools/variants.sh "-DEIM_IC_G=512 -DEIM_IC_THREADS_SM=1024" ...
# For each variant: rebuild libeim.so and time IMM runs on C2 (sampler kernel
# ms, greedy ms, total ms per run); restore the default build at the end.
for defs in "$@"; do
  echo "=== [$defs]"
  EIM_NVCC_DEFS="$defs" python paper_conf_sc_doneyhl25_b200/_build.py --force > /dev/null || { echo build failed; continue; }
  timeout 300 python tools/prof_imm.py ${EIM_VARIANT_CFG:-C2} 4 2>&1 | tail -2
done
python paper_conf_sc_doneyhl25_b200/_build.py --force > /dev/null
