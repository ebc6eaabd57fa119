# Sweep-only probe over compile-time variants (GPU box): bash tools/sweep_variants.sh "<defs>" ...
for defs in "$@"; do
  EIM_NVCC_DEFS="-DEIM_SWEEP_BENCH $defs" python paper_conf_sc_doneyhl25_b200/_build.py --force > /dev/null || { echo build failed; continue; }
  timeout 120 python tools/sweep_bench.py "[$defs]"
done
python paper_conf_sc_doneyhl25_b200/_build.py --force > /dev/null
