# Tuning sweep over compile-time sampler variants (run on the GPU box).
run() { timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 1 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['ms_per_step'],3), round(d['phase_ms']['sample_kernel'],3), d['result']['spilled_samples'])"; }
for defs in "-DEIM_IC_NSG=1" "-DEIM_IC_NSG=1 -DEIM_PARK_EDGE=1" "-DEIM_IC_NSG=2 -DEIM_IC_THREADS_SM=1024" "-DEIM_IC_NSG=4 -DEIM_IC_THREADS_SM=1024"; do
  EIM_NVCC_DEFS="$defs" python paper_conf_sc_doneyhl25_b200/_build.py --force > /dev/null
  for tq in 6144 8192 12288; do EIM_TASK_QUADS=$tq run "[$defs] tq=$tq"; done
done
python paper_conf_sc_doneyhl25_b200/_build.py --force > /dev/null
