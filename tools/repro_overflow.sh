set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for b in 6 8; do
EIM_SPILL_QUADS=1 EIM_TASK_QUADS=1 EIM_RING_W=64 timeout 600 compute-sanitizer --tool memcheck --show-backtrace no python tools/repro_overflow.py C2 $b 200 > gpurun_out/san_c2_$b.log 2>&1; tail -4 gpurun_out/san_c2_$b.log
done
EIM_SPILL_QUADS=1 EIM_TASK_QUADS=1 timeout 300 compute-sanitizer --tool memcheck --show-backtrace no python tools/repro_overflow.py C1 4 2000 > gpurun_out/san_c1b.log 2>&1; tail -4 gpurun_out/san_c1b.log
EIM_SPILL_QUADS=1 EIM_TASK_QUADS=1 EIM_RING_W=64 timeout 300 python tools/repro_overflow.py C2 12 3000 > gpurun_out/repro_c2b.log 2>&1; tail -4 gpurun_out/repro_c2b.log
timeout 1200 python -m pytest tests -m gpu -x -q -k "log_encoded or elim or fresh or flags" > gpurun_out/gpu_tests_next.log 2>&1; tail -5 gpurun_out/gpu_tests_next.log
