ALGAS_TRACE=1 timeout 300 python scripts/probe_call.py C2 12 12 1 4 1024 1 > gpurun_out/probe.log 2>&1
B="--ctas 4 --threads 1024 --width 12 --visited 1 --no-cpu --no-sweep"
timeout 600 python bench.py $B > gpurun_out/bench_a.json 2> gpurun_out/bench_a.err
ALGAS_BENCH_CLOCK_PERIOD=100 timeout 600 python bench.py $B > gpurun_out/bench_b.json 2> gpurun_out/bench_b.err
timeout 1100 python -m pytest tests/test_fullsize_gpu.py -q -rA > gpurun_out/fullsize.log 2>&1; echo rc=$?; tail -15 gpurun_out/fullsize.log
