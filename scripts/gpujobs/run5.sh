set -x
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_C2.log 2>gpurun_out/bench_C2.err; echo bC2=$?
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-sweep --host-threads 4 > gpurun_out/bench_ht4.log 2>gpurun_out/bench_ht4.err; echo bht4=$?
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-sweep --host-threads 4 --state-mirror 1 > gpurun_out/bench_ht4_m1.log 2>gpurun_out/bench_ht4_m1.err; echo bht4m1=$?
timeout 1200 python bench.py --config C4 --steps 10 --warmup 3 --ctas 2,4 --threads 512,1024 --width 16 > gpurun_out/bench_C4.log 2>gpurun_out/bench_C4.err; echo bC4=$?
timeout 1500 python bench.py --config C3 --steps 10 --warmup 3 --ctas 2,4 --threads 512 --width 8,16 > gpurun_out/bench_C3.log 2>gpurun_out/bench_C3.err; echo bC3=$?
