set -x
timeout 600 python -m pytest tests/test_search_gpu.py -q -x -p no:cacheprovider -k "server or watchdog" > gpurun_out/pytest_srv.log 2>&1; echo pytest_rc=$?
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?
timeout 2400 python bench.py --config C5s --steps 5 --warmup 3 --no-cpu --no-sweep --ctas 4 --threads 1024 --width 12,16 --visited 1 > gpurun_out/bench_C5s.log 2>gpurun_out/bench_C5s.err; echo bC5s=$?
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_C2_b.log 2>gpurun_out/bench_C2_b.err; echo bC2=$?
