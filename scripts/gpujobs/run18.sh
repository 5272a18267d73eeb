set -x
timeout 600 python -m pytest tests/test_search_gpu.py tests/test_abi.py -q -p no:cacheprovider -k "server or merge or watchdog" > gpurun_out/pytest_srv.log 2>&1; echo pytest_rc=$?
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-sweep > gpurun_out/bench_e2e_ht1.log 2>gpurun_out/bench_e2e_ht1.err; echo b1=$?
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-sweep --host-threads 2 > gpurun_out/bench_e2e_ht2.log 2>gpurun_out/bench_e2e_ht2.err; echo b2=$?
