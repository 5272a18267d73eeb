set -x
timeout 900 python -m pytest tests/test_search_gpu.py -q -x -p no:cacheprovider -k "server or lattice_exact or beam" > gpurun_out/pytest_sel.log 2>&1; echo pytest_sel_rc=$?
timeout 900 python scripts/sweep_grid.py C2 --T 4,6,8 --threads 512,1024 --width 4,6,8,12 --seeds 8,16,32 > gpurun_out/sweep_grid_C2.jsonl 2> gpurun_out/sweep_grid_C2.err; echo sweep_rc=$?
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_m0.log 2>gpurun_out/bench_m0.err; echo b0=$?
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-sweep --state-mirror 1 > gpurun_out/bench_m1.log 2>gpurun_out/bench_m1.err; echo b1=$?
ls /dev | grep -i gdr; lsmod 2>/dev/null | grep -i -E "gdr|peermem"; nproc
