set -x
nproc; nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/smoke_ncu.csv python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_ncu.log 2>&1; echo ncu_smoke_rc=$?
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.log 2>gpurun_out/bench.err; echo bench_rc=$?
timeout 600 python bench.py --impl reference --steps 10 --warmup 3 > gpurun_out/bench_ref.log 2>gpurun_out/bench_ref.err; echo ref_rc=$?
timeout 1800 python -m pytest tests -m gpu -q -s -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?
timeout 600 compute-sanitizer --tool racecheck python scripts/sanitize_ring.py 128 > gpurun_out/racecheck.log 2>&1; echo race_rc=$?
timeout 600 compute-sanitizer --tool synccheck python scripts/sanitize_ring.py 128 > gpurun_out/synccheck.log 2>&1; echo sync_rc=$?
timeout 600 compute-sanitizer --tool memcheck python scripts/sanitize_ring.py 128 > gpurun_out/memcheck.log 2>&1; echo mem_rc=$?
