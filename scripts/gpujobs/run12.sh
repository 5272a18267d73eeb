set -x
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_C2.log 2>gpurun_out/bench_C2.err; echo bC2=$?
timeout 600 python bench.py --impl reference --steps 10 --warmup 3 > gpurun_out/bench_ref.log 2>gpurun_out/bench_ref.err; echo bref=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"persistent|batch" -c 60 --csv --log-file gpurun_out/launches_C2.csv python bench.py --steps 2 --warmup 1 --no-cpu --no-sweep --no-e2e --ctas 4 --threads 1024 --width 12 --visited 1 > gpurun_out/launches_C2_run.log 2>&1; echo l2=$?
timeout 1200 python scripts/sweep_grid.py C2 --T 4,6,8 --threads 512,1024 --width 8,12 --seeds 32 > gpurun_out/sweep_grid_C2.jsonl 2> gpurun_out/sweep_grid_C2.err; echo sweep_rc=$?
timeout 1200 python bench.py --config C4 --steps 10 --warmup 3 --ctas 2,4 --threads 512,1024 --width 16 > gpurun_out/bench_C4.log 2>gpurun_out/bench_C4.err; echo bC4=$?
timeout 1500 python bench.py --config C3 --steps 10 --warmup 3 --ctas 2,4 --threads 512 --width 8,16 > gpurun_out/bench_C3.log 2>gpurun_out/bench_C3.err; echo bC3=$?
timeout 600 compute-sanitizer --tool racecheck python scripts/sanitize_ring.py 128 > gpurun_out/racecheck.log 2>&1; echo race_rc=$?
timeout 600 compute-sanitizer --tool synccheck python scripts/sanitize_ring.py 128 > gpurun_out/synccheck.log 2>&1; echo sync_rc=$?
timeout 600 compute-sanitizer --tool memcheck python scripts/sanitize_ring.py 128 > gpurun_out/memcheck.log 2>&1; echo mem_rc=$?
du -sh gpurun_out
