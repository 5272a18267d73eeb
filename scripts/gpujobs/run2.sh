set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?
timeout 1800 python -m pytest tests -m gpu -q -s -x -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?
timeout 900 python scripts/ab_merge.py C4 C2 C3 > gpurun_out/ab_merge.jsonl 2> gpurun_out/ab_merge.err; echo ab_rc=$?
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.log 2>gpurun_out/bench.err; echo bench_rc=$?
timeout 600 compute-sanitizer --tool racecheck python scripts/sanitize_ring.py 128 > gpurun_out/racecheck.log 2>&1; echo race_rc=$?
