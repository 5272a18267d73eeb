# full GPU check after the session's changes
set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_full.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu_full.log
grep -E "FAILED|Error" gpurun_out/pytest_gpu_full.log | head -20
timeout 1500 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err; echo bench=$?
tail -c 2200 gpurun_out/bench_final.json
