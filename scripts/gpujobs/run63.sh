# final driver-equivalent pass on the final commit
set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?; tail -1 gpurun_out/smoke.log
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -o faulthandler_timeout=600 > gpurun_out/pytest_gpu_full.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_gpu_full.log
timeout 1500 python bench.py > gpurun_out/bench_final2.json 2> gpurun_out/bench_final2.err; echo bench=$?
tail -c 600 gpurun_out/bench_final2.json
timeout 900 python bench.py --impl reference > gpurun_out/bench_ref2.json 2> gpurun_out/bench_ref2.err; echo ref=$?
tail -c 300 gpurun_out/bench_ref2.json
