# full GPU test suite + smoke + smoke under ncu launch capture (the driver's round-end steps)
set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?; tail -1 gpurun_out/smoke.log
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -o faulthandler_timeout=600 > gpurun_out/pytest_gpu_full.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu_full.log
grep -E "FAILED|Timeout" gpurun_out/pytest_gpu_full.log | head -20
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/smoke_launches.csv python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_ncu.log 2>&1; echo smoke_ncu=$?
