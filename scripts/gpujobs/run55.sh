set -x
timeout 180 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -s -k "sharded" -o faulthandler_timeout=60 > gpurun_out/pytest_ss.log 2>&1; echo ss=$?
tail -3 gpurun_out/pytest_ss.log
