# debug: the hanging NCCL sharded-server test (stack dump after 60 s) and the C3 SHARED parity values
set -x
timeout 180 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -s -k "sharded_server_nccl" -o faulthandler_timeout=60 > gpurun_out/pytest_ss.log 2>&1; echo ss=$?
tail -60 gpurun_out/pytest_ss.log
timeout 900 python -m pytest tests/test_fullsize_gpu.py -q -p no:cacheprovider -s -k "C3_search" > gpurun_out/pytest_c3.log 2>&1; echo c3=$?
grep -E "gpu \[|passed|failed|assert" gpurun_out/pytest_c3.log | head
