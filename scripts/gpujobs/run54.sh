# re-check: NCCL sharded-server test (allocator warmed first), full-size C3/C4 SHARED with larger samples
set -x
timeout 180 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -s -k "sharded" -o faulthandler_timeout=60 > gpurun_out/pytest_ss.log 2>&1; echo ss=$?
tail -3 gpurun_out/pytest_ss.log
timeout 1500 python -m pytest tests/test_fullsize_gpu.py -q -p no:cacheprovider -s -k "C3_search or C4_search" > gpurun_out/pytest_c34.log 2>&1; echo c34=$?
grep -E "gpu \[|passed|failed|Error" gpurun_out/pytest_c34.log | head
