# full-size SHARED parity gap with the DSMEM bitmap (printed per case)
set -x
timeout 1800 python -m pytest tests/test_fullsize_gpu.py -q -p no:cacheprovider -s -k "C2_search or C4_search or C3_search" > gpurun_out/pytest_fullsize.log 2>&1; echo pytest=$?
grep -E "gpu \[|passed|failed" gpurun_out/pytest_fullsize.log
