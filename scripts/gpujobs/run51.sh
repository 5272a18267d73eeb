# screened kNN with base sizes not a multiple of 4; then C5s forward vs R35
set -x
timeout 900 python -m pytest tests/test_search_gpu.py tests/test_partitioned_gpu.py -q -p no:cacheprovider -x -k "knn or partitioned" > gpurun_out/pytest_knn4.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_knn4.log
bash scripts/gpujobs/run50.sh
