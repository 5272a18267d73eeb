set -x
timeout 900 python -m pytest tests/test_partitioned_gpu.py tests/test_search_gpu.py -q -x -p no:cacheprovider > gpurun_out/pytest_part.log 2>&1; echo pytest_rc=$?
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_C2.log 2>gpurun_out/bench_C2.err; echo bC2=$?
timeout 1200 python scripts/build_timing.py C2 --clusters 256 512 --overlap 2 3 --refine 0 1 2 --fan 16 > gpurun_out/build_timing_C2.jsonl 2>gpurun_out/build_timing_C2.err; echo bt=$?
