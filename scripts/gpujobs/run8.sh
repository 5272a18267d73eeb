set -x
timeout 900 python -m pytest tests/test_partitioned_gpu.py -q -x -p no:cacheprovider > gpurun_out/pytest_part.log 2>&1; echo pytest_rc=$?
timeout 1500 python scripts/build_timing.py C2 --no-exact --clusters 256 --overlap 2 --refine 4 8 12 --fan 16 > gpurun_out/build_timing_C2_f16.jsonl 2>gpurun_out/build_timing_C2_f16.err; echo bt=$?
timeout 1500 python scripts/build_timing.py C2 --no-exact --clusters 256 --overlap 2 --refine 4 8 --fan 32 > gpurun_out/build_timing_C2_f32.jsonl 2>gpurun_out/build_timing_C2_f32.err; echo bt=$?
