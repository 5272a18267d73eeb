set -x
timeout 600 python scripts/diag_overflow.py > gpurun_out/diag_overflow.log 2>&1; echo diag=$?
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_C2.log 2>gpurun_out/bench_C2.err; echo bC2=$?
