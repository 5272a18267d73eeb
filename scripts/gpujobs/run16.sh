set -x
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_C2.log 2>gpurun_out/bench_C2.err; echo bC2=$?
timeout 600 python bench.py --impl reference --steps 10 --warmup 3 > gpurun_out/bench_ref.log 2>gpurun_out/bench_ref.err; echo bref=$?
timeout 1200 python scripts/build_timing.py C2 --clusters 256 --overlap 2 --refine 8 --fan 32 > gpurun_out/build_timing_C2_final.jsonl 2>gpurun_out/build_timing_C2_final.err; echo bt=$?
