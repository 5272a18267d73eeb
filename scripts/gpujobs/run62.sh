# the driver's reference arm (the oracle timed alone) still runs
set -x
timeout 1500 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo ref=$?
tail -c 1500 gpurun_out/bench_ref.json
