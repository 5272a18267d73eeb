# R35 reverse-neighbour refinement: parity vs oracle, then partitioned-build quality at C2
set -x
timeout 900 python -m pytest tests/test_partitioned_gpu.py -q -p no:cacheprovider -x -k "refine" > gpurun_out/pytest_rev.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_rev.log
timeout 1500 python scripts/build_timing.py C2 --clusters 256 --overlap 2 --refine 2 4 8 --fan 16 --reverse --no-exact --search-L 12 32 64 > gpurun_out/build_rev_C2.jsonl 2> gpurun_out/build_rev_C2.err; echo bt=$?
cut -c1-400 gpurun_out/build_rev_C2.jsonl
