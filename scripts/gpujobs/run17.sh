set -x
timeout 900 python -m pytest tests/test_search_gpu.py tests/test_partitioned_gpu.py -q -p no:cacheprovider -k "knn or build_graph" > gpurun_out/pytest_knn.log 2>&1; echo pytest_rc=$?
timeout 900 python scripts/knn_gemm_ab.py C2 100000 > gpurun_out/knn_gemm_ab_C2.jsonl 2> gpurun_out/knn_gemm_ab_C2.err; echo ab=$?
timeout 600 ncu --set full --clock-control none -k regex:tc_dot -c 1 -f -o gpurun_out/prof_tc python scripts/knn_gemm_ab.py C1 10000 > gpurun_out/prof_tc.log 2>&1; echo prof=$?
ncu -i gpurun_out/prof_tc.ncu-rep --page raw --csv > gpurun_out/prof_tc_raw.csv 2>/dev/null; rm -f gpurun_out/prof_tc.ncu-rep
timeout 900 python scripts/build_timing.py C2 --clusters 256 --overlap 2 --refine 0 > gpurun_out/build_timing_exact.jsonl 2>&1; echo bt=$?
