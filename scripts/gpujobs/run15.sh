set -x
timeout 900 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -k "knn or watchdog or shared_visited" > gpurun_out/pytest_knn.log 2>&1; echo pytest_rc=$?
timeout 900 python scripts/knn_gemm_ab.py C2 100000 > gpurun_out/knn_gemm_ab_C2.jsonl 2> gpurun_out/knn_gemm_ab_C2.err; echo ab=$?
timeout 600 ncu --set full --clock-control none -k regex:tc_dot -c 1 -f -o gpurun_out/prof_tc python scripts/knn_gemm_ab.py C1 10000 > gpurun_out/prof_tc.log 2>&1; echo prof=$?
ncu -i gpurun_out/prof_tc.ncu-rep --page raw --csv > gpurun_out/prof_tc_raw.csv 2>/dev/null; ncu -i gpurun_out/prof_tc.ncu-rep --page details --csv > gpurun_out/prof_tc_details.csv 2>/dev/null; rm -f gpurun_out/prof_tc.ncu-rep
cuobjdump -sass paper_conf_ipps_chencyzw025_b200/libalgas.so | grep -c UTCHMMA > gpurun_out/utc_count.txt
