# SHARED bitmap in DSMEM (slot clusters): tests + A/B at C2
set -x
timeout 900 python -m pytest tests/test_search_gpu.py tests/test_fullsize_gpu.py -q -p no:cacheprovider -x -k "shared or server or dynamic" > gpurun_out/pytest_dsmem.log 2>&1; echo pytest=$?; tail -5 gpurun_out/pytest_dsmem.log
for v in 1 0 1 0; do ALGAS_VIS_DSMEM=$v timeout 600 python scripts/diag_tail.py C2 "L=12,w=12" "L=13,w=8" "L=12,w=12,T=8,nt=512" "L=10,w=8,T=8,nt=512" "L=11,w=12,T=8,nt=512" 2>>gpurun_out/diag_dsmem.err | sed "s/^/{\"dsmem\": $v, /; s/{\"dsmem\": $v, {/{\"dsmem\": $v, /" >> gpurun_out/diag_dsmem.jsonl; done
cut -c1-400 gpurun_out/diag_dsmem.jsonl
