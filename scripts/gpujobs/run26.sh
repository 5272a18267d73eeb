# cluster-slot start (DSMEM push): tests + A/B at C2
set -x
timeout 900 python -m pytest tests/test_search_gpu.py tests/test_cosine_gpu.py -q -p no:cacheprovider -x -k "shared or server or dynamic or cosine" > gpurun_out/pytest_dsmem2.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_dsmem2.log
for v in 1 0; do ALGAS_VIS_DSMEM=$v timeout 600 python scripts/diag_tail.py C2 "L=12,w=12" "L=13,w=8" "L=10,w=8,T=8,nt=512" "L=11,w=11" 2>>gpurun_out/diag_dsmem2.err | sed "s/^{/{\"dsmem\": $v, /" >> gpurun_out/diag_dsmem2.jsonl; done
python - <<'PY'
import json
for l in open('gpurun_out/diag_dsmem2.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['dsmem'], d['variant'].ljust(24), d['qps'], d['recall'], d['p50'], d['steps_max_cta'], d['us_pickup_to_loop_first'], d['us_pickup_to_loop_last'], c['gather'], c['dist'], c['sort'])
PY
