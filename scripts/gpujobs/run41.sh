# relaxed query-start barrier + no slot_fin fence in cluster mode (current) vs previous commit (build/libalgas_prev.so)
set -x
timeout 900 python -m pytest tests/test_search_gpu.py tests/test_cosine_gpu.py -q -p no:cacheprovider -x -k "shared or server or dynamic or cosine or lattice" > gpurun_out/pytest_rel.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_rel.log
for i in 1 2; do
timeout 600 python scripts/diag_tail.py C2 "L=12,w=12" "L=13,w=8" 2>>gpurun_out/diag_rel.err | sed "s/^{/{\"lib\": \"cur\", /" >> gpurun_out/diag_rel.jsonl
ALGAS_LIB=$PWD/build/libalgas_prev.so timeout 600 python scripts/diag_tail.py C2 "L=12,w=12" "L=13,w=8" 2>>gpurun_out/diag_rel.err | sed "s/^{/{\"lib\": \"prev\", /" >> gpurun_out/diag_rel.jsonl
done
python - <<'PY'
import json
for l in open('gpurun_out/diag_rel.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['lib'], d['variant'].ljust(14), d['qps'], d['recall'], d['p50'], d['p99'], d['steps_max_cta'], d['us_pickup_to_loop_first'], c['gather'], c['dist'], c['sort'])
PY
