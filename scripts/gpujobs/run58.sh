# distributed select for L <= 32 (default) vs warp-0 select (PF bit 32768): exactness + A/B
set -x
timeout 900 python -m pytest tests/test_search_gpu.py tests/test_cosine_gpu.py -q -p no:cacheprovider -x -k "lattice_exact or hand_trace or wide_ctas or dynamic or server or shared or cosine or max_iter or degenerate" > gpurun_out/pytest_ds.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_ds.log
for i in 1 2; do timeout 900 python scripts/diag_tail.py C2 "L=12,w=12" "L=12,w=12,PF=32776" "L=13,w=8" "L=13,w=8,PF=32776" 2>>gpurun_out/diag_ds.err >> gpurun_out/diag_ds.jsonl; done
python - <<'PY'
import json
for l in open('gpurun_out/diag_ds.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['variant'].ljust(24), d['qps'], d['recall'], d['p50'], d['p99'], d['steps_max_cta'], c['gather'], c['dist'], c['sort'])
PY
