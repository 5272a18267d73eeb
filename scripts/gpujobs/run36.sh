set -x
timeout 900 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -x -k "lattice_exact or hand_trace" > gpurun_out/pytest_lb.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_lb.log
timeout 900 python scripts/diag_tail.py C2 "L=12,w=12" "L=13,w=8" "L=12,w=12" 2>gpurun_out/diag_lb.err > gpurun_out/diag_lb.jsonl
python - <<'PY'
import json
for l in open('gpurun_out/diag_lb.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['variant'].ljust(24), d['qps'], d['recall'], d['p50'], d['p99'], d['steps_max_cta'], c['gather'], c['dist'], c['sort'])
PY
