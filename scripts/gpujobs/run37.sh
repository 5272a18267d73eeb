set -x
timeout 900 python scripts/diag_tail.py C2 "L=12,w=12,PF=8" "L=12,w=12,PF=0" "L=12,w=12,PF=4" "L=12,w=12,PF=8" "L=12,w=12,PF=0" 2>gpurun_out/diag_pf0.err > gpurun_out/diag_pf0.jsonl
python - <<'PY'
import json
for l in open('gpurun_out/diag_pf0.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['variant'].ljust(24), d['qps'], d['recall'], d['p50'], d['p99'], d['steps_max_cta'], c['gather'], c['dist'], c['sort'])
PY
