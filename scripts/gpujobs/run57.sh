# T=8 x 512-thread clusters (2 CTAs/SM, DSMEM bitmap) at smaller widths vs T=4 x 1024
set -x
timeout 900 python scripts/diag_tail.py C2 "L=12,w=12" "L=10,w=8,T=8,nt=512" "L=10,w=6,T=8,nt=512" "L=10,w=4,T=8,nt=512" "L=10,w=3,T=8,nt=512" "L=10,w=4,T=8,nt=512,S=8" "L=10,w=6,T=8,nt=512,S=8" 2>gpurun_out/diag_t8b.err > gpurun_out/diag_t8b.jsonl
python - <<'PY'
import json
for l in open('gpurun_out/diag_t8b.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['variant'].ljust(28), d['qps'], d['recall'], d['p50'], d['p99'], d['steps_mean_cta'], d['steps_max_cta'], d['evals'], c['gather'], c['dist'], c['sort'])
PY
