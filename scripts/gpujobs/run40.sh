# R34 prune (a CTA finishes when its best unchecked candidate is farther than the best k-th distance of the query's CTAs)
set -x
timeout 900 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -x -k "shared or server or dynamic" > gpurun_out/pytest_prune.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_prune.log
for v in 0 1; do ALGAS_PRUNE=$v timeout 900 python scripts/diag_tail.py C2 "L=12,w=12" "L=14,w=14" "L=16,w=16" "L=20,w=16" "L=13,w=8" 2>>gpurun_out/diag_prune.err | sed "s/^{/{\"prune\": $v, /" >> gpurun_out/diag_prune.jsonl; done
for v in 0 1; do ALGAS_PRUNE=$v timeout 900 python scripts/diag_tail.py C4 "L=112,w=16,T=4,nt=1024" "L=128,w=16,T=4,nt=1024" "L=160,w=16,T=4,nt=1024" 2>>gpurun_out/diag_prune.err | sed "s/^{/{\"prune\": $v, /" >> gpurun_out/diag_prune.jsonl; done
python - <<'PY'
import json
for l in open('gpurun_out/diag_prune.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['prune'], d['variant'].ljust(26), d['qps'], d['recall'], d['p50'], d['p99'], d['steps_mean_cta'], d['steps_max_cta'], d['evals'], c['gather'], c['dist'], c['sort'])
PY
