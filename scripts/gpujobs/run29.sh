# SHARED bitmap as the only visited set in the step (no smem hash probe): tests + A/B (PF=2056 keeps the hash)
set -x
timeout 900 python -m pytest tests/test_search_gpu.py tests/test_cosine_gpu.py -q -p no:cacheprovider -x -k "shared or server or dynamic or cosine" > gpurun_out/pytest_bmo.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_bmo.log
for c in "C2 L=12,w=12 L=12,w=12,PF=2056 L=11,w=11 L=13,w=8 L=12,w=12,vis=0" "C4 L=112,w=16,T=4,nt=1024 L=112,w=16,T=4,nt=1024,PF=2056"; do
timeout 900 python scripts/diag_tail.py $c 2>>gpurun_out/diag_bmo.err | sed "s/^{/{\"cfg\": \"${c%% *}\", /" >> gpurun_out/diag_bmo.jsonl; done
python - <<'PY'
import json
for l in open('gpurun_out/diag_bmo.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['cfg'], d['variant'].ljust(34), d['qps'], d['recall'], d['p50'], d['p99'], d['steps_max_cta'], d['evals'], c['gather'], c['dist'], c['sort'])
PY
