# 768-thread CTAs (80 registers: two rows per team, 192 rows per pass): exactness + A/B
set -x
timeout 900 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -x -k "lattice_exact or wide_ctas or hand_trace" > gpurun_out/pytest_768.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_768.log
timeout 900 python scripts/diag_tail.py C2 "L=12,w=12,nt=1024" "L=12,w=12,nt=768" "L=13,w=8,nt=768" "L=12,w=16,nt=768" "L=14,w=12,nt=768" "L=12,w=12,nt=1024" "L=12,w=12,nt=768" 2>gpurun_out/diag_768.err > gpurun_out/diag_768.jsonl
timeout 900 python scripts/diag_tail.py C4 "L=112,w=12,T=4,nt=1024" "L=112,w=12,T=4,nt=768" "L=112,w=16,T=4,nt=768" 2>>gpurun_out/diag_768.err >> gpurun_out/diag_768.jsonl
python - <<'PY'
import json
for l in open('gpurun_out/diag_768.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['variant'].ljust(26), d['qps'], d['recall'], d['p50'], d['p99'], d['steps_max_cta'], c['gather'], c['dist'], c['sort'])
PY
