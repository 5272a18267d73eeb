# parallel rank merge for lists up to 128 keys (PF bit 16384): exactness + A/B at C4/C3/C2
set -x
ALGAS_PREFETCH=16392 timeout 900 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -x -k "lattice_exact or wide_ctas or hand_trace" > gpurun_out/pytest_rk.log 2>&1; echo pytest_rk=$?; tail -1 gpurun_out/pytest_rk.log
timeout 900 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -x -k "lattice_exact or wide_ctas" > gpurun_out/pytest_rk0.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_rk0.log
timeout 900 python scripts/diag_tail.py C4 "L=112,w=12,T=4,nt=1024" "L=112,w=12,T=4,nt=1024,PF=16392" "L=128,w=16,T=4,nt=1024" "L=128,w=16,T=4,nt=1024,PF=16392" 2>gpurun_out/diag_rk.err > gpurun_out/diag_rk.jsonl
timeout 900 python scripts/diag_tail.py C2 "L=12,w=12" "L=12,w=12,PF=16392" "L=40,w=16" "L=40,w=16,PF=16392" 2>>gpurun_out/diag_rk.err >> gpurun_out/diag_rk.jsonl
timeout 900 python scripts/diag_tail.py C3 "L=64,w=8,T=4,nt=512" "L=64,w=8,T=4,nt=512,PF=16392" 2>>gpurun_out/diag_rk.err >> gpurun_out/diag_rk.jsonl
python - <<'PY'
import json
for l in open('gpurun_out/diag_rk.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['variant'].ljust(36), d['qps'], d['recall'], d['p50'], d['p99'], d['steps_max_cta'], c['gather'], c['dist'], c['sort'])
PY
