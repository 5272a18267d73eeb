# rank merge for L <= 32 (parallel warps) vs warp-0 bitonic (PF bit 4096): exactness + A/B
set -x
timeout 1200 python -m pytest tests/test_search_gpu.py tests/test_cosine_gpu.py -q -p no:cacheprovider -x > gpurun_out/pytest_rank.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_rank.log
ALGAS_PREFETCH=4104 timeout 900 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -x -k "lattice_exact or hand_trace" > gpurun_out/pytest_rank_bitonic.log 2>&1; echo pytest_b=$?; tail -2 gpurun_out/pytest_rank_bitonic.log
timeout 900 python scripts/diag_tail.py C2 "L=12,w=12" "L=12,w=12,PF=4104" "L=11,w=11" "L=11,w=11,PF=4104" "L=13,w=8" "L=10,w=8,T=8,nt=512" "L=10,w=8,T=8,nt=512,PF=4104" 2>gpurun_out/diag_rank.err > gpurun_out/diag_rank.jsonl
python - <<'PY'
import json
for l in open('gpurun_out/diag_rank.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['variant'].ljust(34), d['qps'], d['recall'], d['p50'], d['p99'], d['steps_max_cta'], d['evals'], c['gather'], c['dist'], c['sort'])
PY
