# same-box A/B: dedicated L<=32 rank merge (restored) vs the generic E=1 instance (PF bit 65536)
set -x
timeout 600 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -x -k "lattice_exact" > gpurun_out/pytest_r32.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_r32.log
for i in 1 2; do timeout 600 python scripts/diag_tail.py C2 "L=12,w=12" "L=12,w=12,PF=65544" "L=13,w=8" "L=13,w=8,PF=65544" 2>>gpurun_out/diag_r32.err >> gpurun_out/diag_r32.jsonl; done
python - <<'PY'
import json
for l in open('gpurun_out/diag_r32.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['variant'].ljust(24), d['qps'], d['recall'], d['p50'], c['gather'], c['dist'], c['sort'])
PY
