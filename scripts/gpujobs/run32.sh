# single-warp shuffle merge (nk <= 32): exactness + A/B; full bench with the in-run ncu traffic pass
set -x
timeout 1200 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -x -k "lattice_exact or hand_trace or dynamic or server or shared" > gpurun_out/pytest_wm.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_wm.log
timeout 900 python scripts/diag_tail.py C2 "L=12,w=12" "L=12,w=12,PF=8200" "L=13,w=8" "L=13,w=8,PF=8200" 2>gpurun_out/diag_wm.err > gpurun_out/diag_wm.jsonl
python - <<'PY'
import json
for l in open('gpurun_out/diag_wm.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['variant'].ljust(24), d['qps'], d['recall'], d['p50'], d['p99'], d['steps_max_cta'], c['gather'], c['dist'], c['sort'])
PY
timeout 1500 python bench.py > gpurun_out/bench32.json 2> gpurun_out/bench32.err; echo bench=$?
tail -c 3000 gpurun_out/bench32.json
