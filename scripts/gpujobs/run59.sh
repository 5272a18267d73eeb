# same-box A/B: HEAD (rank merge generalised to L <= 128) vs the commit before it, C2 and C4
set -x
for i in 1 2; do
timeout 600 python scripts/diag_tail.py C2 "L=12,w=12" 2>>gpurun_out/diag_ab9.err | sed 's/^{/{"lib": "head", /' >> gpurun_out/diag_ab9.jsonl
ALGAS_LIB=$PWD/build/libalgas_prev.so timeout 600 python scripts/diag_tail.py C2 "L=12,w=12" 2>>gpurun_out/diag_ab9.err | sed 's/^{/{"lib": "prev", /' >> gpurun_out/diag_ab9.jsonl
done
python - <<'PY'
import json
for l in open('gpurun_out/diag_ab9.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['lib'], d['variant'].ljust(14), d['qps'], d['recall'], d['p50'], c['gather'], c['dist'], c['sort'])
PY
