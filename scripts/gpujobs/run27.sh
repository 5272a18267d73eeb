# DSMEM bitmap + cluster-slot start vs HBM bitmap at C2/C4/C3 op points
set -x
for c in "C2 L=12,w=12 L=13,w=8" "C4 L=112,w=16,T=4,nt=1024 L=128,w=16,T=4,nt=1024" "C3 L=64,w=8,T=4,nt=512"; do
for v in 1 0; do ALGAS_VIS_DSMEM=$v timeout 900 python scripts/diag_tail.py $c 2>>gpurun_out/diag_dsmem3.err | sed "s/^{/{\"cfg\": \"${c%% *}\", \"dsmem\": $v, /" >> gpurun_out/diag_dsmem3.jsonl; done; done
python - <<'PY'
import json
for l in open('gpurun_out/diag_dsmem3.jsonl'):
    d=json.loads(l); c=d['cyc_per_step']
    print(d['cfg'], d['dsmem'], d['variant'].ljust(26), d['qps'], d['recall'], d['p50'], d['p99'], d['steps_max_cta'], d['us_pickup_to_loop_first'], d['us_pickup_to_loop_last'], c['gather'], c['dist'], c['sort'])
PY
