# R35 more rounds / larger fan at C2
set -x
timeout 1500 python scripts/build_timing.py C2 --clusters 256 --overlap 2 --refine 12 16 --fan 16 --reverse --no-exact --search-L 32 64 128 > gpurun_out/build_rev2_C2.jsonl 2> gpurun_out/build_rev2_C2.err; echo bt=$?
timeout 1500 python scripts/build_timing.py C2 --clusters 256 --overlap 2 --refine 8 --fan 32 --reverse --no-exact --search-L 32 64 128 >> gpurun_out/build_rev2_C2.jsonl 2>> gpurun_out/build_rev2_C2.err; echo bt=$?
python - <<'PY'
import json
for l in open('gpurun_out/build_rev2_C2.jsonl'):
    d=json.loads(l)
    if 'refine_rounds' in d: print(d['refine_rounds'], d['fan'], round(d['build_s'],2), round(d['knn_graph_recall_sample'],3), d['search_recall'], d['search_T4_L_recall_qps'])
PY
