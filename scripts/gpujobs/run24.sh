# gather sub-phase timing (SUBLAP build)
set -x
SUBLAP=1 ALGAS_BUILD_DEFS="-DALGAS_SUBLAP=1" ALGAS_LIB=$PWD/build/libalgas_sublap.so timeout 900 python scripts/diag_tail.py C2 "L=12,w=12,PF=8" "L=12,w=12,PF=520" "L=12,w=12,PF=8,vis=0" "L=12,w=12,PF=520,vis=0" > gpurun_out/diag_sub.jsonl 2> gpurun_out/diag_sub.err; echo rc=$?
python -c "
import json
for l in open('gpurun_out/diag_sub.jsonl'):
    d=json.loads(l); print({k:d[k] for k in d if k not in ('hist_max_iters',)})
"
