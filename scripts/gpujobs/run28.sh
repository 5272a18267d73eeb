# gather sub-phase timing (SUBLAP build) with the DSMEM bitmap
set -x
SUBLAP=1 ALGAS_BUILD_DEFS="-DALGAS_SUBLAP=1" ALGAS_LIB=$PWD/build/libalgas_sublap.so timeout 900 python scripts/diag_tail.py C2 "L=12,w=12" "L=12,w=12,vis=0" > gpurun_out/diag_sub2.jsonl 2> gpurun_out/diag_sub2.err; echo rc=$?
ALGAS_VIS_DSMEM=0 SUBLAP=1 ALGAS_BUILD_DEFS="-DALGAS_SUBLAP=1" ALGAS_LIB=$PWD/build/libalgas_sublap.so timeout 900 python scripts/diag_tail.py C2 "L=12,w=12" >> gpurun_out/diag_sub2.jsonl 2>> gpurun_out/diag_sub2.err; echo rc=$?
python -c "
import json
for l in open('gpurun_out/diag_sub2.jsonl'):
    d=json.loads(l); print({k:d[k] for k in d if k.startswith('sub') or k in ('variant','qps','cyc_per_step')})
"
