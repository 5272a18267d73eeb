# merge-phase probes (diagnosis build)
set -x
SUBLAP=2 ALGAS_BUILD_DEFS="-DALGAS_SUBLAP=3" ALGAS_LIB=$PWD/build/libalgas_sublap.so timeout 900 python scripts/diag_tail.py C2 "L=12,w=12" "L=13,w=8" > gpurun_out/diag_merge.jsonl 2> gpurun_out/diag_merge.err; echo rc=$?
python -c "
import json
for l in open('gpurun_out/diag_merge.jsonl'):
    d=json.loads(l); print({k:d[k] for k in d if k.startswith('m_') or k in ('variant','qps','cyc_per_step')})
"
