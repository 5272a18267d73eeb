# ad-hoc GPU diagnostics (one gpurun call): fixed entry sample
for EF in 0 1; do echo "== ENTRY_FIXED=$EF"; ALGAS_ENTRY_FIXED=$EF timeout 600 python scripts/probe_call.py C2 12,12,1,4,1024,1,32 12,12,1,4,1024,1,256 10,10,1,4,1024,1,256 12,12,1,2,1024,1,256 2>&1 | grep -E "^====|^recall|^latency|^per query"; done > gpurun_out/entry.log
