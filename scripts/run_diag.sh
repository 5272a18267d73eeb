# ad-hoc GPU diagnostics (one gpurun call)
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/pytest_gpu.log
for PF in 8 136 8 136; do echo "== ALGAS_PREFETCH=$PF"; ALGAS_PREFETCH=$PF timeout 300 python scripts/probe_call.py C2 12,12,1,4,1024,1 64,8,1,1,512,0 2>&1 | grep -E "^recall|^latency|^per query"; done > gpurun_out/gc.log 2>&1
