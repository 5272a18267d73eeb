# ad-hoc GPU diagnostics (one gpurun call)
timeout 900 python -m pytest tests/test_search_gpu.py -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/pytest_gpu.log
for PF in 8 8; do echo "== ALGAS_PREFETCH=$PF"; ALGAS_PREFETCH=$PF timeout 300 python scripts/probe_call.py C2 12,12,1,4,1024,1 32,8,1,2,1024,1 2>&1 | grep -E "^recall|^latency|^per query"; done > gpurun_out/fm.log 2>&1
