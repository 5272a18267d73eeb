# ad-hoc GPU diagnostics (one gpurun call): chunk config 7 (4 lanes x 8 chunks) A/B
timeout 900 python -m pytest tests/test_search_gpu.py -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?; tail -1 gpurun_out/pytest_gpu.log
for CC in 0 7 0 7; do echo "== ALGAS_CC=$CC"; ALGAS_CC=$CC timeout 300 python scripts/probe_call.py C2 12,12,1,4,1024,1 32,8,1,2,1024,1 2>&1 | grep -E "^recall|^latency|^per query"; done > gpurun_out/cc.log 2>&1
