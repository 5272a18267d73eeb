# ad-hoc GPU diagnostics (one gpurun call): parity suite + probe
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 600 python scripts/probe_call.py C2 12,12,1,4,1024,1 12,8,1,4,512,1 10,8,1,6,512,1 64,8,1,1,512,0 12,12,1,4,1024,0 > gpurun_out/probe.log 2>&1
