# server path after the host-state refactor + emulated device on the GPU box; e2e
set -x
timeout 900 python -m pytest tests/test_search_gpu.py tests/test_abi.py tests/test_server_emulated.py -q -p no:cacheprovider -x -k "server or merge or watchdog or emulated or shared" > gpurun_out/pytest_srv3.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_srv3.log
timeout 900 python bench.py --no-cpu --no-sweep --no-ncu > gpurun_out/bench46.json 2> gpurun_out/bench46.err; echo b=$?
python -c "
import json; d=json.loads(open('gpurun_out/bench46.json').read().strip().splitlines()[-1]); print(d['value'], d['latency_us'], d['e2e'], len(json.dumps(d)))"
