# server poller without the idle-slot scan under load: tests + e2e
set -x
timeout 900 python -m pytest tests/test_search_gpu.py tests/test_abi.py -q -p no:cacheprovider -x -k "server or merge or watchdog" > gpurun_out/pytest_srv2.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_srv2.log
timeout 900 python bench.py --no-cpu --no-sweep --no-ncu > gpurun_out/bench38.json 2> gpurun_out/bench38.err; echo b=$?
python -c "
import json; d=json.loads(open('gpurun_out/bench38.json').read().strip().splitlines()[-1]); print(d['value'], d['latency_us'], d['e2e'])"
