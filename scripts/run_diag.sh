# ad-hoc GPU diagnostics (one gpurun call)
timeout 900 python -m pytest tests/test_search_gpu.py -x -q -k "server or enqueue" > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?; tail -2 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --ctas 4 --threads 1024 --width 12 --visited 1 --no-cpu --no-sweep > gpurun_out/bench_e2e.json 2> gpurun_out/bench_e2e.err; echo bench rc=$?
timeout 900 python bench.py --config C4 --ctas 4 --threads 1024 --width 16 --visited 1 --no-cpu --no-sweep > gpurun_out/bench_e2e_C4.json 2> gpurun_out/bench_e2e_C4.err; echo bench rc=$?
for f in bench_e2e bench_e2e_C4; do python -c "
import json;l=json.load(open('gpurun_out/$f.json'))
print('$f', l['value'], json.dumps(l['latency_us']), json.dumps(l['e2e']))"; done
