# ad-hoc GPU diagnostics (one gpurun call)
timeout 900 python bench.py --ctas 4 --threads 1024 --width 12 --visited 1 --no-cpu --no-sweep > gpurun_out/bench_e2e.json 2> gpurun_out/bench_e2e.err; echo bench rc=$?
python -c "
import json;l=json.load(open('gpurun_out/bench_e2e.json'))
print(l['value'], json.dumps(l['latency_us']), json.dumps(l['e2e']))"
