# ad-hoc GPU diagnostics (one gpurun call)
for H in 1 1; do timeout 900 python bench.py --ctas 4 --threads 1024 --width 12 --visited 1 --no-cpu --no-sweep --host-threads $H > gpurun_out/bench_e2e_h$H.json 2> gpurun_out/bench_e2e.err; echo bench rc=$?; python -c "
import json;l=json.load(open('gpurun_out/bench_e2e_h$H.json'))
print($H, l['value'], json.dumps(l['e2e']))"; done
