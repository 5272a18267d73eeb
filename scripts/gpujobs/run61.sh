# final C4 / C3 bench lines with the session's final kernel
set -x
timeout 1800 python bench.py --config C4 > gpurun_out/bench_C4.json 2> gpurun_out/bench_C4.err; echo c4=$?
timeout 1800 python bench.py --config C3 > gpurun_out/bench_C3.json 2> gpurun_out/bench_C3.err; echo c3=$?
for c in C4 C3; do python -c "
import json; l=json.loads(open('gpurun_out/bench_$c.json').read().strip().splitlines()[-1]); c=l['config']
print('$c', l['value'], l['latency_us'], l['e2e']['value'], c['itopk'], c['width'], c['ctas_per_query'], c['threads_per_cta'], c['recall'], l['roofline']['frac'], l['roofline']['traffic'])"; done
