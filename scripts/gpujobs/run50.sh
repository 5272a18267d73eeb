# C5s shard: partitioned build with forward rounds (fan 32 x 8, the workload default) vs R35 reverse rounds (fan 16 x 12)
set -x
timeout 1500 python bench.py --config C5s --no-cpu --no-ncu --refine=-16,12 > gpurun_out/bench_C5s_rev.json 2> gpurun_out/bench_C5s_rev.err; echo r=$?
timeout 1500 python bench.py --config C5s --no-cpu --no-ncu > gpurun_out/bench_C5s_fwd.json 2> gpurun_out/bench_C5s_fwd.err; echo f=$?
for f in rev fwd; do python -c "
import json; l=json.loads(open('gpurun_out/bench_C5s_$f.json').read().strip().splitlines()[-1]); c=l['config']
print('$f', l['value'], l['latency_us'], c['itopk'], c['width'], c['recall'], l['work']['setup_s'], l['e2e']['value'])"; done
