# round-2 refresh: gpu tests, smoke, C2 bench (+ncu traffic), C4/C3 bench, ncu --set full of the C2 kernel, launch list
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
timeout 1500 python bench.py > gpurun_out/bench_C2.json 2> gpurun_out/bench_C2.err; echo c2=$?
timeout 1800 python bench.py --config C4 > gpurun_out/bench_C4.json 2> gpurun_out/bench_C4.err; echo c4=$?
timeout 1800 python bench.py --config C3 > gpurun_out/bench_C3.json 2> gpurun_out/bench_C3.err; echo c3=$?
OP=$(python -c "import json;l=json.loads(open('gpurun_out/bench_C2.json').read().strip().splitlines()[-1]);c=l['config'];print(c['itopk'],c['width'],c['offset_beam'],c['ctas_per_query'],c['threads_per_cta'],c.get('visited','private'))")
set -- $OP
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C2.csv \
  python scripts/profile_run.py C2 --nq 10000 --itopk $1 --width $2 --offset $3 --ctas $4 --threads $5 --visited $6 --slots 32 --reps 2 > gpurun_out/launches_run.log 2>&1; echo launches=$?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:persistent_kernel -c 1 -f -o gpurun_out/prof_c2 \
  python scripts/profile_run.py C2 --nq 10000 --itopk $1 --width $2 --offset $3 --ctas $4 --threads $5 --visited $6 --slots 32 --reps 1 > gpurun_out/prof_c2.log 2>&1; echo ncu=$?
ncu -i gpurun_out/prof_c2.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/src_sass_c2.csv.gz
ls -la gpurun_out/prof_c2.ncu-rep
