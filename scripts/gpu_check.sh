# one GPU call: smoke, parity tests, bench (N=1), launch list + one ncu capture
# of the bench's dominant kernel at the bench's operating point
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 1500 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
head -c 1500 gpurun_out/bench.json
if [ "${NCU:-1}" = "1" ]; then
  OP=$(python -c "import json;l=json.load(open('gpurun_out/bench.json'));c=l['config'];print(c['itopk'],c['width'],c['offset_beam'],c['ctas_per_query'],c['threads_per_cta'],c.get('visited','private'))")
  set -- $OP
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python scripts/profile_run.py C2 --nq 10000 --itopk $1 --width $2 --offset $3 --ctas $4 --threads $5 --visited $6 --slots 32 --reps 2 > gpurun_out/launches_run.log 2>&1
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:persistent_kernel -c 1 \
    -o gpurun_out/prof_op python scripts/profile_run.py C2 --nq 10000 --itopk $1 --width $2 --offset $3 --ctas $4 --threads $5 --visited $6 --slots 32 --reps 1 > gpurun_out/prof_op.log 2>&1
  echo ncu rc=$?
fi
