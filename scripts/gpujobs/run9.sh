set -x
NCU="ncu --set full --clock-control none --import-source on -k regex:persistent_kernel -c 1 -f"
timeout 900 $NCU -o gpurun_out/prof_C2 python scripts/profile_run.py C2 --nq 10000 --itopk 12 --width 12 --offset 1 --threads 1024 --ctas 4 --slots 32 --visited shared --reps 1 > gpurun_out/prof_C2.log 2>&1; echo p2=$?
timeout 900 $NCU -o gpurun_out/prof_C4 python scripts/profile_run.py C4 --nq 10000 --itopk 112 --width 16 --offset 1 --threads 1024 --ctas 4 --slots 32 --visited shared --reps 1 > gpurun_out/prof_C4.log 2>&1; echo p4=$?
timeout 1200 $NCU -o gpurun_out/prof_C3 python scripts/profile_run.py C3 --nq 4000 --itopk 64 --width 8 --offset 1 --threads 512 --ctas 4 --slots 32 --visited shared --reps 1 > gpurun_out/prof_C3.log 2>&1; echo p3=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_C2.csv python bench.py --steps 2 --warmup 1 --no-cpu --no-sweep --no-e2e --ctas 4 --threads 1024 --width 12 --visited 1 > gpurun_out/launches_C2_run.log 2>&1; echo l2=$?
timeout 1500 python scripts/build_timing.py C2 --clusters 256 --overlap 2 --refine 8 --fan 32 --search-L 12 16 24 32 48 64 96 128 > gpurun_out/build_timing_C2_curve.jsonl 2>gpurun_out/build_timing_C2_curve.err; echo btc=$?
