set -x
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?
for c in C2 C4 C3; do
timeout 900 python scripts/ab_env.py $c "GM=0" > gpurun_out/ab_def_$c.jsonl 2> gpurun_out/ab_def_$c.err; echo def_$c=$?
ALGAS_LIB=$PWD/build/libalgas_bw8.so ALGAS_BUILD_DEFS="-DALGAS_DIST_BW1024=8" timeout 900 python scripts/ab_env.py $c "GM=0" > gpurun_out/ab_bw8_$c.jsonl 2> gpurun_out/ab_bw8_$c.err; echo bw8_$c=$?
ALGAS_LIB=$PWD/build/libalgas_gx.so ALGAS_BUILD_DEFS="-DALGAS_GATHER_EXPERIMENTS=1" timeout 900 python scripts/ab_env.py $c "GM=0" "GM=4" "GM=4,SR=2" > gpurun_out/ab_gx_$c.jsonl 2> gpurun_out/ab_gx_$c.err; echo gx_$c=$?
done
NCU="ncu --set full --clock-control none --import-source on -k regex:persistent_kernel -c 1 -f"
prof() {  # cfg nq params-for-profile_run report-params
  timeout 1200 $NCU -o gpurun_out/prof_$1 python scripts/profile_run.py $1 --nq $2 $3 > gpurun_out/prof_$1.log 2>&1; echo prof_$1=$?
  python scripts/ncu_report.py gpurun_out/prof_$1.ncu-rep --nq $2 --out gpurun_out/round2_$1_ncu.md --traffic gpurun_out/traffic_$1.json --params $4 --title "persistent_kernel at the $1 bench point" > /dev/null 2>gpurun_out/ncu_report_$1.err; echo rep_$1=$?
  rm -f gpurun_out/prof_$1.ncu-rep
}
prof C2 10000 "--itopk 12 --width 12 --offset 1 --threads 1024 --ctas 4 --slots 32 --visited shared --reps 1" itopk=12,width=12,offset_beam=1,ctas_per_query=4,threads_per_cta=1024,slots=32,visited_mode=1
prof C4 10000 "--itopk 112 --width 16 --offset 1 --threads 1024 --ctas 4 --slots 32 --visited shared --reps 1" itopk=112,width=16,offset_beam=1,ctas_per_query=4,threads_per_cta=1024,slots=32,visited_mode=1
prof C3 10000 "--itopk 64 --width 8 --offset 1 --threads 512 --ctas 4 --slots 32 --visited shared --reps 1" itopk=64,width=8,offset_beam=1,ctas_per_query=4,threads_per_cta=512,slots=32,visited_mode=1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_C2.csv python bench.py --steps 2 --warmup 1 --no-cpu --no-sweep --no-e2e --ctas 4 --threads 1024 --width 12 --visited 1 > gpurun_out/launches_C2_run.log 2>&1; echo l2=$?
timeout 1500 python scripts/build_timing.py C2 --clusters 256 --overlap 2 --refine 8 --fan 32 --search-L 12 16 24 32 48 64 96 128 > gpurun_out/build_timing_C2_curve.jsonl 2>gpurun_out/build_timing_C2_curve.err; echo btc=$?
du -sh gpurun_out
