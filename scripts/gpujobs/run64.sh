# ncu --set full of the final C4 and C3 persistent kernels (bench operating points)
set -x
timeout 900 ncu --set full --import-source on --clock-control none -k regex:persistent_kernel -c 1 -f -o gpurun_out/prof_c4 \
  python scripts/profile_run.py C4 --nq 10000 --itopk 112 --width 12 --offset 1 --ctas 4 --threads 1024 --visited shared --slots 32 --reps 1 > gpurun_out/prof_c4.log 2>&1; echo c4=$?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:persistent_kernel -c 1 -f -o gpurun_out/prof_c3 \
  python scripts/profile_run.py C3 --nq 10000 --itopk 64 --width 8 --offset 1 --ctas 4 --threads 512 --visited shared --slots 32 --reps 1 > gpurun_out/prof_c3.log 2>&1; echo c3=$?
ls -la gpurun_out/prof_c4.ncu-rep gpurun_out/prof_c3.ncu-rep
