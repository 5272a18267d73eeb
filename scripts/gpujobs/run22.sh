# ncu source-level stall attribution of the C2 persistent kernel
set -x
timeout 900 ncu --set full --import-source on --clock-control none -k regex:persistent_kernel -c 1 -f -o gpurun_out/prof_c2 \
  python scripts/profile_run.py C2 --nq 10000 --itopk 12 --width 12 --offset 1 --ctas 4 --threads 1024 --visited shared --slots 32 --reps 1 > gpurun_out/prof_c2.log 2>&1; echo ncu=$?
ncu -i gpurun_out/prof_c2.ncu-rep --page source --csv --print-source cuda > gpurun_out/src_cuda.csv 2> gpurun_out/src_cuda.err; echo s1=$?
ncu -i gpurun_out/prof_c2.ncu-rep --page source --csv --print-source sass > gpurun_out/src_sass.csv 2> gpurun_out/src_sass.err; echo s2=$?
ncu -i gpurun_out/prof_c2.ncu-rep --page raw --csv > gpurun_out/prof_c2_raw.csv 2>/dev/null
ls -la gpurun_out/
gzip -f gpurun_out/src_sass.csv gpurun_out/src_cuda.csv
rm -f gpurun_out/prof_c2.ncu-rep
