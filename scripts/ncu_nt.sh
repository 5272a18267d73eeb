# ncu captures of the dynamic-batching search kernel at C2 for several thread counts
set -x
for nt in 512 1024; do
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:persistent_kernel -c 1 \
    -o gpurun_out/prof_nt${nt} python scripts/profile_run.py C2 --nq 3000 --itopk 64 --width 8 --threads ${nt} --ctas 1 --slots 32 --reps 1 > gpurun_out/prof_nt${nt}.log 2>&1
  echo "nt=$nt rc=$?"
done
