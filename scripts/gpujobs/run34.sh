# debug: ncu on the cluster-slot persistent kernel
set -x
B="--metrics dram__bytes_read.sum,dram__bytes_write.sum --print-units base --csv --clock-control none -k regex:persistent_kernel -c 1"
P="python scripts/profile_run.py C2 --nq 4000 --itopk 12 --width 12 --offset 1 --ctas 4 --threads 1024 --visited shared --reps 1"
timeout 300 ncu $B --replay-mode application $P --slots 32 > gpurun_out/ncu_a.out 2>&1; echo a=$?; grep -E "dram__|ERROR" gpurun_out/ncu_a.out | cut -c150-
timeout 300 ncu $B $P --slots 24 > gpurun_out/ncu_b.out 2>&1; echo b=$?; grep -E "dram__|ERROR" gpurun_out/ncu_b.out | cut -c150-
timeout 300 ncu $B $P --slots 8 > gpurun_out/ncu_c.out 2>&1; echo c=$?; grep -E "dram__|ERROR" gpurun_out/ncu_c.out | cut -c150-
ALGAS_VIS_DSMEM=0 timeout 300 ncu $B $P --slots 32 > gpurun_out/ncu_d.out 2>&1; echo d=$?; grep -E "dram__|ERROR" gpurun_out/ncu_d.out | cut -c150-
timeout 300 ncu $B python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/ncu_e.out 2>&1; echo e=$?; grep -E "dram__|ERROR|smoke" gpurun_out/ncu_e.out | cut -c1-200
