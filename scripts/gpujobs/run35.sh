# debug: ncu on the cluster-slot persistent kernel without the cooperative attribute
set -x
B="--metrics dram__bytes_read.sum,dram__bytes_write.sum --print-units base --csv --clock-control none -k regex:persistent_kernel -c 1"
P="python scripts/profile_run.py C2 --nq 4000 --itopk 12 --width 12 --offset 1 --ctas 4 --threads 1024 --visited shared --reps 1"
timeout 300 ncu $B $P --slots 32 > gpurun_out/ncu_f.out 2>&1; echo f=$?; grep -E "dram__|ERROR" gpurun_out/ncu_f.out | cut -c150-
timeout 600 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -x -k "shared or server or dynamic" > gpurun_out/pytest_nc.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_nc.log
