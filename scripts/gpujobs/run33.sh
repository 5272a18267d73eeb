# debug: ncu dram counters of the persistent kernel (cluster launch) 
set -x
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum --print-units base --csv --clock-control none -k regex:persistent_kernel -c 1 python scripts/profile_run.py C2 --nq 10000 --itopk 12 --width 12 --offset 1 --ctas 4 --threads 1024 --visited shared --slots 32 --reps 1 > gpurun_out/ncu_dbg.out 2> gpurun_out/ncu_dbg.err; echo rc=$?
tail -20 gpurun_out/ncu_dbg.out; tail -5 gpurun_out/ncu_dbg.err
