# compute-sanitizer on the cluster-slot ring path (DSMEM bitmap, cluster barriers, DSMEM push) and the parallel rank merge
set -x
for nt in 256 1024; do
timeout 900 compute-sanitizer --tool racecheck python scripts/sanitize_ring.py $nt > gpurun_out/racecheck_$nt.log 2>&1; echo race_rc=$?
timeout 900 compute-sanitizer --tool synccheck python scripts/sanitize_ring.py $nt > gpurun_out/synccheck_$nt.log 2>&1; echo sync_rc=$?
timeout 900 compute-sanitizer --tool memcheck python scripts/sanitize_ring.py $nt > gpurun_out/memcheck_$nt.log 2>&1; echo mem_rc=$?
done
for f in gpurun_out/*check_*.log; do echo == $f; tail -n 4 $f; done
