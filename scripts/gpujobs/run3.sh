set -x
for c in C2 C4 C3; do
timeout 600 python scripts/ab_env.py $c "GM=0" "GM=3" "GM=3,SR=1" "GM=3,SR=2" "GM=3,SR=4" > gpurun_out/ab_env_$c.jsonl 2> gpurun_out/ab_env_$c.err; echo ab_$c=$?
ALGAS_LIB=$PWD/build/libalgas_bw8.so ALGAS_BUILD_DEFS="-DALGAS_DIST_BW1024=8" timeout 600 python scripts/ab_env.py $c "GM=0" > gpurun_out/ab_bw8_$c.jsonl 2> gpurun_out/ab_bw8_$c.err; echo bw8_$c=$?
done
timeout 600 python scripts/probe_call.py C2 12,12,1,4,1024,1 > gpurun_out/probe_C2.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?
