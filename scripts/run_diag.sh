# ad-hoc GPU diagnostics (one gpurun call): C3 bench line
timeout 1500 python bench.py --config C3 --nq 2000 --ctas 1,2,4,8 --threads 512 --width 8,16 > gpurun_out/bench_C3.json 2> gpurun_out/bench_C3.err; echo C3 rc=$?
