# ad-hoc GPU diagnostics (one gpurun call): refresh C3 / C4 bench lines and the f1 ablation
timeout 900 python scripts/ablation.py C2 > gpurun_out/ablation.log 2>&1; echo ablation rc=$?
timeout 1500 python bench.py --config C3 --nq 2000 --ctas 1,2,4,8 --threads 512 --width 8,16 > gpurun_out/bench_C3.json 2> gpurun_out/bench_C3.err; echo C3 rc=$?
timeout 1500 python bench.py --config C4 --ctas 1,2,4,8 --threads 512,1024 --width 8,16 > gpurun_out/bench_C4.json 2> gpurun_out/bench_C4.err; echo C4 rc=$?
