# A/B: merge-time graph-row cache (PF bit 512), pass-2 L2 prefetch (bit 1024); exactness with both on
set -x
ALGAS_PREFETCH=1544 timeout 900 python -m pytest tests/test_search_gpu.py -q -p no:cacheprovider -k "lattice_exact or hand_trace or dynamic or wide_ctas or spill" > gpurun_out/pytest_pf.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_pf.log
timeout 900 python scripts/diag_tail.py C2 "L=12,w=12,PF=8" "L=12,w=12,PF=520" "L=12,w=12,PF=1032" "L=12,w=12,PF=1544" "L=13,w=8,PF=8" "L=13,w=8,PF=520" "L=13,w=8,PF=1544" "L=12,w=12,PF=8" "L=12,w=12,PF=520" > gpurun_out/diag_pf.jsonl 2> gpurun_out/diag_pf.err; echo rc=$?
cut -c1-420 gpurun_out/diag_pf.jsonl
