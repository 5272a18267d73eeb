# tail/step-count diagnosis at the C2 point
set -x
timeout 900 python scripts/diag_tail.py C2 "L=12,w=12" "L=13,w=8" "L=12,w=12,mi=6" "L=12,w=12,mi=7" "L=12,w=12,mi=8" "L=14,w=14,mi=7" "L=16,w=16,mi=6" "L=12,w=12,S=8" "L=12,w=12,S=128" "L=12,w=12,T=2" "L=12,w=12,T=3" > gpurun_out/diag_tail.jsonl 2> gpurun_out/diag_tail.err; echo rc=$?
cat gpurun_out/diag_tail.jsonl
