# two searches per SM: T=6..8 x 512 threads at reduced width / seeds
set -x
timeout 900 python scripts/diag_tail.py C2 "L=10,w=8,T=8,nt=512" "L=10,w=6,T=8,nt=512" "L=10,w=4,T=8,nt=512" "L=10,w=6,T=8,nt=512,S=8" "L=10,w=8,T=7,nt=512" "L=10,w=6,T=7,nt=512" "L=10,w=6,T=6,nt=512" "L=10,w=4,T=6,nt=512" "L=10,w=4,T=16,nt=256" "L=10,w=2,T=16,nt=256" "L=10,w=8,T=9,nt=512" > gpurun_out/diag_t8.jsonl 2> gpurun_out/diag_t8.err; echo rc=$?
cat gpurun_out/diag_t8.jsonl
