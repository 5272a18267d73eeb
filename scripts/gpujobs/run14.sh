set -x
timeout 600 python -m pytest tests/test_search_gpu.py -q -x -p no:cacheprovider -k "server or watchdog or shared" > gpurun_out/pytest_srv.log 2>&1; echo pytest_rc=$?
timeout 900 python scripts/ab_env.py C2 "PF=8" "PF=264" > gpurun_out/ab_claim_C2.jsonl 2> gpurun_out/ab_claim_C2.err; echo ab2=$?
timeout 900 python scripts/ab_env.py C4 "PF=8" "PF=264" > gpurun_out/ab_claim_C4.jsonl 2> gpurun_out/ab_claim_C4.err; echo ab4=$?
timeout 900 python scripts/ab_env.py C3 "PF=8" "PF=264" > gpurun_out/ab_claim_C3.jsonl 2> gpurun_out/ab_claim_C3.err; echo ab3=$?
timeout 1800 python -m pytest tests/test_fullsize_gpu.py -q -x -s -p no:cacheprovider > gpurun_out/pytest_full.log 2>&1; echo pytest_full=$?
