# C2 SHARED parity gap, repeated (bound 0.008 -> north-star 0.005?)
set -x
for i in 1 2; do timeout 900 python -m pytest tests/test_fullsize_gpu.py -q -p no:cacheprovider -s -k "C2_search and True" 2>&1 | grep -E "shared=True|passed|failed"; done
