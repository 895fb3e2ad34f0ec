mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "trap or sparse or walk or local_search or sigma" -p no:cacheprovider 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_parity_large.py -q -x -k "cfg4_local_search or cfg4_error_matrix_sigma or cfg5_local_search_to" -p no:cacheprovider 2>&1 | tail -2
REPS=5 timeout 300 python tools/ls_bench.py 3,4 trap 2>&1 | cut -c1-100
timeout 300 python tools/ep_bench.py 5 | tail -1
for c in 4; do timeout 300 python tools/sp_rounds.py $c trap 2>&1 | grep "walk=" | cut -c1-100; done
